# plan-time profile (nell2): wall/device per plan, and the per-kernel launch list under ncu
mkdir -p gpurun_out/c19
timeout 600 python tools/plan_profile.py nell2 > gpurun_out/c19/plan_wall.txt 2>&1
cat gpurun_out/c19/plan_wall.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/c19/plan_launches.csv python tools/plan_profile.py nell2 > /dev/null 2>&1
python tools/e2e_breakdown.py nell2 > gpurun_out/c19/e2e_breakdown.txt 2>&1; cat gpurun_out/c19/e2e_breakdown.txt
