# session-3 profile artifacts: launch list of the bench command, full capture of the top kernel
mkdir -p gpurun_out/c28
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c28/launches_nell2.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/c28/launches.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 1 -o gpurun_out/c28/ncu_full_nell2 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c28/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:frag3 -s 2 -c 1 -o gpurun_out/c28/ncu_full_deli4d python bench.py --config deli4d --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c28/ncu_deli.log 2>&1
ls -la gpurun_out/c28
