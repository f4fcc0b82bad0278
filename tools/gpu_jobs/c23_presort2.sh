# presort v2 (key-bit-only segment sorts, AoS per segment): presort tests + e2e A/B
mkdir -p gpurun_out/c23
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "presort or host_inputs or plan_bit_exact" > gpurun_out/c23/pytest_presort.log 2>&1; echo pytest_presort_exit=$?
tail -2 gpurun_out/c23/pytest_presort.log
for i in 1 2; do
timeout 600 python tools/e2e_breakdown.py nell2 > gpurun_out/c23/e2e_on_$i.txt 2>&1
SF_PRESORT=0 timeout 600 python tools/e2e_breakdown.py nell2 > gpurun_out/c23/e2e_off_$i.txt 2>&1
done
tail -n 2 gpurun_out/c23/e2e_*.txt
