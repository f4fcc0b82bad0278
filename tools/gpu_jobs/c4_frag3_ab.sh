mkdir -p gpurun_out
set -x
timeout 900 python -m pytest tests/test_gpu_frag3.py -x -q > gpurun_out/c4_pytest_frag3.log 2>&1; echo pytest_exit=$?
tail -15 gpurun_out/c4_pytest_frag3.log
for c in nell2 nell1; do
  for v in "SF_FIBER=0 SF_L2_HINTS=0" "SF_FIBER=1 SF_L2_HINTS=0" "SF_FIBER=0 SF_L2_HINTS=1" "SF_FIBER=1 SF_L2_HINTS=1"; do
    tag=$(echo $v | tr -d ' =_')
    env $v timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c4_${c}_${tag}.json 2>gpurun_out/c4_${c}_${tag}.err
  done
done
SF_FIBER=0 timeout 600 ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 1 -o gpurun_out/ncu_f3_nell2 python bench.py --config nell2 --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_f3_nell2.log 2>&1
SF_FIBER=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 1 -o gpurun_out/ncu_f3fib_nell2 python bench.py --config nell2 --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_f3fib_nell2.log 2>&1
echo done
