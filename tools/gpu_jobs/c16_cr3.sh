# CR v3 (no per-record sub-range-start compare): nell2 A/B + instruction count
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_frag3.py -x -q > gpurun_out/c16_pytest.log 2>&1; echo pytest_exit=$?
tail -2 gpurun_out/c16_pytest.log
for i in 1 2; do
timeout 600 python bench.py --no-e2e --no-cpu --launch-json @tools/gpu_jobs/cr_nell2.json > gpurun_out/c16_bench_cr_$i.json 2>/dev/null
timeout 600 python bench.py --no-e2e --no-cpu --launch-json @tools/gpu_jobs/nocr_nell2.json > gpurun_out/c16_bench_nocr_$i.json 2>/dev/null
done
for f in gpurun_out/c16_bench_*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['value'], d['roofline']['launch_ms'], d['roofline']['frac'])"; done
timeout 600 ncu --metrics smsp__inst_executed.sum,gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum --clock-control none -k regex:frag3 -s 3 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --launch-json @tools/gpu_jobs/cr_nell2.json 2>/dev/null | grep -E "inst_executed|duration|wavefronts"
