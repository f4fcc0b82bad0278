# compact records with run deltas (CR v2): GPU suite + nell2 bench A/B
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/c14_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c14_pytest.log
for i in 1 2; do
timeout 600 python bench.py --no-e2e --no-cpu --launch-json @tools/gpu_jobs/cr_nell2.json > gpurun_out/c14_bench_cr_$i.json 2>/dev/null
timeout 600 python bench.py --no-e2e --no-cpu --launch-json @tools/gpu_jobs/nocr_nell2.json > gpurun_out/c14_bench_nocr_$i.json 2>/dev/null
done
for f in gpurun_out/c14_bench_*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['value'], d['roofline']['launch_ms'], d['roofline']['frac'])"; done
