# full GPU suite after presort v2 + StepExchange; smoke; default bench line
mkdir -p gpurun_out/c24
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c24/pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c24/pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c24/smoke.log 2>&1; echo smoke_exit=$?; cat gpurun_out/c24/smoke.log
timeout 900 python bench.py > gpurun_out/c24/bench.json 2> gpurun_out/c24/bench.err; echo bench_exit=$?
python -c "import json; d=json.load(open('gpurun_out/c24/bench.json')); print(d['value'], d['roofline']['frac'], d['e2e'], d['plan_step'], d['cpu_baseline'])"
timeout 600 python tools/cpals_bench.py > gpurun_out/c24/cpals.txt 2>&1; tail -5 gpurun_out/c24/cpals.txt
