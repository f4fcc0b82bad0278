# default path after making CR opt-in + L2-tile refinement: GPU suite + smoke + nell2 bench
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c17_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c17_pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c17_smoke.log 2>&1; echo smoke_exit=$?
timeout 900 python bench.py > gpurun_out/c17_bench.json 2> gpurun_out/c17_bench.err; echo bench_exit=$?
python -c "import json; d=json.load(open('gpurun_out/c17_bench.json')); print(d['value'], d['roofline'], d['e2e']['value'])"
