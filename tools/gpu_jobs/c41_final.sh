# final validation of the session: GPU suite (incl. new shard x tiled-plan tests), smoke, default bench
mkdir -p gpurun_out/c41
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c41/pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c41/pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c41/smoke.log 2>&1; echo smoke_exit=$?; cat gpurun_out/c41/smoke.log
timeout 900 python bench.py > gpurun_out/c41/bench.json 2> gpurun_out/c41/bench.err; echo bench_exit=$?
python -c "import json; d=json.load(open('gpurun_out/c41/bench.json')); print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'], d['gpu_launches'])"
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/c41/bench_ref.json 2>&1; echo ref_exit=$?; head -c 300 gpurun_out/c41/bench_ref.json
