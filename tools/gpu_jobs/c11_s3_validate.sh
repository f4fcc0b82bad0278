# session-3 start: validate HEAD (planner tile-key change) -- GPU suite, smoke, default bench line
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c11_build.log 2>&1; echo build_exit=$?
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/c11_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c11_pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c11_smoke.log 2>&1; echo smoke_exit=$?
timeout 900 python bench.py > gpurun_out/c11_bench.json 2> gpurun_out/c11_bench.err; echo bench_exit=$?
cat gpurun_out/c11_bench.json | head -c 600
echo done
