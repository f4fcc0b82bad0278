# O(num_chunks) chunk build: GPU suite + plan time + e2e
mkdir -p gpurun_out/c21
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c21/pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c21/pytest.log
SF_PLAN_TRACE=1 timeout 600 python tools/e2e_breakdown.py nell2 > gpurun_out/c21/e2e.txt 2> gpurun_out/c21/trace.txt
cat gpurun_out/c21/e2e.txt; tail -10 gpurun_out/c21/trace.txt
