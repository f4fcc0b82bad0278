# register-tiled Gram / M V^+ kernels for CP-ALS: CP-ALS tests + timing
mkdir -p gpurun_out/c25
timeout 900 python -m pytest tests/test_gpu_cpals.py -x -q > gpurun_out/c25/pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c25/pytest.log
timeout 600 python tools/cpals_bench.py nell2,nell1,deli4d > gpurun_out/c25/cpals.txt 2>&1; tail -5 gpurun_out/c25/cpals.txt
