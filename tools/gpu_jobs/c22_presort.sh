# upload || presort: new test + GPU suite, e2e A/B (SF_PRESORT=1/0)
mkdir -p gpurun_out/c22
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "presort or host_inputs or plan_bit_exact" > gpurun_out/c22/pytest_presort.log 2>&1; echo pytest_presort_exit=$?
tail -3 gpurun_out/c22/pytest_presort.log
SF_PLAN_TRACE=1 timeout 600 python tools/e2e_breakdown.py nell2 > gpurun_out/c22/e2e_on.txt 2> gpurun_out/c22/trace_on.txt
SF_PRESORT=0 timeout 600 python tools/e2e_breakdown.py nell2 > gpurun_out/c22/e2e_off.txt 2>&1
cat gpurun_out/c22/e2e_on.txt gpurun_out/c22/e2e_off.txt; tail -12 gpurun_out/c22/trace_on.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c22/pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c22/pytest.log
