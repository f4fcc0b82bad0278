# RLE features + 160 MB L2-tile floor: GPU suite, e2e, second held-out random set
mkdir -p gpurun_out/c30
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c30/pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c30/pytest.log
timeout 600 python tools/e2e_breakdown.py nell2 > gpurun_out/c30/e2e.txt 2>&1; tail -2 gpurun_out/c30/e2e.txt
timeout 1500 python tools/l2tile_study.py random:12:2 > gpurun_out/c30/l2_random2.jsonl 2> gpurun_out/c30/err.txt; echo study_exit=$?
