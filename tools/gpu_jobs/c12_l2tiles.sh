# L2-tiled schedule: parity tests touched by it, then the study on the hyper-sparse configs
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/c12_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c12_pytest.log
timeout 1500 python tools/l2tile_study.py nell1,amazon,deli4d > gpurun_out/c12_l2tiles.jsonl 2> gpurun_out/c12_l2tiles.err; echo study_exit=$?
cat gpurun_out/c12_l2tiles.jsonl | cut -c1-250
tail -3 gpurun_out/c12_l2tiles.err
