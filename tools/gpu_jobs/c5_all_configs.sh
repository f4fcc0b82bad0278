# frag3 (default) vs the round-1 SoA kernel (SF_FRAG_IMPL=2) on every synthetic config, + the GPU suite
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/c5_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c5_pytest.log
for c in nell2 vast uber nips enron flickr3d deli3d flickr4d deli4d nell1; do
  timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c5_f3_$c.json 2>gpurun_out/c5_f3_$c.err
  SF_FRAG_IMPL=2 timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c5_f2_$c.json 2>gpurun_out/c5_f2_$c.err
done
echo done
