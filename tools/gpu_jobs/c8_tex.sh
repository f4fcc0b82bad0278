# SF_LAUNCH_TEX A/B (texture-pipe gathers for the last global slot) + its parity tests
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_frag3.py -x -q > gpurun_out/c8_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c8_pytest.log
for c in nell2 vast nips enron flickr3d nell1; do
  SF_TEX=1 timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c8_tex1_$c.json 2>gpurun_out/c8_tex1_$c.err
  SF_TEX=0 timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c8_tex0_$c.json 2>gpurun_out/c8_tex0_$c.err
done
SF_TEX=1 timeout 600 ncu --set full --clock-control none -k regex:frag3 -s 3 -c 1 -o gpurun_out/c8_ncu_tex_nell2 python bench.py --config nell2 --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c8_ncu.log 2>&1
echo done
