# (1) texture vs LSU gather micro, (2) R=16 lane map VEC=8 A/B (SF_LIB_PATH), (3) deli4d mode-3 ncu f3 vs f2
mkdir -p gpurun_out
./tools/micro/tex_vs_ldg > gpurun_out/c6_tex_vs_ldg.txt 2>&1
V8=$PWD/paper_conf_cluster_linwds24_b200/libscalfrag_r16v8.so
SF_LIB_PATH=$V8 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_frag3.py tests/test_gpu_table3.py -x -q > gpurun_out/c6_pytest_r16v8.log 2>&1; echo pytest_r16v8_exit=$?
for c in vast uber nips enron flickr3d deli3d flickr4d; do
  SF_LIB_PATH=$V8 timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c6_v8_$c.json 2>gpurun_out/c6_v8_$c.err
  timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c6_v4_$c.json 2>gpurun_out/c6_v4_$c.err
done
timeout 900 ncu --set full --clock-control none -k regex:frag -s 7 -c 1 -o gpurun_out/c6_ncu_deli4d_m3_f3 python bench.py --config deli4d --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c6_ncu_f3.log 2>&1
SF_FRAG_IMPL=2 timeout 900 ncu --set full --clock-control none -k regex:frag -s 7 -c 1 -o gpurun_out/c6_ncu_deli4d_m3_f2 python bench.py --config deli4d --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c6_ncu_f2.log 2>&1
echo done
