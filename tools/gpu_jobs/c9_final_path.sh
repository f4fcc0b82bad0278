# frag3-only build: GPU suite, default bench line, ncu launch list + full capture of the top kernel
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/c9_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c9_pytest.log
timeout 900 python bench.py > gpurun_out/c9_bench.json 2> gpurun_out/c9_bench.err; echo bench_exit=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c9_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/c9_launches.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 3 -o gpurun_out/c9_ncu_full_nell2 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c9_ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:frag3 -s 3 -c 3 -o gpurun_out/c9_ncu_full_nell1 python bench.py --config nell1 --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c9_ncu_full_nell1.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c9_smoke.log 2>&1; echo smoke_exit=$?
echo done
