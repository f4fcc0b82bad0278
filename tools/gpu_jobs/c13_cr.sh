# compact 8-byte records (CR): GPU suite, nell2 bench A/B (CR vs NO_COMPACT, same launches),
# row-frequency histograms and the L2-tile study over every config
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/c13_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c13_pytest.log
for i in 1 2; do
timeout 600 python bench.py --no-e2e --no-cpu --launch-json @tools/gpu_jobs/cr_nell2.json > gpurun_out/c13_bench_cr_$i.json 2>/dev/null
timeout 600 python bench.py --no-e2e --no-cpu --launch-json @tools/gpu_jobs/nocr_nell2.json > gpurun_out/c13_bench_nocr_$i.json 2>/dev/null
done
for f in gpurun_out/c13_bench_*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['value'], d['roofline']['launch_ms'], d['roofline']['frac'])"; done
timeout 900 python tools/row_freq_dump.py nell2,deli4d,nell1,amazon,vast,flickr3d,deli3d,uber,nips,enron,flickr4d > gpurun_out/c13_rowfreq.jsonl 2> gpurun_out/c13_rowfreq.err; echo rowfreq_exit=$?
timeout 1500 python tools/l2tile_study.py nell2,vast,flickr3d,deli3d,uber,nips,enron,flickr4d,amazon > gpurun_out/c13_l2tiles.jsonl 2> gpurun_out/c13_l2tiles.err; echo study_exit=$?
tail -2 gpurun_out/c13_l2tiles.err
