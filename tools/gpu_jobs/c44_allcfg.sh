# end-of-session bench lines for every config (BASELINE.md §4a refresh)
mkdir -p gpurun_out/c44
for c in nell2 vast uber nips enron flickr3d deli3d flickr4d; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > gpurun_out/c44/bench_$c.json 2> gpurun_out/c44/bench_$c.err
done
for c in deli4d nell1; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/c44/bench_$c.json 2> gpurun_out/c44/bench_$c.err
done
timeout 900 python tools/amazon_bench.py > gpurun_out/c44/amazon_1gpu.json 2> gpurun_out/c44/amazon.err
for f in gpurun_out/c44/bench_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(round(d['value'],1), round(d['roofline']['frac'],3), (d.get('e2e') or {}).get('value'), [round(v['ms'],3) for v in d['per_mode'].values()])"; done
head -c 300 gpurun_out/c44/amazon_1gpu.json
