# session-3 bench lines for every config (selector + L2-tile refinement), ncu full capture of
# an L2-tiled nell-1 launch
mkdir -p gpurun_out/c18
for c in nell2 vast uber nips enron flickr3d deli3d flickr4d; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > gpurun_out/c18/bench_$c.json 2> gpurun_out/c18/bench_$c.err
done
for c in deli4d nell1; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/c18/bench_$c.json 2> gpurun_out/c18/bench_$c.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 1 -o gpurun_out/c18/ncu_nell1_l2t python bench.py --config nell1 --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/c18/ncu_nell1.log 2>&1
for f in gpurun_out/c18/bench_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(round(d['value'],1), round(d['roofline']['frac'],3), (d.get('e2e') or {}).get('value'), [round(v['ms'],3) for v in d['per_mode'].values()])"; done
