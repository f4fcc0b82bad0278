# final session-3 bench lines for every config + default bench line + GPU suite + smoke
mkdir -p gpurun_out/c33
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c33/pytest.log 2>&1; echo pytest_exit=$?
tail -2 gpurun_out/c33/pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c33/smoke.log 2>&1; echo smoke_exit=$?
timeout 900 python bench.py > gpurun_out/c33/bench_default.json 2> gpurun_out/c33/bench_default.err; echo bench_exit=$?
for c in vast uber nips enron flickr3d deli3d flickr4d; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > gpurun_out/c33/bench_$c.json 2> gpurun_out/c33/bench_$c.err
done
for c in deli4d nell1; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/c33/bench_$c.json 2> gpurun_out/c33/bench_$c.err
done
for f in gpurun_out/c33/bench_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(round(d['value'],1), round(d['roofline']['frac'],3), (d.get('e2e') or {}).get('value'), [round(v['ms'],3) for v in d['per_mode'].values()])"; done
