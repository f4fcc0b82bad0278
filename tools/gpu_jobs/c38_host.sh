# cached occupancy / smem opt-in: GPU suite + small-config bench lines
mkdir -p gpurun_out/c38
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c38/pytest.log 2>&1; echo pytest_exit=$?
tail -2 gpurun_out/c38/pytest.log
for c in nell2 uber nips; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/c38/bench_$c.json 2> gpurun_out/c38/bench_$c.err
done
for f in gpurun_out/c38/bench_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(round(d['value'],1), round(d['roofline']['frac'],3), [round(v['ms'],4) for v in d['per_mode'].values()])"; done
