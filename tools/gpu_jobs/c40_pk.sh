# branch-free packed-field decode: 4-way configs A/B (bench lines) + parity subset
mkdir -p gpurun_out/c40
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_table3.py -x -q > gpurun_out/c40/pytest.log 2>&1; echo pytest_exit=$?
tail -2 gpurun_out/c40/pytest.log
for c in deli4d enron nips uber flickr4d; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/c40/bench_$c.json 2> gpurun_out/c40/bench_$c.err
done
for f in gpurun_out/c40/bench_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(round(d['value'],1), [round(v['ms'],4) for v in d['per_mode'].values()])"; done
