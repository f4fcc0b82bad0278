# quick sweeps of the Table III shapes with tiny-output modes: shared-memory block staging vs L2 tiles
mkdir -p gpurun_out/c45
for c in flickr4d deli3d flickr3d; do
  timeout 1200 python sweep.py --config $c --quick > gpurun_out/c45/sweep_$c.jsonl 2> gpurun_out/c45/err_$c.txt
done
grep -h summary gpurun_out/c45/sweep_*.jsonl | python -c "
import sys, json
for l in sys.stdin:
    d = json.loads(l); print(d['config'], d['mode'], round(d['pick_ms'],3), round(d['best_ms'],3), round(d['pick_over_best'],3), d['best'].get('staged'), d['best'].get('flags'))"
