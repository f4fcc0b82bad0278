# exhaustive launch sweeps (incl. L2-tiled plans) vs the selector's pick, session-3 build
mkdir -p gpurun_out/c43
timeout 1200 python sweep.py --config nell2 > gpurun_out/c43/sweep_nell2.jsonl 2> gpurun_out/c43/err_nell2.txt
timeout 1500 python sweep.py --config nell1 --quick > gpurun_out/c43/sweep_nell1.jsonl 2> gpurun_out/c43/err_nell1.txt
timeout 1500 python sweep.py --config deli4d --quick > gpurun_out/c43/sweep_deli4d.jsonl 2> gpurun_out/c43/err_deli4d.txt
grep -h summary gpurun_out/c43/sweep_*.jsonl | python -c "
import sys, json
for l in sys.stdin:
    d = json.loads(l); print(d['config'], d['mode'], round(d['pick_ms'],3), round(d['best_ms'],3), round(d['pick_over_best'],3), d['n_launches'])"
