# plan host-phase trace (nell2, warm e2e-like sequence) + vast CR A/B
mkdir -p gpurun_out/c20
SF_PLAN_TRACE=1 timeout 600 python tools/e2e_breakdown.py nell2 > gpurun_out/c20/e2e.txt 2> gpurun_out/c20/trace.txt
cat gpurun_out/c20/e2e.txt; tail -40 gpurun_out/c20/trace.txt
for i in 1 2; do
timeout 600 python bench.py --config vast --no-e2e --no-cpu --launch-json @tools/gpu_jobs/base_vast.json > gpurun_out/c20/vast_base_$i.json 2>/dev/null
timeout 600 python bench.py --config vast --no-e2e --no-cpu --launch-json @tools/gpu_jobs/cr_vast.json > gpurun_out/c20/vast_cr_$i.json 2>/dev/null
done
for f in gpurun_out/c20/vast_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(round(d['value'],1), [round(v['ms'],4) for v in d['per_mode'].values()])"; done
