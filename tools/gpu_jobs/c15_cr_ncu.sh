# CR vs plain records: ncu full capture of one nell2 mode-0 launch each; L2-tile refinement
# default picks on the hyper-sparse configs (bench lines)
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 1 -o gpurun_out/c15_cr python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --launch-json @tools/gpu_jobs/cr_nell2.json > gpurun_out/c15_cr.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 1 -o gpurun_out/c15_nocr python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --launch-json @tools/gpu_jobs/nocr_nell2.json > gpurun_out/c15_nocr.log 2>&1
for c in nell1 deli4d amazon; do
timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/c15_bench_$c.json 2> gpurun_out/c15_bench_$c.err
SF_L2_TILES=0 timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/c15_bench_${c}_nol2.json 2>> gpurun_out/c15_bench_$c.err
done
for f in gpurun_out/c15_bench_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(round(d['value'],1), round(d['ms_per_step'],3), {k: (round(v['ms'],3), v['launch']['staged_mask'], v['launch']['flags']) for k, v in d['per_mode'].items()})"; done
ls -la gpurun_out/c15_*
