#!/bin/bash
# Run on the GPU box (via gpurun): bench line, ncu launch list and one full ncu capture
# of the dominant kernel.  Outputs land in gpurun_out/; summarise here with
# tools/ncu_summary.py and copy the summaries into profiles/.
set -x
TAG=${1:-r01}
CFG=${2:-nell2}
python bench.py --config $CFG --steps 20 --warmup 5 > gpurun_out/bench_${TAG}_${CFG}.json 2> gpurun_out/bench_${TAG}_${CFG}.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_${CFG}.csv \
    python bench.py --config $CFG --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:frag3 -s 3 -c 3 \
    -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
ls -la gpurun_out/
