mkdir -p gpurun_out/c26
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/c26/launches.csv python tools/cpals_one.py > gpurun_out/c26/log.txt 2>&1
echo done
