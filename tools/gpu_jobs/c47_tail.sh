# presort with a 3:1-split last segment: presort/host/shard tests + e2e
mkdir -p gpurun_out/c47
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "presort or host_inputs or shards or plan_bit_exact" > gpurun_out/c47/pytest.log 2>&1; echo pytest_exit=$?
tail -2 gpurun_out/c47/pytest.log
for i in 1 2; do timeout 600 python bench.py --no-cpu --steps 5 --warmup 3 > gpurun_out/c47/b$i.json 2>/dev/null; python -c "import json; d=json.load(open('gpurun_out/c47/b$i.json')); print(d['value'], d['e2e']['ms_per_step'])"; done
timeout 600 python tools/e2e_breakdown.py nell2 | tail -2
