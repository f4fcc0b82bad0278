# L2 prefetch of the next stage's rows (SF_LAUNCH_PREFETCH) for unstaged / L2-tiled plans: A/B via launch-json
mkdir -p gpurun_out/c46
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "launch_variants or ranks_and_orders" > gpurun_out/c46/pytest.log 2>&1; echo pytest_exit=$?
tail -2 gpurun_out/c46/pytest.log
python - <<'PY'
import json, subprocess, sys
for cfg in ["nell1", "deli4d", "flickr3d"]:
    d = json.load(open(f"profiles/r01s3/bench_final/bench_{cfg}.json"))
    base, pf = {}, {}
    for k, v in d["per_mode"].items():
        L = v["launch"]
        st = {str(m): r for m, r in enumerate(L["block_rows"]) if L["staged_mask"] >> m & 1}
        e = {"kernel": 2, "block_threads": L["block_threads"], "chunk_nnz": L["chunk_nnz"], "staged": st, "flags": L["flags"]}
        base[k] = e
        pf[k] = dict(e, flags=L["flags"] | 256)
    json.dump(base, open(f"gpurun_out/c46/base_{cfg}.json", "w"))
    json.dump(pf, open(f"gpurun_out/c46/pf_{cfg}.json", "w"))
PY
for c in nell1 deli4d flickr3d; do
  for v in base pf base pf; do
    timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --no-e2e --launch-json @gpurun_out/c46/${v}_$c.json > gpurun_out/c46/b_${c}_$v.json 2>/dev/null
    python -c "import json; d=json.load(open('gpurun_out/c46/b_${c}_$v.json')); print('$c $v', round(d['value'],1), [round(x['ms'],3) for x in d['per_mode'].values()])"
  done
done
