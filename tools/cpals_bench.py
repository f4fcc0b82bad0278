"""CP-ALS (F1) timing on B200: time per sweep and the MTTKRP share of it (the paper cites
~90 % for CPD)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_cluster_linwds24_b200 as sf  # noqa: E402

out = {}
for name in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["nell2", "nell1"]):
    cfg = synth.CONFIGS[name]
    inds, vals = synth.config_tensor_device(cfg)
    facs = synth.config_factors_device(cfg)
    with sf.Tensor(cfg.dims, inds, vals) as T:
        del inds, vals
        T.cp_als(facs, iters=1)  # plans + warm-up
        torch.cuda.synchronize()
        iters = 5
        t0 = time.perf_counter()
        fits = T.cp_als(facs, iters=iters)
        torch.cuda.synchronize()
        sweep_ms = (time.perf_counter() - t0) * 1e3 / iters
        # MTTKRP alone, same plans
        ys = [torch.empty((d, cfg.rank), device="cuda") for d in cfg.dims]
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(iters):
            for n in range(cfg.nmodes):
                T.mttkrp(n, facs, ys[n])
        e1.record()
        torch.cuda.synchronize()
        mt_ms = e0.elapsed_time(e1) / iters
    out[name] = {"sweep_ms": sweep_ms, "mttkrp_ms_per_sweep": mt_ms, "mttkrp_share": mt_ms / sweep_ms,
                 "fits": fits, "rank": cfg.rank}
    print(json.dumps({name: out[name]}), flush=True)
json.dump(out, open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "gpurun_out",
                                 "cpals_bench.json"), "w"), indent=1)
