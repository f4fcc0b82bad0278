"""Where does the end-to-end time go? (create / factor H2D / plan per mode / mttkrp / D2H)"""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import synth
import paper_conf_cluster_linwds24_b200 as sf

cfg = synth.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "nell2"]
inds, vals = synth.config_tensor(cfg)
h_inds = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
h_vals = torch.from_numpy(vals).pin_memory()
h_facs = [torch.from_numpy(f).pin_memory() for f in synth.config_factors(cfg)]
R = cfg.rank
for rep in range(3):
    torch.cuda.synchronize()
    t = {}
    t0 = time.perf_counter()
    T = sf.Tensor(cfg.dims, h_inds, h_vals)
    torch.cuda.synchronize(); t["create"] = time.perf_counter() - t0
    t0 = time.perf_counter()
    df = [f.cuda(non_blocking=True) for f in h_facs]
    torch.cuda.synchronize(); t["factors_h2d"] = time.perf_counter() - t0
    for n in range(cfg.nmodes):
        t0 = time.perf_counter(); T.plan(n, R); torch.cuda.synchronize(); t[f"plan{n}"] = time.perf_counter() - t0
        t[f"plan{n}_dev_ms"] = T.plan_info(n, R)["plan_ms"] / 1e3
    outs = []
    t0 = time.perf_counter()
    for n in range(cfg.nmodes):
        o = torch.empty((cfg.dims[n], R), device="cuda"); T.mttkrp(n, df, o); outs.append(o)
    torch.cuda.synchronize(); t["mttkrp"] = time.perf_counter() - t0
    t0 = time.perf_counter()
    hs = [o.cpu() for o in outs]
    t["d2h"] = time.perf_counter() - t0
    t0 = time.perf_counter(); T.close(); torch.cuda.synchronize(); t["destroy"] = time.perf_counter() - t0
    print({k: round(v * 1e3, 2) for k, v in t.items()}, "total ms", round(sum(v for k, v in t.items() if not k.endswith("dev_ms")) * 1e3, 1))
