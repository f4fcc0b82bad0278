#!/usr/bin/env python
"""Time one mode of a config under several explicit launches (one plan each, released after),
for A/B experiments and targeted ncu captures (`ncu --metrics ... python tools/launch_variants.py`).

  python tools/launch_variants.py amazon 2 @variants.json [reps]

variants.json: {"name": {launch dict as bench.py --launch-json takes}, ...}; "auto" = the selector.
Prints one JSON line per variant: ms (mean of reps event-timed launches), the launch, tiles.
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    torch.cuda.init()
    l2f = os.environ.get("L2FETCH")  # experiment: cudaLimitMaxL2FetchGranularity (bytes)
    if l2f is not None:
        import ctypes
        import glob
        so = glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                    "libcudart.so*"))[0]
        rt = ctypes.CDLL(so)
        torch.zeros(1, device="cuda")
        rc = rt.cudaDeviceSetLimit(5, ctypes.c_size_t(int(l2f)))
        v = ctypes.c_size_t(0)
        rt.cudaDeviceGetLimit(ctypes.byref(v), 5)
        print(json.dumps({"l2_fetch_granularity_set": int(l2f), "rc": rc, "now": v.value}), flush=True)
    cfg = synth.CONFIGS[sys.argv[1]]
    n = int(sys.argv[2])
    src = sys.argv[3]
    variants = json.load(open(src[1:])) if src.startswith("@") else json.loads(src)
    reps = int(sys.argv[4]) if len(sys.argv) > 4 else 5
    R = cfg.rank
    inds, vals = synth.config_tensor_device(cfg)
    facs = synth.config_factors_device(cfg)
    T = sf.Tensor(cfg.dims, inds, vals)
    del inds, vals
    torch.cuda.empty_cache()
    out = torch.empty((cfg.dims[n], R), device="cuda")
    for name, d in variants.items():
        if d == "auto":
            T.plan(n, R)
        else:
            d = dict(d)
            if "staged" in d:
                d["staged"] = {int(k): int(v) for k, v in d["staged"].items()}
            T.set_launch(n, R, sf.Launch.make(**d))
        info = T.plan_info(n, R)
        T.mttkrp(n, facs, out)  # warm-up
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
        for a, b in ev:
            a.record()
            T.mttkrp(n, facs, out)
            b.record()
        torch.cuda.synchronize()
        ms = statistics.mean(a.elapsed_time(b) for a, b in ev)
        print(json.dumps({"config": cfg.name, "mode": n, "variant": name, "ms": ms, "launch": info["launch"],
                          "num_tiles": info["num_tiles"]}), flush=True)
        T.plan_release(n, R)
        torch.cuda.empty_cache()
    T.close()


if __name__ == "__main__":
    main()
