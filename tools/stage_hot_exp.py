#!/usr/bin/env python
"""Experiment: shared-memory staging of a small gathered factor COMBINED with the hot-row
cache for the large ones (deli-4d modes 0-2 gather the 1,443-row mode-3 factor on every
nonzero: staging it removes a third of the L2 gather traffic).  Prints one JSON line per
launch: config, mode, launch, ms (10 launches, CUDA events)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    name = sys.argv[1] if len(sys.argv) > 1 else "deli4d"
    cfg = synth.CONFIGS[name]
    R, N = cfg.rank, cfg.nmodes
    facs = synth.config_factors_device(cfg)
    inds, vals = synth.config_tensor_device(cfg)
    T = sf.Tensor(cfg.dims, inds, vals)
    del inds, vals
    torch.cuda.empty_cache()
    s = torch.cuda.Stream()
    small = min(range(N), key=lambda m: cfg.dims[m])
    for n in range(N):
        if n == small:
            continue
        out = torch.empty((cfg.dims[n], R), device="cuda")
        T.plan(n, R)
        pick = T.plan_info(n, R)["launch"]
        launches = [("pick", None)]
        for br in (256, 512, 768, cfg.dims[small]):
            for th in (512, 1024):
                for ch in (64, 128):
                    for hot in (0, 32):
                        launches.append((f"stage{small}:{br} th{th} ch{ch} hot{hot}",
                                         sf.Launch.make(kernel=sf.KERNEL_FRAG, block_threads=th, chunk_nnz=ch,
                                                        staged={small: br}, hot_kb=hot * 1024)))
        for label, L in launches:
            try:
                if L is None:
                    T.plan(n, R)
                else:
                    T.set_launch(n, R, L)
            except sf.SfError as e:
                print(json.dumps({"config": name, "mode": n, "launch": label, "err": str(e)}), flush=True)
                continue
            for _ in range(3):
                T.mttkrp(n, facs, out, stream=s)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(10):
                T.mttkrp(n, facs, out, stream=s)
            e1.record(s)
            torch.cuda.synchronize()
            print(json.dumps({"config": name, "mode": n, "launch": label, "ms": round(e0.elapsed_time(e1) / 10, 4),
                              "pick": pick if L is None else None}), flush=True)
        T.plan_release(n, R)
    T.close()


if __name__ == "__main__":
    main()
