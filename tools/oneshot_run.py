#!/usr/bin/env python
"""One call of the one-shot path for every mode (sf_mttkrp_streamed_modes) on a config's
pinned host COO -- the workload for an ncu capture of seg_sorted_kernel / the segment sorts:

  ncu --set full -k regex:seg_sorted -c 3 -o prof python tools/oneshot_run.py nell2
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    cfg = synth.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "nell2"]
    segments = int(sys.argv[2]) if len(sys.argv) > 2 else 16
    d_inds, d_vals = synth.config_tensor_device(cfg)
    h_inds = [a.cpu().pin_memory() for a in d_inds]
    h_vals = d_vals.cpu().pin_memory()
    del d_inds, d_vals
    facs = synth.config_factors_device(cfg)
    outs = [torch.empty((d, cfg.rank), device="cuda") for d in cfg.dims]
    t0 = time.perf_counter()
    sf.mttkrp_streamed_modes(cfg.dims, h_inds, h_vals, facs, outs, segments, 4)
    torch.cuda.synchronize()
    print(f"{cfg.name}: one-shot all modes {1e3 * (time.perf_counter() - t0):.1f} ms", flush=True)


if __name__ == "__main__":
    main()
