#!/usr/bin/env python
"""Plan-time profile: create a config's tensor on the device, then plan every mode twice
(the second time warm, after sf_plan_release); prints wall and device (plan_ms) per plan.
Run under `ncu --metrics gpu__time_duration.sum` for the per-kernel launch list."""
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
    d_inds, d_vals = synth.config_tensor_device(cfg)
    T = sf.Tensor(cfg.dims, d_inds, d_vals)
    torch.cuda.synchronize()
    for rep in range(2):
        for n in range(cfg.nmodes):
            t0 = time.perf_counter()
            T.plan(n, cfg.rank)
            torch.cuda.synchronize()
            wall = (time.perf_counter() - t0) * 1e3
            print(f"rep {rep} mode {n}: wall {wall:.2f} ms, device {T.plan_info(n, cfg.rank)['plan_ms']:.2f} ms",
                  flush=True)
        for n in range(cfg.nmodes):
            T.plan_release(n, cfg.rank)
    T.close()


if __name__ == "__main__":
    main()
