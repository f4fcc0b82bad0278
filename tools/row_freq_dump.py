#!/usr/bin/env python
"""Per-mode row-frequency histograms of the synthetic configs (for the L2-tile cost model):
for every mode m, log2 bins b of the per-row nonzero count c (c in [2^b, 2^(b+1))):
rows[b] and nnz[b].  One JSON line per config.  usage: row_freq_dump.py nell1,amazon"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    import torch
    for name in sys.argv[1].split(","):
        cfg = synth.CONFIGS[name]
        d_inds, d_vals = synth.config_tensor_device(cfg)
        del d_vals
        modes = []
        for m in range(cfg.nmodes):
            c = torch.bincount(d_inds[m].view(torch.int32).long(), minlength=cfg.dims[m])
            c = c[c > 0]
            b = torch.floor(torch.log2(c.double())).long()
            rows = torch.bincount(b, minlength=40)[:40].tolist()
            nnz = torch.bincount(b, weights=c.double(), minlength=40)[:40].tolist()
            modes.append({"rows": rows, "nnz": [int(x) for x in nnz]})
            del c, b
        print(json.dumps({"config": name, "dims": list(cfg.dims), "nnz": cfg.nnz, "rank": cfg.rank,
                          "modes": modes}), flush=True)
        del d_inds
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
