#!/usr/bin/env python
"""Timeline of bench.py's end-to-end step (the overlapped user pipeline over the public API):
host timestamps after every call and CUDA-event times on the upload / compute / D2H streams.

  python tools/e2e_trace.py [nell1]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    cfg = synth.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "nell1"]
    N, R = cfg.nmodes, cfg.rank
    dev = torch.device("cuda", 0)
    d_inds, d_vals = synth.config_tensor_device(cfg)
    h_inds = [a.cpu().pin_memory() for a in d_inds]
    h_vals = d_vals.cpu().pin_memory()
    del d_inds, d_vals
    h_facs = [f.cpu().pin_memory() for f in synth.config_factors_device(cfg)]
    h_out = [torch.empty((cfg.dims[n], R), dtype=torch.float32).pin_memory() for n in range(N)]
    df = [torch.empty_like(f, device=dev) for f in h_facs]
    stream, h2d_s, d2h_s = (torch.cuda.Stream(device=dev) for _ in range(3))
    order = sorted(range(N), key=lambda n: -cfg.dims[n])
    up_order = [m for m in range(N) if m != order[0]] + [order[0]]
    for rep in range(3):
        torch.cuda.synchronize()
        marks = []
        t0 = time.perf_counter()
        base = torch.cuda.Event(enable_timing=True)
        base.record(torch.cuda.current_stream())

        def mark(name):
            marks.append((name, round((time.perf_counter() - t0) * 1e3, 2)))

        evs = {}

        def ev(name, s):
            e = torch.cuda.Event(enable_timing=True)
            e.record(s)
            evs[name] = e

        T2 = sf.Tensor(cfg.dims, h_inds, h_vals)
        mark("create")
        ev_f = {}
        with torch.cuda.stream(h2d_s):
            for m in up_order:
                df[m].copy_(h_facs[m], non_blocking=True)
                ev_f[m] = torch.cuda.Event(enable_timing=True)
                ev_f[m].record(h2d_s)
        mark("factor copies issued")
        for n in order:
            T2.plan(n, R)
            mark(f"plan {n}")
            o = torch.empty((cfg.dims[n], R), dtype=torch.float32, device=dev)
            for m in range(N):
                if m != n:
                    stream.wait_event(ev_f[m])
            ev(f"mttkrp {n} start", stream)
            T2.mttkrp(n, df, o, stream=stream)
            ev(f"mttkrp {n} end", stream)
            d2h_s.wait_stream(stream)
            with torch.cuda.stream(d2h_s):
                h_out[n].copy_(o, non_blocking=True)
                o.record_stream(d2h_s)
            ev(f"d2h {n} end", d2h_s)
            mark(f"mttkrp {n} issued")
        torch.cuda.synchronize()
        mark("synced")
        T2.close()
        mark("closed")
        gpu = {k: round(base.elapsed_time(e), 2) for k, e in evs.items()}
        gpu.update({f"factor {m} uploaded": round(base.elapsed_time(e), 2) for m, e in ev_f.items()})
        print(json.dumps({"rep": rep, "host_ms": marks, "gpu_ms": dict(sorted(gpu.items(), key=lambda kv: kv[1]))}),
              flush=True)


if __name__ == "__main__":
    main()
