#!/usr/bin/env python
"""GPU timeline of the end-to-end path's planning (sf_tensor_create from pinned host COO, then
sf_plan of every mode, largest-Y first, as bench.py's e2e leg does), recorded with the CUDA
profiler interface of torch.profiler (CUPTI sees every kernel and copy in the process,
including libscalfrag's).  Prints, per plan window (host marks), the busy GPU time per kernel
name, the idle gaps and the total, as JSON lines.

  python tools/plan_timeline.py nell2 [--out gpurun_out/plan_trace.json]
"""
import argparse
import collections
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="nell2")
    ap.add_argument("--out", default=None, help="also write the chrome trace here")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--release", action="store_true", help="release each plan after building it (amazon)")
    args = ap.parse_args()
    import torch
    from torch.profiler import ProfilerActivity, profile

    import paper_conf_cluster_linwds24_b200 as sf
    cfg = synth.CONFIGS[args.config]
    N, R = cfg.nmodes, cfg.rank
    d_inds, d_vals = synth.config_tensor_device(cfg)
    h_inds = [a.cpu().pin_memory() for a in d_inds]
    h_vals = d_vals.cpu().pin_memory()
    del d_inds, d_vals
    torch.cuda.empty_cache()
    order = sorted(range(N), key=lambda n: -cfg.dims[n])

    def one(marks, t0):
        T = sf.Tensor(cfg.dims, h_inds, h_vals)
        torch.cuda.synchronize()
        marks.append(("create", time.perf_counter() - t0))
        for n in order:
            T.plan(n, R)
            torch.cuda.synchronize()
            marks.append((f"plan {n}", time.perf_counter() - t0))
            if args.release:
                T.plan_release(n, R)
        T.close()

    one([], time.perf_counter())  # warm-up (module load, allocator)
    for rep in range(args.reps):
        marks = []
        with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
            t0 = time.perf_counter()
            one(marks, t0)
        if args.out and rep == args.reps - 1:
            os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
            prof.export_chrome_trace(args.out)
        evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
        # kernel / memcpy intervals in microseconds on the profiler's clock
        iv = sorted((e.time_range.start, e.time_range.end, e.name) for e in evs)
        if not iv:
            print(json.dumps({"error": "no CUDA events recorded"}))
            return
        g0 = iv[0][0]
        # window boundaries: host marks are on perf_counter; align the first GPU event with
        # the create window start (upload starts right away)
        wins, prev = [], 0.0
        for name, t in marks:
            wins.append((name, prev * 1e6, t * 1e6))
            prev = t
        total_host = marks[-1][1] * 1e3
        for name, a, b in wins:
            by = collections.Counter()
            union, cur = 0.0, None
            for s, e, k in iv:
                s0, e0 = s - g0, e - g0
                if e0 <= a or s0 >= b:
                    continue
                s1, e1 = max(s0, a), min(e0, b)
                by[k[:70]] += (e1 - s1)
                if cur is None or s1 > cur[1]:
                    if cur is not None:
                        union += cur[1] - cur[0]
                    cur = [s1, e1]
                else:
                    cur[1] = max(cur[1], e1)
            if cur is not None:
                union += cur[1] - cur[0]
            top = {k: round(v / 1e3, 3) for k, v in by.most_common(14)}
            print(json.dumps({"rep": rep, "window": name, "host_ms": round((b - a) / 1e3, 3),
                              "gpu_busy_ms": round(union / 1e3, 3),
                              "kernel_sum_ms": round(sum(by.values()) / 1e3, 3), "top_ms": top}), flush=True)
        print(json.dumps({"rep": rep, "total_host_ms": round(total_host, 3)}), flush=True)


if __name__ == "__main__":
    main()
