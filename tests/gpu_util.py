"""Helpers for the -m gpu parity tests: drive the CUDA path through the C ABI
binding and compare with the oracle."""
import numpy as np
import torch

import oracle
import paper_conf_cluster_linwds24_b200 as sf

TOL = 1e-4  # north_star: max |Δ| / (|v|·∏|A| scale) <= 1e-4 per element


def dev_inds(inds, dev="cuda:0"):
    return [torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).to(dev) for a in inds]


def dev_f(x, dev="cuda:0"):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).to(dev)


def run(dims, inds, vals, facs, R, modes=None, launch=None, device_input=True, shard=None):
    """Returns {mode: Y (np.float32)} and the handle's plan infos."""
    dev = torch.device("cuda:0")
    if device_input:
        ti, tv = dev_inds(inds), dev_f(vals)
    else:
        ti, tv = [np.ascontiguousarray(a, np.uint32) for a in inds], np.ascontiguousarray(vals, np.float32)
    tf = [dev_f(f) for f in facs]
    out, infos = {}, {}
    with sf.Tensor(dims, ti, tv) as t:
        if shard:
            t.set_shard(*shard)
        for n in (modes if modes is not None else range(len(dims))):
            if launch is not None:
                L = launch(n) if callable(launch) else launch
                t.set_launch(n, R, L)
            else:
                t.plan(n, R)
            info = t.plan_info(n, R)
            # the library writes the plan's out block (all of Y unsharded, the local row block of
            # a shard); NaN-filled so any row it fails to write is caught; embedded in a full Y
            y = torch.full((info["out_rows"], R), float("nan"), dtype=torch.float32, device=dev)
            t.mttkrp(n, tf, y)
            torch.cuda.synchronize()
            full = np.zeros((dims[n], R), np.float32)
            full[info["out_row0"]:info["out_row0"] + info["out_rows"]] = y.cpu().numpy()
            out[n] = full
            infos[n] = info
    return out, infos


def assert_parity(Yg, dims, inds, vals, facs, R, n, tol=TOL):
    Y, S = oracle.mttkrp(dims, inds, vals, facs, R, n)
    assert np.all(np.isfinite(Yg)), "non-finite output"
    rel, zv = oracle.max_rel_err(Yg, Y, S)
    assert rel <= tol, f"mode {n}: max rel err {rel:.3e} > {tol}"
    assert zv == 0.0, f"mode {n}: nonzero value {zv} in a row with no contribution"
    return rel
