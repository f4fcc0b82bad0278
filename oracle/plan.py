"""Oracle for the integer preprocessing -- TEST INFRASTRUCTURE ONLY.

The CUDA planner (sf_plan) must reproduce every array here bit-exactly
(north_star: "Tiling, sorting and partitioning must be bit-exact as integer
work").  Each step is written with plain numpy; the one library primitive is a
stable sort (``np.argsort(kind="stable")``).

Definitions (readings R9-R12):

* Matricized order ("ScalFrag first matricizes the input tensor
  and then chunks the matricized tensor"): nonzeros sorted stably by the key
  (i_n, i_s), where s is the gathered mode with the smallest dimension (ties:
  the higher mode index) -- the fiber key with the most reuse of A_s rows
  (reading R10).  Ties keep input order.
* Shards (multi-GPU): rank p of P owns matricized positions
  [floor(p*nnz/P), floor((p+1)*nnz/P)).
* Tiles ("tensor blocks ... based on the resource constraints of hardware",
  PAPER.md L34): for the staged mode set S (ascending) with block rows b_m,
  tile(e) = fold over m in S of  t*ceil(I_m/b_m) + i_m(e) // b_m.
  The kernel order is the matricized order re-sorted stably by tile, i.e.
  the lexicographic order (tile, i_n, i_s, input position).
* Chunks ("segments"): each tile's run is cut every C
  nonzeros; chunk = (begin, end, tile).
* Features: numSlices, numFibers, sliceRatio, fiberRatio,
  maxNnzPerSlice, maxNnzPerFiber (reading R4 for the duplicated name), plus
  slice-length moments and a log2 histogram.
"""
from __future__ import annotations

import numpy as np


def secondary_mode(nmodes: int, mode: int, dims=None) -> int:
    """DESIGN.md reading R10: the gathered mode with the smallest dimension (ties: the
    higher mode index); without dims, the highest-numbered mode != n."""
    others = [m for m in range(nmodes) if m != mode]
    if dims is None:
        return max(others)
    return min(others, key=lambda m: (int(dims[m]), -m))


def matricized_order(dims, inds, mode):
    """Stable argsort by (i_n, i_s)  (uint64 key i_n * I_s + i_s)."""
    s = secondary_mode(len(dims), mode, dims)
    key = inds[mode].astype(np.uint64) * np.uint64(dims[s]) + inds[s].astype(np.uint64)
    return np.argsort(key, kind="stable").astype(np.int64)


def shard_range(nnz: int, nranks: int, rank: int):
    return (rank * nnz) // nranks, ((rank + 1) * nnz) // nranks


def tile_ids(dims, inds, staged, block_rows, sel=None):
    t = None
    for m in sorted(staged):
        idx = inds[m] if sel is None else inds[m][sel]
        q = idx.astype(np.uint64) // np.uint64(block_rows[m])
        T = np.uint64(-(-int(dims[m]) // int(block_rows[m])))
        t = q if t is None else t * T + q
    if t is None:
        n = len(inds[0]) if sel is None else len(sel)
        t = np.zeros(n, np.uint64)
    return t


def plan_order(dims, inds, mode, staged=(), block_rows=None, nranks=1, rank=0):
    """Kernel order of this rank's nonzeros: positions into the input COO."""
    nnz = len(inds[0])
    perm0 = matricized_order(dims, inds, mode)
    lo, hi = shard_range(nnz, nranks, rank)
    local = perm0[lo:hi]
    if not staged:
        return local
    t = tile_ids(dims, inds, staged, block_rows, sel=local)
    return local[np.argsort(t, kind="stable")]


def chunks(tiles_sorted, C):
    """Chunk list (begin, end, tile) over a tile-sorted id array."""
    n = len(tiles_sorted)
    out = []
    if n == 0:
        return np.zeros((0, 3), np.int64)
    starts = np.flatnonzero(np.r_[True, tiles_sorted[1:] != tiles_sorted[:-1]])
    ends = np.r_[starts[1:], n]
    for a, b in zip(starts, ends):
        for c in range(int(a), int(b), C):
            out.append((c, min(c + C, int(b)), int(tiles_sorted[a])))
    return np.array(out, dtype=np.int64)


def features(dims, inds, mode):
    """PAPER.md L195 feature vector for mode `mode` (exact integers + derived ratios)."""
    N = len(dims)
    In = int(dims[mode])
    nnz = len(inds[0])
    s = secondary_mode(N, mode, dims)
    cnt = np.bincount(inds[mode].astype(np.int64), minlength=In) if nnz else np.zeros(In, np.int64)
    nz = cnt[cnt > 0]
    key = inds[mode].astype(np.uint64) * np.uint64(dims[s]) + inds[s].astype(np.uint64)
    uk, fc = np.unique(key, return_counts=True) if nnz else (np.zeros(0), np.zeros(0, np.int64))
    hist = np.zeros(40, np.int64)
    if len(nz):
        # floor(log2 c) exactly: frexp gives c = m * 2^e, m in [0.5, 1), exact below 2^53
        b = np.frexp(nz.astype(np.float64))[1].astype(np.int64) - 1
        np.add.at(hist, b, 1)
    num_slices = int(len(nz))
    num_fibers = int(len(uk))
    # sum of squares <= nnz^2 < 2^64 for nnz < 2^32: exact in uint64
    sum_sq = int(np.sum(nz.astype(np.uint64) ** np.uint64(2), dtype=np.uint64)) if len(nz) else 0
    f = dict(
        nnz=int(nnz), nmodes=N, mode=int(mode), dim=In, secondary=int(s),
        num_slices=num_slices, num_fibers=num_fibers,
        max_nnz_per_slice=int(nz.max()) if len(nz) else 0,
        max_nnz_per_fiber=int(fc.max()) if len(fc) else 0,
        sum_sq_nnz_per_slice=sum_sq,
        slice_hist=hist,
    )
    f["slice_ratio"] = num_slices / In if In else 0.0
    f["fiber_ratio"] = num_fibers / num_slices if num_slices else 0.0
    f["avg_nnz_per_slice"] = nnz / num_slices if num_slices else 0.0
    f["avg_nnz_per_fiber"] = nnz / num_fibers if num_fibers else 0.0
    var = (sum_sq / num_slices - f["avg_nnz_per_slice"] ** 2) if num_slices else 0.0
    f["std_nnz_per_slice"] = float(np.sqrt(max(var, 0.0)))
    return f
