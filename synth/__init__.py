"""Seeded synthetic inputs shaped like the paper's FROSTT workloads.

This package is the one module both sides may use: the oracle (tests, bench
cpu_baseline) and the CUDA path (tests, bench).  It holds none of the MTTKRP
arithmetic -- only random numbers.  The recipe (DESIGN.md "Input recipe",
SURVEY.md §8(d) D-2) is implemented in ``csrc/sfgen_core.h``.

Shapes come from BASELINE.json ``configs`` (FROSTT exact dims; the paper's
Table III, gives the rounded dims/nnz/density).  The Zipf
exponents are proposals, unpinned against real
FROSTT statistics.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
import threading
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsfgen.so")
_SRC = [os.path.join(_HERE, "csrc", "sfgen.c")]
_lock = threading.Lock()
_lib = None

VAL_KINDS = {"unit": 0, "signed": 1, "int": 2, "ones": 3, "bin": 4}


def build(force: bool = False) -> str:
    """Compile libsfgen.so with gcc (host generator; no GPU needed)."""
    newest = max(os.path.getmtime(p) for p in _SRC + [os.path.join(_HERE, "csrc", "sfgen_core.h")])
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < newest:
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", "-std=c11",
                               "-o", tmp] + _SRC)
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_SO)
            P = ctypes.c_void_p
            u64 = ctypes.c_uint64
            L.sfgen_coo.argtypes = [ctypes.c_int, P, u64, u64, u64, P, P, P, ctypes.c_int,
                                    ctypes.c_int, P, P]
            L.sfgen_coo.restype = None
            L.sfgen_factor.argtypes = [u64, u64, u64, ctypes.c_int, ctypes.c_int, P]
            L.sfgen_factor.restype = None
            L.sfgen_permute_many.argtypes = [u64, u64, ctypes.c_int, u64, P, P]
            L.sfgen_permute_many.restype = None
            L.sfgen_hash.argtypes = [u64, u64, u64]
            L.sfgen_hash.restype = u64
            _lib = L
    return _lib


def zipf_table(I: int, s: float, K: int = 1024):
    """Geometric bucket table for a power law P(x) ~ (x+1)^-s on [0, I).

    edges: e_0 = 0, e_k = round(I^(k/K)), e_K = I, de-duplicated (strictly increasing).
    Bucket k has weight  int_{e_k}^{e_{k+1}} (x+1)^-s dx  (fp64, computed once here);
    thr[k-1] = floor(2^64 * CDF_k) for k = 1..nb-1.  Sampling inside a bucket is uniform.
    Returns (edges uint64[nb+1], thr uint64[nb-1]); nb == 0 encodes "uniform".
    """
    if s == 0.0 or I <= 1:
        return np.zeros(0, np.uint64), np.zeros(0, np.uint64)
    raw = [0] + [int(round(I ** (k / K))) for k in range(1, K)] + [int(I)]
    edges = sorted(set(min(max(e, 0), int(I)) for e in raw))
    e = np.array(edges, dtype=np.float64)
    a, b = e[:-1] + 1.0, e[1:] + 1.0
    if abs(s - 1.0) < 1e-12:
        w = np.log(b / a)
    else:
        w = (b ** (1.0 - s) - a ** (1.0 - s)) / (1.0 - s)
    cdf = np.cumsum(w) / np.sum(w)
    thr = []
    for c in cdf[:-1]:
        v = int(math.ldexp(float(c), 64))
        thr.append(min(v, 2 ** 64 - 1))
    return np.array(edges, dtype=np.uint64), np.array(thr, dtype=np.uint64)


@dataclass
class Config:
    name: str
    dims: tuple
    nnz: int
    rank: int
    zipf: tuple
    seed: int
    fseed: int
    note: str = ""
    tables: list = field(default_factory=list, repr=False)

    @property
    def nmodes(self):
        return len(self.dims)


def _cfg(k, name, dims, nnz, rank, zipf, note):
    return Config(name, tuple(dims), int(nnz), int(rank), tuple(zipf), 20240000 + k, 20241000 + 10 * k, note)


# BASELINE.json configs[0..4] (SURVEY.md §8(a) constants table; D-2 Zipf proposals)
CONFIGS = {
    "tiny": _cfg(1, "tiny", (100, 80, 60), 10_000, 16, (0.0, 0.0, 0.0),
                 "BASELINE.json configs[0]: synthetic 3-way 100x80x60, nnz=10k, R=16"),
    "tiny_skew": _cfg(1, "tiny_skew", (100, 80, 60), 10_000, 16, (1.0, 1.0, 1.0),
                      "skewed twin of configs[0]"),
    "nell2": _cfg(2, "nell2", (12092, 9184, 28818), 76_879_419, 32, (0.5, 0.5, 0.5),
                  "BASELINE.json configs[1]: nell-2-shaped, R=32"),
    "deli4d": _cfg(3, "deli4d", (532924, 17262471, 2480308, 1443), 140_126_181, 32,
                   (1.0, 1.0, 1.0, 0.3), "BASELINE.json configs[2]: delicious(4d)-shaped, R=32"),
    "nell1": _cfg(4, "nell1", (2902330, 2143368, 25495389), 143_599_552, 32, (0.8, 0.8, 0.8),
                  "BASELINE.json configs[3]: nell-1-shaped, R=32"),
    "amazon": _cfg(5, "amazon", (4821207, 1774269, 1805187), 1_741_809_018, 16, (0.8, 0.8, 1.0),
                   "BASELINE.json configs[4]: amazon-reviews-shaped, R=16"),
    # the other PAPER.md Table III tensors (L256-267) as synthetic shapes
    # (FROSTT exact dims; rank not stated by the paper: R = 16; Zipf exponents proposals)
    "vast": _cfg(6, "vast", (165427, 11374, 2), 26_021_945, 16, (0.5, 0.5, 0.0),
                 "Table III vast-shaped 165K x 11K x 2, 26M nnz"),
    "flickr3d": _cfg(7, "flickr3d", (319686, 28153045, 1607191), 112_890_310, 16, (1.0, 1.0, 1.0),
                     "Table III flickr-3d-shaped 320K x 28M x 2M, 113M nnz"),
    "deli3d": _cfg(8, "deli3d", (532924, 17262471, 2480308), 140_126_181, 16, (1.0, 1.0, 1.0),
                   "Table III deli-3d-shaped 533K x 17M x 3M, 140M nnz"),
    "uber": _cfg(9, "uber", (183, 24, 1140, 1717), 3_309_490, 16, (0.3, 0.3, 0.5, 0.5),
                 "Table III uber-shaped 183 x 24 x 1140 x 1717, 3M nnz"),
    "nips": _cfg(10, "nips", (2482, 2862, 14036, 17), 3_101_609, 16, (0.8, 0.8, 0.8, 0.3),
                 "Table III nips-shaped 2K x 3K x 14K x 17, 3M nnz"),
    "enron": _cfg(11, "enron", (6066, 5699, 244268, 1176), 54_202_099, 16, (1.0, 1.0, 0.8, 0.5),
                  "Table III enron-shaped 6K x 6K x 244K x 1K, 54M nnz"),
    "flickr4d": _cfg(12, "flickr4d", (319686, 28153045, 1607191, 731), 112_890_310, 16, (1.0, 1.0, 1.0, 0.3),
                     "Table III flickr-4d-shaped 320K x 28M x 2M x 731, 113M nnz"),
}
TABLE_III = ["vast", "nell2", "flickr3d", "deli3d", "nell1", "uber", "nips", "enron", "flickr4d", "deli4d"]


def tables_for(dims, zipf):
    return [zipf_table(int(I), float(s)) for I, s in zip(dims, zipf)]


def gen_coo(dims, nnz, seed, zipf=None, relabel=True, val_kind="unit", lo=0, hi=None,
            tables=None):
    """Elements [lo, hi) of the seeded COO tensor: (list of uint32[n] per mode, float32[n])."""
    dims = [int(d) for d in dims]
    N = len(dims)
    hi = int(nnz) if hi is None else int(hi)
    n = hi - lo
    if tables is None:
        tables = tables_for(dims, zipf if zipf is not None else (0.0,) * N)
    inds = [np.empty(n, dtype=np.uint32) for _ in range(N)]
    vals = np.empty(n, dtype=np.float32)
    if n == 0:
        return inds, vals
    nb = np.array([len(t[0]) - 1 if len(t[0]) else 0 for t in tables], dtype=np.int32)
    edge_ptrs = (ctypes.c_void_p * N)(*[t[0].ctypes.data if len(t[0]) else None for t in tables])
    thr_ptrs = (ctypes.c_void_p * N)(*[t[1].ctypes.data if len(t[1]) else None for t in tables])
    ind_ptrs = (ctypes.c_void_p * N)(*[a.ctypes.data for a in inds])
    d = np.array(dims, dtype=np.uint64)
    lib().sfgen_coo(N, d.ctypes.data, seed, lo, hi, nb.ctypes.data, edge_ptrs, thr_ptrs,
                    1 if relabel else 0, VAL_KINDS[val_kind], ind_ptrs, vals.ctypes.data)
    return inds, vals


def gen_factor(rows, rank, seed, stream, kind="unit"):
    out = np.empty((int(rows), int(rank)), dtype=np.float32)
    if out.size:
        lib().sfgen_factor(seed, stream, rows, rank, VAL_KINDS[kind], out.ctypes.data)
    return out


def gen_factors(dims, rank, seed, kind="unit"):
    return [gen_factor(I, rank, seed, m, kind) for m, I in enumerate(dims)]


def config_tensor(cfg: Config | str, lo=0, hi=None, val_kind="unit"):
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    if not cfg.tables:
        cfg.tables = tables_for(cfg.dims, cfg.zipf)
    return gen_coo(cfg.dims, cfg.nnz, cfg.seed, cfg.zipf, True, val_kind, lo, hi, cfg.tables)


def config_factors(cfg: Config | str, kind="unit"):
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    return gen_factors(cfg.dims, cfg.rank, cfg.fseed, kind)


def permute(I, seed, m, xs):
    xs = np.ascontiguousarray(xs, dtype=np.uint64)
    out = np.empty_like(xs)
    lib().sfgen_permute_many(I, seed, m, len(xs), xs.ctypes.data, out.ctypes.data)
    return out


# ---------------------------------------------------------------------------
# Device twin (csrc/sfgen_cuda.cu): the same draws generated directly in HBM.
# ---------------------------------------------------------------------------
_SO_CUDA = os.path.join(_HERE, "libsfgen_cuda.so")
_SRC_CUDA = os.path.join(_HERE, "csrc", "sfgen_cuda.cu")
_lib_cuda = None


def build_cuda(force: bool = False) -> str:
    newest = max(os.path.getmtime(p) for p in [_SRC_CUDA, os.path.join(_HERE, "csrc", "sfgen_core.h")])
    if force or not os.path.exists(_SO_CUDA) or os.path.getmtime(_SO_CUDA) < newest:
        tmp = _SO_CUDA + f".tmp{os.getpid()}"
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-shared", "-Xcompiler", "-fPIC", "-cudart", "static", "-o", tmp, _SRC_CUDA])
        os.replace(tmp, _SO_CUDA)
    return _SO_CUDA


def lib_cuda():
    global _lib_cuda
    with _lock:
        if _lib_cuda is None:
            build_cuda()
            L = ctypes.CDLL(_SO_CUDA)
            P, u64 = ctypes.c_void_p, ctypes.c_uint64
            L.sfgen_coo_device.argtypes = [ctypes.c_int, P, u64, u64, u64, P, P, P, P, P, ctypes.c_int,
                                           ctypes.c_int, P, P, P]
            L.sfgen_coo_device.restype = ctypes.c_int
            L.sfgen_factor_device.argtypes = [u64, u64, u64, ctypes.c_int, ctypes.c_int, P, P]
            L.sfgen_factor_device.restype = ctypes.c_int
            _lib_cuda = L
    return _lib_cuda


def gen_coo_device(dims, nnz, seed, zipf=None, relabel=True, val_kind="unit", lo=0, hi=None, tables=None,
                   device="cuda"):
    """Device twin of gen_coo: torch int32 (uint32 bit pattern) index tensors + float32 values."""
    import torch
    dims = [int(d) for d in dims]
    N = len(dims)
    hi = int(nnz) if hi is None else int(hi)
    n = hi - lo
    if tables is None:
        tables = tables_for(dims, zipf if zipf is not None else (0.0,) * N)
    dev = torch.device(device)
    inds = [torch.empty(n, dtype=torch.int32, device=dev) for _ in range(N)]
    vals = torch.empty(n, dtype=torch.float32, device=dev)
    if n == 0:
        return inds, vals
    edges = np.concatenate([t[0] for t in tables] + [np.zeros(1, np.uint64)])
    thr = np.concatenate([t[1] for t in tables] + [np.zeros(1, np.uint64)])
    eoff = np.cumsum([0] + [len(t[0]) for t in tables])[:-1].astype(np.int32)
    toff = np.cumsum([0] + [len(t[1]) for t in tables])[:-1].astype(np.int32)
    nb = np.array([len(t[0]) - 1 if len(t[0]) else 0 for t in tables], dtype=np.int32)
    d_edges = torch.from_numpy(edges.view(np.int64)).to(dev)
    d_thr = torch.from_numpy(thr.view(np.int64)).to(dev)
    d_eoff, d_toff, d_nb = (torch.from_numpy(a).to(dev) for a in (eoff, toff, nb))
    d_dims = torch.tensor(dims, dtype=torch.int64, device=dev)
    d_ptrs = torch.tensor([a.data_ptr() for a in inds], dtype=torch.int64, device=dev)
    stream = torch.cuda.current_stream(dev).cuda_stream
    rc = lib_cuda().sfgen_coo_device(N, d_dims.data_ptr(), seed, lo, hi, d_edges.data_ptr(), d_thr.data_ptr(),
                                     d_nb.data_ptr(), d_eoff.data_ptr(), d_toff.data_ptr(), 1 if relabel else 0,
                                     VAL_KINDS[val_kind], d_ptrs.data_ptr(), vals.data_ptr(), stream)
    if rc != 0:
        raise RuntimeError(f"sfgen_coo_device failed: cuda error {rc}")
    torch.cuda.synchronize(dev)
    return inds, vals


def gen_factors_device(dims, rank, seed, kind="unit", device="cuda"):
    import torch
    out = []
    stream = torch.cuda.current_stream(torch.device(device)).cuda_stream
    for m, I in enumerate(dims):
        f = torch.empty((int(I), int(rank)), dtype=torch.float32, device=device)
        rc = lib_cuda().sfgen_factor_device(seed, m, int(I), int(rank), VAL_KINDS[kind], f.data_ptr(), stream)
        if rc != 0:
            raise RuntimeError(f"sfgen_factor_device failed: cuda error {rc}")
        out.append(f)
    torch.cuda.synchronize()
    return out


def config_tensor_device(cfg, val_kind="unit", lo=0, hi=None, device="cuda"):
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    if not cfg.tables:
        cfg.tables = tables_for(cfg.dims, cfg.zipf)
    return gen_coo_device(cfg.dims, cfg.nnz, cfg.seed, cfg.zipf, True, val_kind, lo, hi, cfg.tables, device)


def config_factors_device(cfg, kind="unit", device="cuda"):
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    return gen_factors_device(cfg.dims, cfg.rank, cfg.fseed, kind, device)
