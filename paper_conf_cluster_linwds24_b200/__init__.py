"""ScalFrag on B200: thin Python binding of libscalfrag.so (include/scalfrag.h).

Argument marshalling only -- every step of the hot path (ingest, sort, tiles,
features, selection, MTTKRP) runs inside the CUDA library.  There is no CPU
fallback: if the extension is missing the import of ``lib()`` fails loudly.

Arrays may be torch tensors (host, pinned or CUDA) or numpy arrays; index arrays
are passed as their raw 32-bit pattern (uint32 semantics; torch.int32 tensors are
accepted as long as every index < 2^31).
"""
from __future__ import annotations

import ctypes
import os
import threading

from . import _build

_HERE = os.path.dirname(os.path.abspath(__file__))
_lock = threading.Lock()
_lib = None

SF_MAX_MODES = 8
SF_HIST_BINS = 40
KERNEL_AUTO, KERNEL_COO, KERNEL_FRAG = 0, 1, 2
LAUNCH_NO_OWNER_STORES = 4
LAUNCH_DETERMINISTIC = 32
LAUNCH_L2_TILES = 64

STATUS = {0: "SF_OK", 1: "SF_ERR_INVALID_ARG", 2: "SF_ERR_INDEX_OUT_OF_RANGE",
          3: "SF_ERR_OUT_OF_MEMORY", 4: "SF_ERR_NOT_PLANNED", 5: "SF_ERR_UNSUPPORTED",
          6: "SF_ERR_CUDA", 7: "SF_ERR_NCCL"}


class SfError(RuntimeError):
    def __init__(self, status, detail):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {detail}")


class Launch(ctypes.Structure):
    _fields_ = [("kernel", ctypes.c_int32), ("block_threads", ctypes.c_int32),
                ("ctas_per_sm", ctypes.c_int32), ("chunk_nnz", ctypes.c_int32),
                ("staged_mask", ctypes.c_uint32), ("block_rows", ctypes.c_uint32 * SF_MAX_MODES),
                ("flags", ctypes.c_uint32), ("hot_kb", ctypes.c_uint32)]

    def as_dict(self):
        return {"kernel": {0: "auto", 1: "coo", 2: "frag"}.get(self.kernel, self.kernel),
                "block_threads": self.block_threads, "ctas_per_sm": self.ctas_per_sm,
                "chunk_nnz": self.chunk_nnz, "staged_mask": self.staged_mask,
                "block_rows": list(self.block_rows), "flags": self.flags, "hot_kb": self.hot_kb}

    @classmethod
    def make(cls, kernel=KERNEL_FRAG, block_threads=512, ctas_per_sm=0, chunk_nnz=128,
             staged=None, flags=0, hot_kb=0):
        """staged: {mode: block_rows}; flags: LAUNCH_* bits (include/scalfrag.h);
        hot_kb: hot-row cache budget in KiB (0 = off)"""
        l = cls()
        l.flags = flags
        l.hot_kb = hot_kb
        l.kernel, l.block_threads, l.ctas_per_sm, l.chunk_nnz = kernel, block_threads, ctas_per_sm, chunk_nnz
        mask = 0
        for m, r in (staged or {}).items():
            mask |= 1 << m
            l.block_rows[m] = r
        l.staged_mask = mask
        return l


class Features(ctypes.Structure):
    _fields_ = [("nnz", ctypes.c_uint64), ("dim", ctypes.c_uint64), ("num_slices", ctypes.c_uint64),
                ("num_fibers", ctypes.c_uint64), ("max_nnz_per_slice", ctypes.c_uint64),
                ("max_nnz_per_fiber", ctypes.c_uint64), ("sum_sq_nnz_per_slice", ctypes.c_uint64),
                ("slice_hist", ctypes.c_uint64 * SF_HIST_BINS), ("nmodes", ctypes.c_int32),
                ("mode", ctypes.c_int32), ("secondary", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("slice_ratio", ctypes.c_double), ("fiber_ratio", ctypes.c_double),
                ("avg_nnz_per_slice", ctypes.c_double), ("avg_nnz_per_fiber", ctypes.c_double),
                ("std_nnz_per_slice", ctypes.c_double)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_ if k not in ("slice_hist", "reserved")}
        d["slice_hist"] = list(self.slice_hist)
        return d


class PlanInfo(ctypes.Structure):
    _fields_ = [("feat", Features), ("launch", Launch), ("nnz_local", ctypes.c_uint64),
                ("num_tiles", ctypes.c_uint64), ("num_chunks", ctypes.c_uint64),
                ("row_begin", ctypes.c_uint64), ("row_end", ctypes.c_uint64),
                ("out_row0", ctypes.c_uint64), ("out_rows", ctypes.c_uint64),
                ("device_bytes", ctypes.c_uint64), ("plan_ms", ctypes.c_double)]

    def as_dict(self):
        return {"features": self.feat.as_dict(), "launch": self.launch.as_dict(),
                "nnz_local": self.nnz_local, "num_tiles": self.num_tiles,
                "num_chunks": self.num_chunks, "row_begin": self.row_begin,
                "row_end": self.row_end, "out_row0": self.out_row0, "out_rows": self.out_rows,
                "device_bytes": self.device_bytes, "plan_ms": self.plan_ms}


EXPORTED = ["sf_tensor_create", "sf_tensor_create_ex", "sf_tensor_destroy", "sf_set_shard",
            "sf_plan", "sf_set_launch", "sf_features", "sf_plan_info", "sf_plan_export",
            "sf_mttkrp", "sf_mttkrp_streamed", "sf_mttkrp_streamed_modes", "sf_status_string", "sf_last_error",
            "sf_kernel_launches", "sf_version", "sf_rows_op", "sf_selector_features",
            "sf_selector_candidates", "sf_set_selector_model", "sf_cpals", "sf_plan_release",
            "sf_trim_cache", "sf_shard_rows", "sf_comm_unique_id", "sf_comm_attach",
            "sf_comm_attach_transport", "sf_comm_detach", "sf_comm_check", "sf_allgather_rows", "sf_exchange_map",
            "sf_tensor_create_dist", "sf_device_bytes"]

# int fn(void* ctx, const void* send, void* recv, const uint64_t* bytes, const uint64_t* displs,
#        int nranks, void* stream)
ALLGATHERV_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                 ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64), ctypes.c_int,
                                 ctypes.c_void_p)


def lib(build_if_missing: bool = True):
    """Load libscalfrag.so (building it in-tree with nvcc if absent)."""
    global _lib
    with _lock:
        if _lib is None:
            so = _build.SO
            if not os.path.exists(so):
                if not build_if_missing:
                    raise RuntimeError(f"{so} missing: run __graft_entry__.build()")
                _build.build()
            L = ctypes.CDLL(so)
            P, I, U64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64
            L.sf_tensor_create.argtypes = [I, P, U64, P, P, ctypes.POINTER(P)]
            L.sf_tensor_create_ex.argtypes = [I, P, U64, P, P, I, I, ctypes.POINTER(P)]
            L.sf_tensor_destroy.argtypes = [P]
            L.sf_set_shard.argtypes = [P, I, I]
            L.sf_plan.argtypes = [P, I, I]
            L.sf_set_launch.argtypes = [P, I, I, ctypes.POINTER(Launch)]
            L.sf_features.argtypes = [P, I, ctypes.POINTER(Features)]
            L.sf_plan_info.argtypes = [P, I, I, ctypes.POINTER(PlanInfo)]
            L.sf_plan_export.argtypes = [P, I, I, P, P]
            L.sf_mttkrp.argtypes = [P, I, P, I, P, P]
            L.sf_mttkrp_streamed.argtypes = [I, P, U64, P, P, P, I, I, P, I, I]
            L.sf_mttkrp_streamed_modes.argtypes = [I, P, U64, P, P, P, I, P, I, I, P]
            L.sf_rows_op.argtypes = [P, I, P, P, I, I, P]
            L.sf_selector_features.argtypes = [P, I, I, P, ctypes.POINTER(I)]
            L.sf_selector_candidates.argtypes = [P, I, I, P, ctypes.POINTER(I)]
            L.sf_set_selector_model.argtypes = [P, P, P, P, P, I, I]
            L.sf_cpals.argtypes = [P, I, P, I, ctypes.c_double, P, ctypes.POINTER(I), P]
            L.sf_plan_release.argtypes = [P, I, I]
            L.sf_trim_cache.argtypes = []
            L.sf_shard_rows.argtypes = [P, I, I, ctypes.POINTER(U64), ctypes.POINTER(U64)]
            L.sf_comm_unique_id.argtypes = [P]
            L.sf_comm_attach.argtypes = [P, I, I, P]
            L.sf_comm_attach_transport.argtypes = [P, I, I, ALLGATHERV_FN, P]
            L.sf_comm_detach.argtypes = [P]
            L.sf_comm_check.argtypes = [P, P]
            L.sf_allgather_rows.argtypes = [P, I, I, P, P, P]
            L.sf_exchange_map.argtypes = [I, P, P, P]
            L.sf_device_bytes.argtypes = [ctypes.POINTER(U64), ctypes.POINTER(U64), I]
            L.sf_tensor_create_dist.argtypes = [I, P, U64, U64, U64, P, P, ctypes.POINTER(P)]
            for fn in EXPORTED:
                if fn not in ("sf_status_string", "sf_last_error", "sf_kernel_launches", "sf_version"):
                    getattr(L, fn).restype = ctypes.c_int
            L.sf_status_string.argtypes = [I]
            L.sf_status_string.restype = ctypes.c_char_p
            L.sf_last_error.argtypes = []
            L.sf_last_error.restype = ctypes.c_char_p
            L.sf_kernel_launches.argtypes = []
            L.sf_kernel_launches.restype = U64
            L.sf_version.argtypes = []
            L.sf_version.restype = ctypes.c_char_p
            _lib = L
    return _lib


# The deployed learned selector (tools/train_selector.py) is compiled into libscalfrag.so
# and installed when it loads (_build.write_model_inc); set_selector_model replaces it.
MODEL_PATH = os.path.join(_HERE, "selector_model.json")


def _install_model(L, path):
    """Install the learned launch selector (tools/train_selector.py) into the library."""
    import json
    import numpy as np
    m = json.load(open(path))
    t = m["tree"]
    arrs = [np.ascontiguousarray(t[k], dtype=dt) for k, dt in
            (("feature", np.int32), ("threshold", np.float64), ("left", np.int32), ("right", np.int32),
             ("value", np.int32))]
    rc = L.sf_set_selector_model(*[a.ctypes.data for a in arrs], len(arrs[0]), int(m["n_features"]))
    if rc != 0:
        raise SfError(rc, L.sf_last_error().decode())


def set_selector_model(model):
    """model: dict with 'tree' (feature/threshold/left/right/value lists) and 'n_features',
    None to fall back to the rule-based selector, or "default" for the compiled-in model."""
    if isinstance(model, str) and model == "default":
        _install_model(lib(), MODEL_PATH)
        return
    L = lib()
    if model is None:
        _check(L.sf_set_selector_model(None, None, None, None, None, 0, 0))
        return
    import json
    import tempfile
    with tempfile.NamedTemporaryFile("w", suffix=".json", delete=False) as f:
        json.dump(model, f)
    _install_model(L, f.name)
    os.unlink(f.name)


def _check(rc):
    if rc != 0:
        raise SfError(rc, lib().sf_last_error().decode())


def _ptr(x):
    if x is None:
        return None
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    if isinstance(x, int):
        return x
    raise TypeError(f"cannot take a pointer of {type(x)}")


def _stream_handle(stream):
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except Exception:
            pass
        return 0
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def trim_cache():
    """Return the library's cached device blocks to the driver."""
    _check(lib().sf_trim_cache())


def kernel_launches() -> int:
    return int(lib().sf_kernel_launches())


def device_bytes(reset_peak=False):
    """(bytes held by live library buffers, high-water mark) -- sf_device_bytes."""
    a, b = ctypes.c_uint64(0), ctypes.c_uint64(0)
    _check(lib().sf_device_bytes(ctypes.byref(a), ctypes.byref(b), int(bool(reset_peak))))
    return a.value, b.value


def version() -> str:
    return lib().sf_version().decode()


class Tensor:
    """Handle of a device-resident COO tensor (sf_tensor_t)."""

    def __init__(self, dims, inds, vals, segments=0, streams=0):
        self.dims = tuple(int(d) for d in dims)
        self.nmodes = len(self.dims)
        self.nnz = int(len(vals))
        d = (ctypes.c_uint64 * self.nmodes)(*self.dims)
        ip = (ctypes.c_void_p * self.nmodes)(*[_ptr(a) for a in inds])
        h = ctypes.c_void_p()
        _check(lib().sf_tensor_create_ex(self.nmodes, d, self.nnz, ip, _ptr(vals), int(segments),
                                         int(streams), ctypes.byref(h)))
        self._h = h

    @classmethod
    def create_dist(cls, dims, nnz_total, pos_begin, inds, vals):
        """Distributed ingest (sf_tensor_create_dist): this rank's slice [pos_begin, pos_begin +
        len(vals)) of an nnz_total-nonzero tensor; attach a comm before planning."""
        self = cls.__new__(cls)
        self.dims = tuple(int(d) for d in dims)
        self.nmodes = len(self.dims)
        self.nnz = int(len(vals))
        d = (ctypes.c_uint64 * self.nmodes)(*self.dims)
        ip = (ctypes.c_void_p * self.nmodes)(*[_ptr(a) for a in inds])
        h = ctypes.c_void_p()
        _check(lib().sf_tensor_create_dist(self.nmodes, d, int(nnz_total), int(pos_begin), self.nnz, ip, _ptr(vals),
                                           ctypes.byref(h)))
        self._h = h
        return self

    def close(self):
        if getattr(self, "_h", None):
            lib().sf_tensor_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def set_shard(self, nranks, rank):
        _check(lib().sf_set_shard(self._h, int(nranks), int(rank)))

    def shard_rows(self, mode, rank):
        """Rows [begin, end) of Y that mttkrp(mode) writes into `out` (the local row block
        of a shard; all of Y unsharded)."""
        b, e = ctypes.c_uint64(0), ctypes.c_uint64(0)
        _check(lib().sf_shard_rows(self._h, int(mode), int(rank), ctypes.byref(b), ctypes.byref(e)))
        return b.value, e.value

    def comm_attach(self, nranks, rank, unique_id: bytes):
        """NCCL communicator for the boundary exchange (+ sf_set_shard(nranks, rank))."""
        buf = ctypes.create_string_buffer(bytes(unique_id), 128)
        _check(lib().sf_comm_attach(self._h, int(nranks), int(rank), buf))

    def comm_attach_transport(self, nranks, rank, fn):
        """Boundary exchange over a Python allgatherv (ALLGATHERV_FN; kept alive here)."""
        self._transport = fn if isinstance(fn, ALLGATHERV_FN) else ALLGATHERV_FN(fn)
        _check(lib().sf_comm_attach_transport(self._h, int(nranks), int(rank), self._transport, None))

    def comm_detach(self):
        _check(lib().sf_comm_detach(self._h))

    def comm_check(self, stream=None):
        """Collective self-test of the attached transport (sf_comm_check)."""
        _check(lib().sf_comm_check(self._h, _stream_handle(stream)))

    def allgather_rows(self, mode, local, full, stream=None):
        """Replicated Y (full, I_mode x R on every rank) from the row-sharded local blocks."""
        _check(lib().sf_allgather_rows(self._h, int(mode), int(full.shape[1]), _ptr(local), _ptr(full),
                                       _stream_handle(stream)))
        return full

    def plan(self, mode, rank, deterministic=False):
        """sf_plan (selector's launch); deterministic=True plans the A7 two-pass carry
        combine instead (unstaged owner-store fragment plan, bitwise reproducible Y)."""
        if deterministic:
            self.set_launch(mode, rank, Launch.make(kernel=KERNEL_FRAG, flags=LAUNCH_DETERMINISTIC))
        else:
            _check(lib().sf_plan(self._h, int(mode), int(rank)))

    def plan_release(self, mode, rank):
        _check(lib().sf_plan_release(self._h, int(mode), int(rank)))

    def set_launch(self, mode, rank, launch: Launch):
        _check(lib().sf_set_launch(self._h, int(mode), int(rank), ctypes.byref(launch)))

    def features(self, mode) -> dict:
        f = Features()
        _check(lib().sf_features(self._h, int(mode), ctypes.byref(f)))
        return f.as_dict()

    def plan_info(self, mode, rank) -> dict:
        p = PlanInfo()
        _check(lib().sf_plan_info(self._h, int(mode), int(rank), ctypes.byref(p)))
        return p.as_dict()

    def plan_export(self, mode, rank):
        import numpy as np
        info = self.plan_info(mode, rank)
        perm = np.empty(info["nnz_local"], np.uint64)
        chunks = np.empty((info["num_chunks"], 3), np.uint64)
        _check(lib().sf_plan_export(self._h, int(mode), int(rank), perm.ctypes.data if perm.size else None,
                                    chunks.ctypes.data if chunks.size else None))
        return perm, chunks

    def selector_features(self, mode, rank):
        x = (ctypes.c_double * 32)()
        n = ctypes.c_int(0)
        _check(lib().sf_selector_features(self._h, int(mode), int(rank), x, ctypes.byref(n)))
        return [x[i] for i in range(n.value)]

    def selector_candidates(self, mode, rank):
        arr = (Launch * 16)()
        n = ctypes.c_int(0)
        _check(lib().sf_selector_candidates(self._h, int(mode), int(rank), arr, ctypes.byref(n)))
        out = []
        for i in range(n.value):
            l = Launch()
            ctypes.memmove(ctypes.byref(l), ctypes.byref(arr[i]), ctypes.sizeof(Launch))
            out.append(l)
        return out

    def cp_als(self, factors, iters=10, tol=0.0, stream=None):
        """CP-ALS (Algorithm 1) in place on device factor tensors; returns the fit per sweep."""
        import numpy as np
        rank = int(factors[0].shape[1])
        fp = (ctypes.c_void_p * self.nmodes)(*[_ptr(f) for f in factors])
        fits = np.zeros(max(iters, 1), np.float64)
        done = ctypes.c_int(0)
        _check(lib().sf_cpals(self._h, rank, fp, int(iters), float(tol), fits.ctypes.data, ctypes.byref(done),
                              _stream_handle(stream)))
        return fits[:done.value].tolist()

    def mttkrp(self, mode, factors, out, rank=None, stream=None):
        """out <- mode-`mode` MTTKRP (device tensors; stream-ordered)."""
        rank = int(out.shape[1]) if rank is None else int(rank)
        fp = (ctypes.c_void_p * self.nmodes)(*[_ptr(f) if (m != mode and f is not None) else None
                                               for m, f in enumerate(factors)])
        _check(lib().sf_mttkrp(self._h, int(mode), fp, rank, _ptr(out), _stream_handle(stream)))
        return out


def mttkrp_streamed(dims, inds, vals, factors, mode, out, segments=8, streams=4):
    """One-shot streamed MTTKRP of a HOST COO tensor (the paper's pipeline, §IV-C)."""
    N = len(dims)
    d = (ctypes.c_uint64 * N)(*[int(x) for x in dims])
    ip = (ctypes.c_void_p * N)(*[_ptr(a) for a in inds])
    fp = (ctypes.c_void_p * N)(*[_ptr(f) if (m != mode and f is not None) else None
                                 for m, f in enumerate(factors)])
    _check(lib().sf_mttkrp_streamed(N, d, int(len(vals)), ip, _ptr(vals), fp, int(out.shape[1]), int(mode),
                                    _ptr(out), int(segments), int(streams)))
    return out


def mttkrp_streamed_modes(dims, inds, vals, factors, outs, segments=8, streams=4, stream=None):
    """One-shot streamed MTTKRP of every mode n with outs[n] is not None (HOST COO, one upload
    for all modes; the work is ordered after what `stream` already holds)."""
    N = len(dims)
    d = (ctypes.c_uint64 * N)(*[int(x) for x in dims])
    ip = (ctypes.c_void_p * N)(*[_ptr(a) for a in inds])
    fp = (ctypes.c_void_p * N)(*[_ptr(f) if f is not None else None for f in factors])
    op = (ctypes.c_void_p * N)(*[_ptr(o) if o is not None else None for o in outs])
    rank = next((int(o.shape[1]) for o in outs if o is not None), 1)  # no output: the library rejects it
    _check(lib().sf_mttkrp_streamed_modes(N, d, int(len(vals)), ip, _ptr(vals), fp, rank, op, int(segments),
                                          int(streams), _stream_handle(stream)))
    return outs


def comm_unique_id() -> bytes:
    """A new 128-byte NCCL unique id (rank 0; broadcast it to the other ranks)."""
    buf = ctypes.create_string_buffer(128)
    _check(lib().sf_comm_unique_id(buf))
    return buf.raw


def exchange_map(ranges):
    """Host-only exchange rule (sf_exchange_map): ranges = [(row_begin, row_end)] per rank.
    Returns (send_first[k], owner[k])."""
    import numpy as np
    P = len(ranges)
    r = np.ascontiguousarray(np.array(ranges, dtype=np.uint64).reshape(P, 2))
    sendf = np.zeros(P, np.int32)
    owner = np.zeros(P, np.int32)
    _check(lib(build_if_missing=True).sf_exchange_map(P, r.ctypes.data, sendf.ctypes.data, owner.ctypes.data))
    return sendf.tolist(), owner.tolist()


ROWS_PACK, ROWS_ADD, ROWS_ZERO = 0, 1, 2


def rows_op(Y, rows, buf, op, stream=None):
    """Boundary-row pack / add / zero on device tensors (sf_rows_op)."""
    _check(lib().sf_rows_op(_ptr(Y), int(Y.shape[1]), _ptr(rows), _ptr(buf), int(rows.numel()), int(op),
                            _stream_handle(stream)))
