"""Multi-GPU plumbing for row-sharded MTTKRP.

Rank p of P owns matricized positions [floor(p*nnz/P), floor((p+1)*nnz/P)) of every mode
(sf_set_shard), so sf_mttkrp writes one local row block [row_begin, row_end) and adjacent
ranks share at most the row straddling a cut.  The boundary exchange that turns the
partial blocks into a row-sharded Y (owner = lowest rank touching a row; partials added
in rank order) runs INSIDE libscalfrag (csrc/sf_comm.cu), at the end of every sf_mttkrp,
over one of two transports:

* NCCL (production): rank 0 creates the 128-byte unique id (sf_comm_unique_id), it is
  broadcast through torch.distributed, every rank calls sf_comm_attach -- the exchange is
  then a grouped ncclBroadcast allgatherv on the caller's stream;
* a torch.distributed allgatherv (TorchAllgatherv, passed as an sf_allgatherv_fn callback):
  host-staged over gloo, for multi-rank tests with several ranks on one GPU, where NCCL
  cannot run (two ranks may not share a device).

This module only marshals: the exchange rule (sf_exchange_map), packing, zeroing and the
owner adds are C/CUDA.
"""
from __future__ import annotations

import ctypes

import torch
import torch.distributed as dist

from . import ALLGATHERV_FN, comm_unique_id


class _DevBytes:
    """A raw device pointer as a uint8 CUDA array (torch consumes __cuda_array_interface__)."""

    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": "|u1", "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def _dev_view(ptr, n, device):
    return torch.as_tensor(_DevBytes(ptr, n), device=device)


class TorchAllgatherv:
    """allgatherv over a torch.distributed group, host-staged (works with gloo).

    Rank k contributes bytes[k] bytes; every rank receives block k at recv + displs[k].
    `allgatherv_host` is the transport proper (host tensors); calling the object is the
    sf_allgatherv_fn callback the library invokes with device pointers."""

    def __init__(self, group=None, device=None):
        self.group = group
        self.device = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.cfn = ALLGATHERV_FN(self._callback)
        self.errors = []

    def allgatherv_host(self, send, nbytes):
        """send: uint8 host tensor of this rank's nbytes[rank] bytes -> list of P host tensors."""
        P = len(nbytes)
        mx = max(max(nbytes), 1)
        pad = torch.zeros(mx, dtype=torch.uint8)
        me = dist.get_rank(self.group)
        if nbytes[me]:
            pad[:nbytes[me]] = send[:nbytes[me]]
        out = [torch.empty(mx, dtype=torch.uint8) for _ in range(P)]
        dist.all_gather(out, pad, group=self.group)
        return [out[k][:nbytes[k]] for k in range(P)]

    def _callback(self, ctx, send, recv, bytes_p, displs_p, nranks, stream):
        try:
            nbytes = [int(bytes_p[k]) for k in range(nranks)]
            displs = [int(displs_p[k]) for k in range(nranks)]
            s = torch.cuda.ExternalStream(stream, device=self.device) if stream else \
                torch.cuda.default_stream(self.device)
            s.synchronize()  # the packed send block is produced on the caller's stream
            me = dist.get_rank(self.group)
            hs = _dev_view(send, nbytes[me], self.device).cpu() if nbytes[me] else torch.empty(0, dtype=torch.uint8)
            blocks = self.allgatherv_host(hs, nbytes)
            with torch.cuda.stream(s):
                for k in range(nranks):
                    if nbytes[k]:
                        _dev_view(recv + displs[k], nbytes[k], self.device).copy_(blocks[k])
            s.synchronize()
            return 0
        except Exception as e:  # never raise through the C ABI: report, return failure
            import sys
            self.errors.append(repr(e))
            print(f"TorchAllgatherv: {e!r}", file=sys.stderr, flush=True)
            return 1


_NCCL_IDS = {}


def attach(T, world, rank, group=None, nccl=None):
    """Shard handle T as rank `rank` of `world` and attach the exchange transport:
    NCCL when the default process group is NCCL (or nccl=True), else TorchAllgatherv."""
    if nccl is None:
        nccl = dist.get_backend(group) == "nccl"
    if nccl:
        # one NCCL unique id per process group: the library shares the communicator between
        # every handle attached with it (ncclCommInitRank runs once)
        key = id(group)
        if key not in _NCCL_IDS:
            obj = [comm_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0, group=group)
            _NCCL_IDS[key] = obj[0]
        T.comm_attach(world, rank, _NCCL_IDS[key])
        return None
    tr = TorchAllgatherv(group)
    T.comm_attach_transport(world, rank, tr.cfn)
    T._torch_transport = tr
    return tr
