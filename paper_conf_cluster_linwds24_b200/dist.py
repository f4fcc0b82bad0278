"""Multi-GPU boundary-row exchange for row shards.

Each rank owns matricized positions [floor(p*nnz/P), floor((p+1)*nnz/P)) of every mode,
so its partial Y touches a contiguous row range [row_begin, row_end).  Adjacent ranks
share at most the row that straddles a cut (a heavy row may straddle several).  The
owner of a shared row is the LOWEST rank touching it.  Per call:

  1. pack this rank's first/last row partials          (sf_rows_op PACK, my kernel)
  2. all_gather the 2*R-float packets                   (NCCL over NVLink; gloo in CPU tests)
  3. zero this rank's copy of a first row it does not own  (sf_rows_op ZERO)
  4. the owner adds every other rank's partial of its rows (sf_rows_op ADD)

After the call every rank holds the exact (up to fp32 summation order) rows it owns
and zeros elsewhere: a row-sharded Y, the layout CP-ALS's row-local update
A_n = M V^+ (Alg. 1 line 5) consumes.  The owner map depends only on
the plans' row ranges, so it is computed once per plan (one tiny all_gather) and
cached; the per-call exchange is one all_gather of 2*R floats per rank.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def owner_maps(ranges):
    """ranges[k] = (row_begin, row_end) of rank k (row_end == row_begin: empty shard).

    Returns per rank k:
      zero_rows[k]: rows of Y_k to zero (first row owned by a lower rank), list
      add_src[k]:   list of (target_row, src_rank, slot) for the owner k, slot 0 = first
                    row packet of src_rank, 1 = last row packet.
    """
    P = len(ranges)
    first = [ranges[k][0] if ranges[k][1] > ranges[k][0] else None for k in range(P)]
    last = [ranges[k][1] - 1 if ranges[k][1] > ranges[k][0] else None for k in range(P)]

    def owner(row):
        for k in range(P):
            if first[k] is not None and first[k] <= row <= last[k]:
                return k
        return None

    zero_rows = [[] for _ in range(P)]
    add_src = [[] for _ in range(P)]
    for k in range(P):
        if first[k] is None:
            continue
        o = owner(first[k])
        if o != k:
            zero_rows[k].append(first[k])
            add_src[o].append((first[k], k, 0))
        # a shard's last row can be owned by a lower rank only if the whole shard is
        # that single row (then first == last and it was handled above)
    return zero_rows, add_src


class BoundaryExchange:
    """Caches the owner maps per (row_begin, row_end) and runs steps 1-4."""

    def __init__(self, world, rank, R, device, rows_op=None, group=None, host_staging=False):
        """host_staging: run the all_gather on CPU copies (gloo), for multi-rank tests on
        one GPU where NCCL cannot be used (two ranks may not share a device)."""
        self.world, self.rank, self.R, self.device = world, rank, R, device
        self.group = group
        self.host_staging = host_staging
        if rows_op is None:
            from . import rows_op as _rows_op
            rows_op = _rows_op
        self.rows_op = rows_op
        self._cache = {}
        self.send = torch.empty((2, R), dtype=torch.float32, device=device)
        self.recv = torch.empty((2 * world, R), dtype=torch.float32, device=device)
        self._recv_list = list(self.recv.view(world, 2, R).unbind(0))

    def _maps(self, row_begin, row_end):
        key = (int(row_begin), int(row_end))
        if key not in self._cache:
            cdev = "cpu" if self.host_staging else self.device
            mine = torch.tensor([key[0], key[1]], dtype=torch.int64, device=cdev)
            allr = [torch.empty_like(mine) for _ in range(self.world)]
            dist.all_gather(allr, mine, group=self.group)
            ranges = [tuple(int(x) for x in t.cpu().tolist()) for t in allr]
            zero_rows, add_src = owner_maps(ranges)
            me = self.rank
            pack = torch.tensor([ranges[me][0] if ranges[me][1] > ranges[me][0] else -1,
                                 ranges[me][1] - 1 if ranges[me][1] > ranges[me][0] else -1],
                                dtype=torch.int64, device=self.device)
            # gathered buffer is [world * 2, R]; target row per slot (-1 = skip)
            tgt = [-1] * (2 * self.world)
            for row, src, slot in add_src[me]:
                tgt[2 * src + slot] = row
            zero = zero_rows[me] or [-1]
            self._cache[key] = (pack, torch.tensor(tgt, dtype=torch.int64, device=self.device),
                                torch.tensor(zero, dtype=torch.int64, device=self.device), ranges)
        return self._cache[key]

    def combine(self, Y, row_begin, row_end, stream=None):
        pack, tgt, zero, _ = self._maps(row_begin, row_end)
        ctx = torch.cuda.stream(stream) if (stream is not None and Y.is_cuda) else _null()
        with ctx:
            self.rows_op(Y, pack, self.send, 0, stream)
            if self.host_staging:
                if Y.is_cuda:
                    torch.cuda.current_stream().synchronize()
                hs = self.send.cpu()
                hr = [torch.empty_like(hs) for _ in range(self.world)]
                dist.all_gather(hr, hs, group=self.group)
                self.recv.copy_(torch.cat(hr, 0))
            else:
                dist.all_gather(self._recv_list, self.send, group=self.group)
            self.rows_op(Y, zero, None, 2, stream)
            self.rows_op(Y, tgt, self.recv, 1, stream)
        return Y


class StepExchange:
    """Steps 1-4 for several outputs at once (e.g. every mode of a CP-ALS sweep / bench step)
    with ONE all_gather: item i's packets sit at [src][i][slot] of the gathered buffer, so a
    step pays one collective latency instead of one per mode.  Items share the rank R."""

    def __init__(self, world, rank, R, device, rows_op=None, group=None, host_staging=False):
        self.ex = BoundaryExchange(world, rank, R, device, rows_op=rows_op, group=group,
                                   host_staging=host_staging)
        self._cache = {}

    def _layout(self, keys):
        if keys not in self._cache:
            ex, W, K = self.ex, self.ex.world, len(keys)
            per = []
            for i, (rb, re_) in enumerate(keys):
                pack, _, zero, ranges = ex._maps(rb, re_)
                _, add_src = owner_maps(ranges)
                tgt = [-1] * (2 * W * K)
                for row, src, slot in add_src[ex.rank]:
                    tgt[(src * K + i) * 2 + slot] = row
                per.append((pack, zero, torch.tensor(tgt, dtype=torch.int64, device=ex.device)))
            send = torch.empty((K * 2, ex.R), dtype=torch.float32, device=ex.device)
            recv = torch.empty((W * K * 2, ex.R), dtype=torch.float32, device=ex.device)
            self._cache[keys] = (per, send, recv, list(recv.view(W, K * 2, ex.R).unbind(0)))
        return self._cache[keys]

    def combine(self, items, stream=None):
        """items: [(Y, row_begin, row_end), ...]; every Y ends row-sharded (see module doc)."""
        ex = self.ex
        keys = tuple((int(rb), int(re_)) for _, rb, re_ in items)
        per, send, recv, recv_list = self._layout(keys)
        cuda = any(Y.is_cuda for Y, _, _ in items)
        ctx = torch.cuda.stream(stream) if (stream is not None and cuda) else _null()
        with ctx:
            for i, (Y, _, _) in enumerate(items):
                ex.rows_op(Y, per[i][0], send[2 * i:2 * i + 2], 0, stream)
            if ex.host_staging:
                if cuda:
                    torch.cuda.current_stream().synchronize()
                hs = send.cpu()
                hr = [torch.empty_like(hs) for _ in range(ex.world)]
                dist.all_gather(hr, hs, group=ex.group)
                recv.copy_(torch.cat(hr, 0))
            else:
                dist.all_gather(recv_list, send, group=ex.group)
            for i, (Y, _, _) in enumerate(items):
                ex.rows_op(Y, per[i][1], None, 2, stream)
                ex.rows_op(Y, per[i][2], recv, 1, stream)
        return [Y for Y, _, _ in items]


class _null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False
