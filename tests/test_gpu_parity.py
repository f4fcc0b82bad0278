"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Floating point: max |Y_gpu - Y| / S <= 1e-4 per element (north_star), S the
|.|-scale; rows without contributions must be exactly 0.  Exact-integer data
(values {1..4}, factors {-2..2}, all partial sums < 2^24) must match bitwise.
Integer preprocessing (perm, chunks, features) must match oracle/plan.py ==.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_cluster_linwds24_b200 as sf
from oracle import plan as oplan
from tests import gpu_util as G

pytestmark = pytest.mark.gpu

FRAG, COO = sf.KERNEL_FRAG, sf.KERNEL_COO


def _cfg_data(name, val_kind="unit", fac_kind="unit"):
    cfg = synth.CONFIGS[name]
    inds, vals = synth.config_tensor(cfg, val_kind=val_kind)
    facs = synth.gen_factors(cfg.dims, cfg.rank, cfg.fseed, fac_kind)
    return cfg, inds, vals, facs


@pytest.mark.parametrize("name", ["tiny", "tiny_skew"])
def test_configs0_all_modes_auto(cuda_device, name):
    cfg, inds, vals, facs = _cfg_data(name)
    Y, info = G.run(cfg.dims, inds, vals, facs, cfg.rank)
    for n in range(cfg.nmodes):
        G.assert_parity(Y[n], cfg.dims, inds, vals, facs, cfg.rank, n)


def _launches(dims, n):
    """Launch variants; chunk_nnz is a per-warp chunk."""
    others = [m for m in range(len(dims)) if m != n]
    yield sf.Launch.make(kernel=COO)
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=16, staged={})
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=128, block_threads=256, staged={})
    # stage every gathered mode in small blocks: many tiles, ragged last block
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=32, staged={m: max(1, dims[m] // 3 + 1) for m in others})
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=64, block_threads=1024, staged={others[0]: 7})
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=256, block_threads=128, ctas_per_sm=1,
                         staged={others[-1]: dims[others[-1]]})
    # L2 tiles (SF_LAUNCH_L2_TILES): tiled order, no shared-memory staging, every CTA takes a
    # share of every tile; one and two tiled modes, ragged last block
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=32, staged={others[-1]: max(1, dims[others[-1]] // 4 + 1)},
                         flags=sf.LAUNCH_L2_TILES)
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=64, block_threads=256,
                         staged={m: max(1, dims[m] // 3 + 1) for m in others}, flags=sf.LAUNCH_L2_TILES)
    # hot-row cache (launch.hot_kb): a budget of a few rows (only the most frequent rows are
    # hot), every row hot, with L2 tiles, with shared-memory staging, with memset + atomics
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=48, hot_kb=1)
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=64, hot_kb=1 << 16)
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=64, staged={others[-1]: max(1, dims[others[-1]] // 4 + 1)},
                         flags=sf.LAUNCH_L2_TILES, hot_kb=2)
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=48, staged={others[0]: 7}, hot_kb=2)
    yield sf.Launch.make(kernel=FRAG, chunk_nnz=100, flags=sf.LAUNCH_NO_OWNER_STORES, hot_kb=3)


@pytest.mark.parametrize("name", ["tiny", "tiny_skew"])
def test_launch_variants(cuda_device, name):
    cfg, inds, vals, facs = _cfg_data(name, "signed", "signed")
    for n in range(cfg.nmodes):
        for L in _launches(cfg.dims, n):
            try:
                Y, _ = G.run(cfg.dims, inds, vals, facs, cfg.rank, modes=[n], launch=L)
            except sf.SfError as e:
                raise AssertionError(f"mode {n} launch {L.as_dict()}: {e}")
            G.assert_parity(Y[n], cfg.dims, inds, vals, facs, cfg.rank, n)


@pytest.mark.parametrize("R", [16, 32, 64, 1, 7, 12])
@pytest.mark.parametrize("dims", [(100, 80, 60), (300, 200), (10, 12, 14, 16), (5, 6, 4, 3, 7)])
def test_ranks_and_orders(cuda_device, R, dims):
    nnz = 3001  # ragged
    inds, vals = synth.gen_coo(dims, nnz, 99, zipf=(0.8,) * len(dims), val_kind="signed")
    facs = synth.gen_factors(dims, R, 77, "signed")
    for staged, flags, hot in ((False, 0, 0), (True, 0, 0), (True, sf.LAUNCH_L2_TILES, 0), (False, 0, 1),
                               (True, sf.LAUNCH_L2_TILES, 1)):
        def L(n):
            if not staged:
                return sf.Launch.make(kernel=FRAG, chunk_nnz=100, hot_kb=hot)
            # L2 tiles: one tiled mode, so the others can take hot rows
            st = {m: max(1, dims[m] // 2) for m in range(len(dims)) if m != n}
            if flags:
                st = {max(st): st[max(st)]}
            return sf.Launch.make(kernel=FRAG, chunk_nnz=100, flags=flags, staged=st, hot_kb=hot)
        Y, _ = G.run(dims, inds, vals, facs, R, launch=L)
        for n in range(len(dims)):
            G.assert_parity(Y[n], dims, inds, vals, facs, R, n)


def test_exact_integers_bitwise(cuda_device):
    dims, R = (200, 150, 170), 32
    inds, vals = synth.gen_coo(dims, 20000, 5, zipf=(1.0, 1.0, 1.0), val_kind="int")
    facs = synth.gen_factors(dims, R, 6, "int")
    for n in range(3):
        Y, S = oracle.mttkrp(dims, inds, vals, facs, R, n)
        assert np.max(S) < 2 ** 24
        for L in _launches(dims, n):
            Yg, _ = G.run(dims, inds, vals, facs, R, modes=[n], launch=L)
            assert np.array_equal(Yg[n].astype(np.float64), Y), L.as_dict()


def _run_case(kind):
    """Index sets whose slice / fiber runs start, end and cross the feature kernel's 256-key
    warp tiles in every way: single nonzero, one run of exactly a tile, runs one past a tile,
    mixed run lengths, a heavy slice spanning hundreds of tiles."""
    rng = np.random.default_rng(17)
    if kind == "one":
        return (3, 4, 5), [np.array([2], np.uint32), np.array([1], np.uint32), np.array([4], np.uint32)]
    if kind in ("tile", "tile+1", "tile-1"):
        n = 256 + {"tile": 0, "tile+1": 1, "tile-1": -1}[kind]
        return (3, 4, 5), [np.full(n, 1, np.uint32), np.full(n, 2, np.uint32), np.full(n, 3, np.uint32)]
    if kind == "mixed":
        lens = [300, 1, 255, 256, 1, 1, 700, 2, 257, 513, 3, 1024]
        i0 = np.concatenate([np.full(L, k, np.uint32) for k, L in enumerate(lens)])
        n = len(i0)
        i1 = (rng.integers(0, 3, n) * (rng.random(n) < 0.9)).astype(np.uint32)  # long fibers too
        i2 = rng.integers(0, 40, n).astype(np.uint32)
        perm = rng.permutation(n)
        return (len(lens), 3, 40), [i0[perm], i1[perm], i2[perm]]
    # heavy: one slice of mode 0 holds half the nonzeros
    n = 100003
    i0 = np.where(rng.random(n) < 0.5, 0, rng.integers(0, 5000, n)).astype(np.uint32)
    i1 = rng.integers(0, 3, n).astype(np.uint32)
    i2 = rng.integers(0, 70000, n).astype(np.uint32)
    return (5000, 3, 70000), [i0, i1, i2]


@pytest.mark.parametrize("kind", ["one", "tile", "tile+1", "tile-1", "mixed", "heavy"])
def test_features_run_edges(cuda_device, kind):
    dims, inds = _run_case(kind)
    vals = np.ones(len(inds[0]), np.float32)
    with sf.Tensor(dims, G.dev_inds(inds), G.dev_f(vals)) as t:
        for n in range(3):
            f = t.features(n)
            of = oplan.features(dims, inds, n)
            for k in ("num_slices", "num_fibers", "max_nnz_per_slice", "max_nnz_per_fiber",
                      "sum_sq_nnz_per_slice", "secondary"):
                assert f[k] == of[k], (kind, n, k)
            assert f["slice_hist"] == list(of["slice_hist"]), (kind, n)


def test_plan_bit_exact_vs_oracle(cuda_device):
    dims = (300, 41, 530)
    inds, vals = synth.gen_coo(dims, 25000, 8, zipf=(1.0, 0.5, 0.8))
    facs = synth.gen_factors(dims, 16, 9)
    ti, tv = G.dev_inds(inds), G.dev_f(vals)
    with sf.Tensor(dims, ti, tv) as t:
        for n in range(3):
            f = t.features(n)
            of = oplan.features(dims, inds, n)
            for k in ("num_slices", "num_fibers", "max_nnz_per_slice", "max_nnz_per_fiber",
                      "sum_sq_nnz_per_slice", "secondary"):
                assert f[k] == of[k], k
            assert f["slice_hist"] == list(of["slice_hist"])
            others = [m for m in range(3) if m != n]
            for staged, flags in (({}, 0), ({others[0]: 13}, 0), ({others[0]: 40, others[1]: 7}, 0),
                                  ({others[1]: 50}, sf.LAUNCH_L2_TILES)):
                L = sf.Launch.make(kernel=FRAG, chunk_nnz=100, staged=staged, flags=flags)
                t.set_launch(n, 16, L)
                perm, chunks = t.plan_export(n, 16)
                ref = oplan.plan_order(dims, inds, n, tuple(sorted(staged)), staged)
                assert np.array_equal(perm.astype(np.int64), ref)
                tiles = oplan.tile_ids(dims, inds, tuple(sorted(staged)), staged, sel=ref)
                ref_chunks = oplan.chunks(tiles, 100)
                assert np.array_equal(chunks.astype(np.int64), ref_chunks)
                info = t.plan_info(n, 16)
                assert info["num_tiles"] == len(np.unique(tiles))


def test_shards_emulated_on_one_gpu(cuda_device):
    """§8(e): P shards of the matricized order; their outputs sum to the 1-GPU result
    (exact on integer data); each shard touches only its row range."""
    dims, R = (120, 90, 70), 16
    inds, vals = synth.gen_coo(dims, 15000, 21, zipf=(1.2, 0.5, 0.5), val_kind="int")
    facs = synth.gen_factors(dims, R, 22, "int")
    for n in range(3):
        Yfull, _ = oracle.mttkrp(dims, inds, vals, facs, R, n)
        for P in (2, 3, 8):
            acc = np.zeros_like(Yfull)
            perm0 = oplan.matricized_order(dims, inds, n)
            for p in range(P):
                Y, info = G.run(dims, inds, vals, facs, R, modes=[n], shard=(P, p))
                lo, hi = oplan.shard_range(len(vals), P, p)
                rows = inds[n][perm0[lo:hi]]
                assert info[n]["nnz_local"] == hi - lo
                if hi > lo:
                    assert info[n]["row_begin"] == rows.min() and info[n]["row_end"] == rows.max() + 1
                outside = np.ones(dims[n], bool)
                outside[info[n]["row_begin"]:info[n]["row_end"]] = False
                assert not Y[n][outside].any()
                acc += Y[n]
            assert np.array_equal(acc, Yfull)


def test_host_inputs_pageable_and_pinned(cuda_device):
    cfg, inds, vals, facs = _cfg_data("tiny_skew")
    Y, _ = G.run(cfg.dims, inds, vals, facs, cfg.rank, device_input=False)
    for n in range(3):
        G.assert_parity(Y[n], cfg.dims, inds, vals, facs, cfg.rank, n)
    # pinned torch host tensors, many segments / streams
    ti = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    tv = torch.from_numpy(vals).pin_memory()
    tf = [G.dev_f(f) for f in facs]
    with sf.Tensor(cfg.dims, ti, tv, segments=7, streams=3) as t:
        for n in range(3):
            t.plan(n, cfg.rank)
            y = torch.empty((cfg.dims[n], cfg.rank), device="cuda:0")
            t.mttkrp(n, tf, y)
            torch.cuda.synchronize()
            G.assert_parity(y.cpu().numpy(), cfg.dims, inds, vals, facs, cfg.rank, n)


@pytest.mark.parametrize("segments,streams", [(1, 1), (4, 4), (13, 3)])
def test_streamed_one_shot(cuda_device, segments, streams):
    cfg, inds, vals, facs = _cfg_data("tiny_skew", "signed", "signed")
    tf = [G.dev_f(f) for f in facs]
    for n in range(3):
        y = torch.full((cfg.dims[n], cfg.rank), float("nan"), device="cuda:0")
        sf.mttkrp_streamed(cfg.dims, inds, vals, tf, n, y, segments, streams)
        G.assert_parity(y.cpu().numpy(), cfg.dims, inds, vals, facs, cfg.rank, n)


@pytest.mark.parametrize("dims,R,nnz,mask", [
    ((100, 80, 60), 16, 10_000, (1, 1, 1)),        # 16-byte records, every mode
    ((100, 80, 60), 32, 10_000, (1, 0, 1)),        # a subset of modes (A_2 still gathered)
    ((30, 20, 40, 7), 32, 20_000, (1, 1, 1, 1)),   # N = 4: 32-byte records
    ((9, 11, 13, 5, 3), 64, 5_000, (0, 1, 0, 1, 1)),
    ((100, 80, 60), 12, 10_000, (1, 1, 1)),        # rank outside 16/32/64: one atomic per nonzero
])
@pytest.mark.parametrize("segments,streams", [(1, 1), (5, 3), (16, 4)])
def test_streamed_modes_one_shot(cuda_device, dims, R, nnz, mask, segments, streams):
    """sf_mttkrp_streamed_modes: one upload of the host COO, every requested mode computed from
    each segment (A8 (ii)); each Y against the fp64 oracle."""
    inds, vals = synth.gen_coo(dims, nnz, 77, zipf=(1.0,) * len(dims), val_kind="signed")
    facs = synth.gen_factors(dims, R, 78, "signed")
    tf = [G.dev_f(f) for f in facs]
    outs = [torch.full((dims[n], R), float("nan"), device="cuda:0") if mask[n] else None
            for n in range(len(dims))]
    if sum(mask) == 1:  # the one computed mode's factor may be NULL
        tf[mask.index(1)] = None
    sf.mttkrp_streamed_modes(dims, inds, vals, tf, outs, segments, streams)
    torch.cuda.synchronize()
    for n in range(len(dims)):
        if mask[n]:
            G.assert_parity(outs[n].cpu().numpy(), dims, inds, vals, facs, R, n)


def test_streamed_modes_edge(cuda_device):
    """Empty tensor (every Y exactly 0), N = 8 (beyond the record widths: one atomic per
    nonzero), and a single nonzero on a 2-way tensor with more segments than nonzeros."""
    dims, R = (10, 9, 8), 16
    facs = [G.dev_f(f) for f in synth.gen_factors(dims, R, 6)]
    outs = [torch.full((d, R), 7.0, device="cuda:0") for d in dims]
    e = [np.zeros(0, np.uint32)] * 3
    sf.mttkrp_streamed_modes(dims, e, np.zeros(0, np.float32), facs, outs, 4, 2)
    assert all(not o.any() for o in outs)
    dims8 = (3, 4, 5, 3, 4, 5, 3, 4)
    inds, vals = synth.gen_coo(dims8, 3000, 9, val_kind="signed")
    facs8 = synth.gen_factors(dims8, R, 10, "signed")
    outs = [torch.full((d, R), float("nan"), device="cuda:0") for d in dims8]
    sf.mttkrp_streamed_modes(dims8, inds, vals, [G.dev_f(f) for f in facs8], outs, 3, 2)
    for n in range(8):
        G.assert_parity(outs[n].cpu().numpy(), dims8, inds, vals, facs8, R, n)
    dims2 = (5, 6)
    one = [np.array([4], np.uint32), np.array([2], np.uint32)]
    f2 = synth.gen_factors(dims2, 32, 11)
    outs = [torch.full((d, 32), float("nan"), device="cuda:0") for d in dims2]
    sf.mttkrp_streamed_modes(dims2, one, np.array([0.5], np.float32), [G.dev_f(f) for f in f2], outs, 8, 4)
    for n in range(2):
        G.assert_parity(outs[n].cpu().numpy(), dims2, one, np.array([0.5], np.float32), f2, 32, n)


def test_streamed_modes_orders_after_the_callers_stream(cuda_device):
    """`stream` orders the one-shot work after what the caller queued on it: factors written on
    that stream behind a long-running kernel must be the ones the MTTKRPs read."""
    dims, R = (60, 50, 40), 16
    inds, vals = synth.gen_coo(dims, 20_000, 31, val_kind="signed")
    facs = synth.gen_factors(dims, R, 32, "signed")
    s = torch.cuda.Stream()
    tf = [torch.zeros((d, R), device="cuda:0") for d in dims]
    src = [G.dev_f(f) for f in facs]
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        torch.cuda._sleep(50_000_000)  # ~25 ms of spinning before the factors land
        for t_, f_ in zip(tf, src):
            t_.copy_(f_, non_blocking=True)
    outs = [torch.full((d, R), float("nan"), device="cuda:0") for d in dims]
    sf.mttkrp_streamed_modes(dims, inds, vals, tf, outs, 3, 2, stream=s)
    torch.cuda.synchronize()
    for n in range(3):
        G.assert_parity(outs[n].cpu().numpy(), dims, inds, vals, facs, R, n)


def test_streamed_modes_errors(cuda_device):
    dims, R = (10, 9, 8), 16
    inds, vals = synth.gen_coo(dims, 1000, 5)
    facs = [G.dev_f(f) for f in synth.gen_factors(dims, R, 6)]
    with pytest.raises(sf.SfError):  # no output mode
        sf.mttkrp_streamed_modes(dims, inds, vals, facs, [None, None, None])
    bad = [a.copy() for a in inds]
    bad[1][500] = 9  # == dims[1]
    outs = [torch.empty((d, R), device="cuda:0") for d in dims]
    with pytest.raises(sf.SfError) as ei:
        sf.mttkrp_streamed_modes(dims, bad, vals, facs, outs, 4, 2)
    assert ei.value.status == 2  # SF_ERR_INDEX_OUT_OF_RANGE
    # the offending nonzero was skipped, every other one summed
    keep = np.ones(1000, bool)
    keep[500] = False
    for n in range(3):
        G.assert_parity(outs[n].cpu().numpy(), dims, [a[keep] for a in inds], vals[keep],
                        [f.cpu().numpy() for f in facs], R, n)


def test_edge_cases(cuda_device):
    dims, R = (10, 9, 8), 16
    facs = synth.gen_factors(dims, R, 1)
    tf = [G.dev_f(f) for f in facs]
    # empty tensor -> Y == 0
    e = [np.zeros(0, np.uint32)] * 3
    with sf.Tensor(dims, e, np.zeros(0, np.float32)) as t:
        t.plan(0, R)
        y = torch.full((10, R), 7.0, device="cuda:0")
        t.mttkrp(0, tf, y)
        torch.cuda.synchronize()
        assert not y.any()
    # one nonzero
    one = [np.array([3], np.uint32), np.array([8], np.uint32), np.array([7], np.uint32)]
    Y, _ = G.run(dims, one, np.array([0.5], np.float32), facs, R)
    for n in range(3):
        G.assert_parity(Y[n], dims, one, np.array([0.5], np.float32), facs, R, n)
    # out-of-range index is rejected at create
    bad = [np.array([3], np.uint32), np.array([9], np.uint32), np.array([0], np.uint32)]
    with pytest.raises(sf.SfError) as ei:
        sf.Tensor(dims, G.dev_inds(bad), G.dev_f(np.ones(1, np.float32)))
    assert ei.value.status == 2
    with pytest.raises(sf.SfError) as ei:
        sf.Tensor(dims, bad, np.ones(1, np.float32))
    assert ei.value.status == 2
    # mttkrp before plan
    with sf.Tensor(dims, one, np.ones(1, np.float32)) as t:
        with pytest.raises(sf.SfError) as ei:
            t.mttkrp(0, tf, torch.empty((10, R), device="cuda:0"))
        assert ei.value.status == 4
        with pytest.raises(sf.SfError):
            t.plan(3, R)  # bad mode
    # a single heavy row + a single heavy fiber (atomic chains across chunks)
    n = 50000
    heavy = [np.full(n, 2, np.uint32), np.full(n, 4, np.uint32), np.arange(n, dtype=np.uint32) % 8]
    v = synth.gen_coo((8,), n, 3)[1]
    Y, _ = G.run(dims, heavy, v, facs, R, launch=sf.Launch.make(kernel=FRAG, chunk_nnz=64))
    for m in range(3):
        G.assert_parity(Y[m], dims, heavy, v, facs, R, m)


def test_kernel_launch_counter(cuda_device):
    before = sf.kernel_launches()
    cfg, inds, vals, facs = _cfg_data("tiny")
    G.run(cfg.dims, inds, vals, facs, cfg.rank, modes=[0])
    assert sf.kernel_launches() > before


@pytest.mark.parametrize("dims,R", [((4, 5, 3, 6, 2, 3), 4), ((3, 4, 2, 5, 3, 2, 4, 2), 3),
                                    ((50, 1, 40), 32), ((1, 70, 60), 16), ((20, 30, 25), 128)])
def test_generic_paths_and_degenerate_dims(cuda_device, dims, R):
    """N = 6..8 and R = 128 run the generic COO kernel; size-1 modes; exact integers."""
    nnz = 1500
    inds, vals = synth.gen_coo(dims, nnz, 3, val_kind="int")
    facs = synth.gen_factors(dims, R, 4, "int")
    Y, _ = G.run(dims, inds, vals, facs, R)
    for n in range(len(dims)):
        Yo, S = oracle.mttkrp(dims, inds, vals, facs, R, n)
        assert np.max(S) < 2 ** 24
        assert np.array_equal(Y[n].astype(np.float64), Yo), n


@pytest.mark.parametrize("segments,streams", [(2, 2), (7, 3), (16, 4)])
def test_presort_upload_bit_exact(cuda_device, segments, streams, monkeypatch):
    """A8 upload || presort: per-segment sorted runs merged at the first plan give the same
    matricized order, features, chunks and Y as the full sort (oracle/plan.py ==)."""
    dims = (300, 41, 530)
    inds, vals = synth.gen_coo(dims, 25013, 12, zipf=(1.0, 0.5, 0.8))  # ragged segments
    facs = synth.gen_factors(dims, 16, 13, "signed")
    ti = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    tv = torch.from_numpy(vals).pin_memory()
    tf = [G.dev_f(f) for f in facs]
    for flag in ("", "no_presort"):
        monkeypatch.setenv("SF_DEBUG", flag)
        with sf.Tensor(dims, ti, tv, segments=segments, streams=streams) as t:
            for n in range(3):
                others = [m for m in range(3) if m != n]
                L = sf.Launch.make(kernel=FRAG, chunk_nnz=100, staged={others[0]: 13})
                t.set_launch(n, 16, L)  # first plan of the mode: consumes the merged runs
                f = t.features(n)
                of = oplan.features(dims, inds, n)
                for k in ("num_slices", "num_fibers", "max_nnz_per_slice", "max_nnz_per_fiber"):
                    assert f[k] == of[k], (flag, k)
                perm, chunks = t.plan_export(n, 16)
                ref = oplan.plan_order(dims, inds, n, (others[0],), {others[0]: 13})
                assert np.array_equal(perm.astype(np.int64), ref), (flag, n)
                y = torch.empty((dims[n], 16), device="cuda:0")
                t.mttkrp(n, tf, y)
                torch.cuda.synchronize()
                G.assert_parity(y.cpu().numpy(), dims, inds, vals, facs, 16, n)


@pytest.mark.parametrize("block_rows", [1 << 17, 3 << 17, 100_000])
def test_l2_tiles_of_the_other_mode_bit_exact(cuda_device, block_rows):
    """3-way L2-tiled plans that tile the non-secondary gathered mode o: its coarse index rides
    above the sort key (tile ids without a random gather) when block_rows is a multiple of
    2^17, else the gathered tile keys; same order, chunks, features and Y as the oracle."""
    dims, R = (50_000, 300, 600_000), 16
    inds, vals = synth.gen_coo(dims, 200_003, 21, zipf=(0.9, 0.6, 1.0), val_kind="int")
    facs = synth.gen_factors(dims, R, 22, "int")
    tf = [G.dev_f(f) for f in facs]
    for host in (False, True):
        ti = ([torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds] if host else G.dev_inds(inds))
        tv = torch.from_numpy(vals).pin_memory() if host else G.dev_f(vals)
        with sf.Tensor(dims, ti, tv) as t:
            for n in (0, 1):
                f = t.features(n)
                of = oplan.features(dims, inds, n)
                for k in ("num_slices", "num_fibers", "max_nnz_per_slice", "max_nnz_per_fiber",
                          "sum_sq_nnz_per_slice"):
                    assert f[k] == of[k], (n, k)
                assert f["slice_hist"] == list(of["slice_hist"])
                L = sf.Launch.make(kernel=FRAG, chunk_nnz=64, staged={2: block_rows}, flags=sf.LAUNCH_L2_TILES)
                t.set_launch(n, R, L)
                perm, chunks = t.plan_export(n, R)
                ref = oplan.plan_order(dims, inds, n, (2,), {2: block_rows})
                assert np.array_equal(perm.astype(np.int64), ref), (host, n, block_rows)
                tiles = oplan.tile_ids(dims, inds, (2,), {2: block_rows}, sel=ref)
                assert np.array_equal(chunks.astype(np.int64), oplan.chunks(tiles, 64))
                y = torch.empty((dims[n], R), device="cuda:0")
                t.mttkrp(n, tf, y)
                torch.cuda.synchronize()
                Y, _ = oracle.mttkrp(dims, inds, vals, facs, R, n)
                assert np.array_equal(y.cpu().numpy().astype(np.float64), Y), (host, n)


@pytest.mark.parametrize("segments", [3, 8])
def test_presort_wide_keys_bit_exact(cuda_device, segments, monkeypatch):
    """A handle whose modes mix presorted keys and keys that with the input position need more
    than 64 bits (those are sorted at their first plan, not during the upload): same matricized
    order, features and chunks as the full sort (oracle/plan.py ==).  Position bits 19: mode 2
    (key 1e8 x 1e6, 47 bits) is wide, modes 0 and 1 (1e6 x 2e6, 41 bits) are presorted."""
    dims = (1_000_000, 2_000_000, 100_000_000)
    inds, vals = synth.gen_coo(dims, 300_007, 14, zipf=(1.1, 0.5, 1.1))
    ti = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    tv = torch.from_numpy(vals).pin_memory()
    for flag in ("", "no_presort"):
        monkeypatch.setenv("SF_DEBUG", flag)
        with sf.Tensor(dims, ti, tv, segments=segments, streams=3) as t:
            for n in range(3):
                t.set_launch(n, 16, sf.Launch.make(kernel=FRAG, chunk_nnz=100))
                f = t.features(n)
                of = oplan.features(dims, inds, n)
                for k in ("num_slices", "num_fibers", "max_nnz_per_slice", "max_nnz_per_fiber",
                          "sum_sq_nnz_per_slice"):
                    assert f[k] == of[k], (flag, n, k)
                perm, chunks = t.plan_export(n, 16)
                ref = oplan.plan_order(dims, inds, n, (), {})
                assert np.array_equal(perm.astype(np.int64), ref), (flag, n)
                assert np.array_equal(chunks.astype(np.int64), oplan.chunks(np.zeros(len(ref), np.int64), 100))


@pytest.mark.parametrize("kind", ["l2tiles", "staged", "hot"])
def test_shards_with_tiled_plans(cuda_device, kind):
    """§8(e) with tiled plans: each shard's L2-tiled / shared-memory-tiled / hot-row-cache
    plan covers only its slice of the matricized order; the P partial outputs sum to the
    full result exactly (integer data) and to the oracle; host input (upload || presort)."""
    dims, R = (150, 110, 90), 32
    inds, vals = synth.gen_coo(dims, 24007, 31, zipf=(1.0, 0.6, 0.8), val_kind="int")
    facs = synth.gen_factors(dims, R, 32, "int")
    for n in range(3):
        others = [m for m in range(3) if m != n]
        flags = {"l2tiles": sf.LAUNCH_L2_TILES, "staged": 0, "hot": sf.LAUNCH_L2_TILES}[kind]
        L = sf.Launch.make(kernel=FRAG, chunk_nnz=64, staged={others[-1]: max(1, dims[others[-1]] // 3)},
                           flags=flags, hot_kb=2 if kind == "hot" else 0)
        Yfull, _ = oracle.mttkrp(dims, inds, vals, facs, R, n)
        for P in (2, 5):
            acc = np.zeros_like(Yfull)
            for p in range(P):
                Y, info = G.run(dims, inds, vals, facs, R, modes=[n], launch=L, shard=(P, p), device_input=False)
                acc += Y[n]
            assert np.array_equal(acc, Yfull), (kind, n, P)


def test_smem_optin_never_lowered(cuda_device):
    """Two plans of the same kernel instantiation with different shared-memory needs: the
    smaller plan's occupancy query / launch must not lower the opt-in below what the larger
    plan needs (a later launch of the larger plan failed with "invalid argument")."""
    dims, R = (300, 200, 100), 32
    inds, vals = synth.gen_coo(dims, 20000, 3, zipf=(0.8, 0.8, 0.8))
    facs = synth.gen_factors(dims, R, 4)
    tf = [G.dev_f(f) for f in facs]
    with sf.Tensor(dims, G.dev_inds(inds), G.dev_f(vals)) as t:
        big = sf.Launch.make(kernel=FRAG, block_threads=1024, chunk_nnz=128)
        small = sf.Launch.make(kernel=FRAG, block_threads=256, chunk_nnz=64)
        ys = {}
        for n, L in ((0, big), (1, small), (2, big)):
            t.set_launch(n, R, L)
        for n in (0, 1, 0, 2, 1, 0):
            ys[n] = torch.empty((dims[n], R), device="cuda:0")
            t.mttkrp(n, tf, ys[n])
        torch.cuda.synchronize()
        for n in range(3):
            G.assert_parity(ys[n].cpu().numpy(), dims, inds, vals, facs, R, n)
