"""Pins for the integer preprocessing oracle (oracle/plan.py) against brute force
written differently (Python tuple sorts and dict counts)."""
import numpy as np
import pytest

from oracle import plan


def _coo(seed, dims, nnz):
    rng = np.random.default_rng(seed)
    inds = [rng.integers(0, d, nnz).astype(np.uint32) for d in dims]
    for a in inds:  # duplicates and equal keys
        a[nnz // 2:nnz // 2 + 5] = a[:5]
    return inds


@pytest.mark.parametrize("dims", [(13, 7, 11), (5, 9, 4, 6), (300, 2, 5000)])
def test_matricized_order_brute(dims):
    inds = _coo(1, dims, 700)
    N = len(dims)
    for n in range(N):
        # reading R10: secondary = smallest gathered dim, ties -> higher mode index
        cand = [m for m in range(N) if m != n]
        s = sorted(cand, key=lambda m: (dims[m], -m))[0]
        ref = sorted(range(700), key=lambda e: (int(inds[n][e]), int(inds[s][e]), e))
        assert list(plan.matricized_order(dims, inds, n)) == ref


@pytest.mark.parametrize("nranks", [1, 2, 3, 8])
def test_plan_order_tiles_and_shards_brute(nranks):
    dims = (40, 33, 57)
    inds = _coo(2, dims, 900)
    staged = (1, 2)
    br = {1: 8, 2: 10}
    for n in (0,):
        s = 1  # smallest gathered dim (33 < 57)
        base = sorted(range(900), key=lambda e: (int(inds[n][e]), int(inds[s][e]), e))
        allpos = []
        for p in range(nranks):
            lo, hi = plan.shard_range(900, nranks, p)
            local = base[lo:hi]

            def tile(e):
                q1 = int(inds[1][e]) // 8
                q2 = int(inds[2][e]) // 10
                return q1 * ((57 + 9) // 10) + q2
            ref = sorted(local, key=lambda e: (tile(e), int(inds[n][e]), int(inds[s][e]), e))
            got = list(plan.plan_order(dims, inds, n, staged, br, nranks, p))
            assert got == ref
            allpos += got
        assert sorted(allpos) == list(range(900))


def test_shard_ranges_cover():
    for nnz in (0, 1, 7, 1000, 10**9 + 7):
        for P in (1, 2, 3, 4, 8):
            r = [plan.shard_range(nnz, P, p) for p in range(P)]
            assert r[0][0] == 0 and r[-1][1] == nnz
            assert all(r[p][1] == r[p + 1][0] for p in range(P - 1))
            assert max(b - a for a, b in r) - min(b - a for a, b in r) <= 1


def test_chunks_properties():
    rng = np.random.default_rng(3)
    t = np.sort(rng.integers(0, 20, 5000)).astype(np.uint64)
    for C in (1, 7, 64, 10000):
        ch = plan.chunks(t, C)
        assert ch[0, 0] == 0 and ch[-1, 1] == len(t)
        assert np.all(ch[1:, 0] == ch[:-1, 1])
        assert np.all(ch[:, 1] - ch[:, 0] <= C) and np.all(ch[:, 1] > ch[:, 0])
        for a, b, tile in ch:
            assert np.all(t[a:b] == tile)
        # a new chunk starts at every tile change
        changes = set(np.flatnonzero(t[1:] != t[:-1]) + 1)
        assert changes <= set(ch[:, 0].tolist())


def test_features_brute():
    dims = (50, 20, 70)
    inds = _coo(4, dims, 3000)
    for n in range(3):
        f = plan.features(dims, inds, n)
        s = sorted([m for m in range(3) if m != n], key=lambda m: (dims[m], -m))[0]
        sl, fb = {}, {}
        for e in range(3000):
            i = int(inds[n][e])
            sl[i] = sl.get(i, 0) + 1
            k = (i, int(inds[s][e]))
            fb[k] = fb.get(k, 0) + 1
        assert f["num_slices"] == len(sl) and f["num_fibers"] == len(fb)
        assert f["max_nnz_per_slice"] == max(sl.values())
        assert f["max_nnz_per_fiber"] == max(fb.values())
        assert f["sum_sq_nnz_per_slice"] == sum(c * c for c in sl.values())
        h = np.zeros(40, np.int64)
        for c in sl.values():
            h[c.bit_length() - 1] += 1
        assert np.array_equal(f["slice_hist"], h)
        assert f["slice_ratio"] == len(sl) / dims[n]
        assert f["fiber_ratio"] == len(fb) / len(sl)


def _golden_plan():
    import json
    import os
    return json.load(open(os.path.join(os.path.dirname(__file__), "golden", "plan_chunks_shards.json")))


@pytest.mark.parametrize("case", _golden_plan()["chunks"], ids=lambda c: str(c["tiles"])[:24] + f"/C{c['C']}")
def test_chunks_golden(case):
    """Hand-computed chunk lists (tests/golden/plan_chunks_shards.json, R9)."""
    got = plan.chunks(np.array(case["tiles"], dtype=np.uint64), case["C"])
    assert got.tolist() == case["expect"], case["why"]


@pytest.mark.parametrize("case", _golden_plan()["shard_range"], ids=lambda c: f"{c['nnz']}/{c['P']}")
def test_shard_range_golden(case):
    """Hand-computed floor(p*nnz/P) cuts, incl. the nell-1 / amazon 8-GPU cuts."""
    P = case["P"]
    got = [plan.shard_range(case["nnz"], P, p) for p in range(P)]
    cuts = case["cuts"]
    assert got == [(cuts[p], cuts[p + 1]) for p in range(P)], case["why"]
