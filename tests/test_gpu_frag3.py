"""-m gpu: the frag3 kernel's options against the oracle (§8(a) A6/A7).

* SF_LAUNCH_DETERMINISTIC: the A7 two-pass carry combine -- parity, bitwise identical
  output across runs, bit-exact on exact-integer data, heavy rows spanning many groups
  and shards.
* group partition edge cases: fewer nonzeros than lane groups.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_cluster_linwds24_b200 as sf
from tests import gpu_util as G

pytestmark = pytest.mark.gpu

FRAG = sf.KERNEL_FRAG


def _det(th=512, C=128):
    return sf.Launch.make(kernel=FRAG, block_threads=th, chunk_nnz=C, flags=sf.LAUNCH_DETERMINISTIC)


@pytest.mark.parametrize("name", ["tiny", "tiny_skew"])
def test_deterministic_parity_and_reproducible(cuda_device, name):
    cfg = synth.CONFIGS[name]
    inds, vals = synth.config_tensor(cfg, val_kind="signed")
    facs = synth.gen_factors(cfg.dims, cfg.rank, cfg.fseed, "signed")
    for n in range(cfg.nmodes):
        for L in (_det(), _det(1024, 16), _det(128, 256)):
            runs = [G.run(cfg.dims, inds, vals, facs, cfg.rank, modes=[n], launch=L)[0][n] for _ in range(3)]
            G.assert_parity(runs[0], cfg.dims, inds, vals, facs, cfg.rank, n)
            for y in runs[1:]:
                assert np.array_equal(y.view(np.uint32), runs[0].view(np.uint32))
            info = G.run(cfg.dims, inds, vals, facs, cfg.rank, modes=[n], launch=L)[1][n]
            assert info["launch"]["staged_mask"] == 0  # the option forces an unstaged plan


def test_deterministic_heavy_rows_and_shards(cuda_device):
    """A row with ~40 % of the nonzeros spans hundreds of lane groups; shards split it."""
    dims, R = (50, 300, 400), 32
    inds, vals = synth.gen_coo(dims, 60000, 41, zipf=(2.5, 0.5, 0.5), val_kind="int")
    facs = synth.gen_factors(dims, R, 42, "int")
    Y, S = oracle.mttkrp(dims, inds, vals, facs, R, 0)
    assert np.max(S) < 2 ** 24
    Yg, _ = G.run(dims, inds, vals, facs, R, modes=[0], launch=_det(1024, 16))
    assert np.array_equal(Yg[0].astype(np.float64), Y)
    acc = np.zeros_like(Y)
    for p in range(3):
        Yp, _ = G.run(dims, inds, vals, facs, R, modes=[0], launch=_det(256, 32), shard=(3, p))
        acc += Yp[0]
    assert np.array_equal(acc, Y)
    # signed data: reproducible bits, within tolerance
    inds, vals = synth.gen_coo(dims, 60000, 43, zipf=(2.5, 0.5, 0.5), val_kind="signed")
    facs = synth.gen_factors(dims, R, 44, "signed")
    a = G.run(dims, inds, vals, facs, R, modes=[0], launch=_det(1024, 16))[0][0]
    b = G.run(dims, inds, vals, facs, R, modes=[0], launch=_det(1024, 16))[0][0]
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    G.assert_parity(a, dims, inds, vals, facs, R, 0)


def test_plan_deterministic_python_api(cuda_device):
    cfg = synth.CONFIGS["tiny_skew"]
    inds, vals = synth.config_tensor(cfg)
    facs = synth.config_factors(cfg)
    dev = torch.device("cuda:0")
    with sf.Tensor(cfg.dims, G.dev_inds(inds), G.dev_f(vals)) as t:
        t.plan(0, cfg.rank, deterministic=True)
        assert t.plan_info(0, cfg.rank)["launch"]["flags"] & sf.LAUNCH_DETERMINISTIC
        y = torch.empty((cfg.dims[0], cfg.rank), device=dev)
        t.mttkrp(0, [G.dev_f(f) for f in facs], y)
        torch.cuda.synchronize()
        G.assert_parity(y.cpu().numpy(), cfg.dims, inds, vals, facs, cfg.rank, 0)


@pytest.mark.parametrize("nnz", [1, 5, 37, 130, 1025])
def test_fewer_nonzeros_than_groups(cuda_device, nnz):
    """1024-thread CTAs x 148+ SMs >> nnz: most lane groups get empty sub-ranges."""
    dims, R = (40, 30, 20), 32
    inds, vals = synth.gen_coo(dims, nnz, 51, zipf=(0.5, 0.5, 0.5), val_kind="signed")
    facs = synth.gen_factors(dims, R, 52, "signed")
    for L in (sf.Launch.make(kernel=FRAG, block_threads=1024, chunk_nnz=16),
              sf.Launch.make(kernel=FRAG, block_threads=1024, chunk_nnz=16, staged={1: 7}),
              _det(1024, 16)):
        Y, _ = G.run(dims, inds, vals, facs, R, launch=L)
        for n in range(3):
            G.assert_parity(Y[n], dims, inds, vals, facs, R, n)


@pytest.mark.parametrize("dims", [
    (524289, 524289, 524289, 524289, 65536),   # 20+20+20+20+16 = 96 bits: packed 16-byte records
    (524289, 524289, 524289, 524289, 65537),   # 97 bits: unpacked 32-byte records
    (3000, 524289, 70, 524289),                # N = 4 packed, mixed widths (fields straddle words)
])
def test_record_packing_boundaries(cuda_device, dims):
    R = 16
    inds, vals = synth.gen_coo(dims, 20000, 61, zipf=(0.9,) * len(dims), val_kind="int")
    facs = synth.gen_factors(dims, R, 62, "int")
    for staged in (False, True):
        def L(n):
            if not staged:
                return sf.Launch.make(kernel=FRAG, chunk_nnz=64)
            m = min((m for m in range(len(dims)) if m != n), key=lambda m: dims[m])
            return sf.Launch.make(kernel=FRAG, chunk_nnz=64, staged={m: 97})
        Y, _ = G.run(dims, inds, vals, facs, R, launch=L)
        for n in range(len(dims)):
            Yo, S = oracle.mttkrp(dims, inds, vals, facs, R, n)
            assert np.max(S) < 2 ** 24
            assert np.array_equal(Y[n].astype(np.float64), Yo), (dims, n, staged)


@pytest.mark.parametrize("hot_kb", [1, 4])
def test_deterministic_with_hot_rows(cuda_device, hot_kb):
    """The A7 deterministic combine on a hot-row plan (hot slots gathered from the per-call
    dense copy): parity with the oracle and bitwise reproducible across runs; 3- and 4-way."""
    for dims, R in (((300, 200, 150), 32), ((40, 50, 60, 30), 16)):
        inds, vals = synth.gen_coo(dims, 30011, 17, zipf=(1.2,) * len(dims), val_kind="signed")
        facs = synth.gen_factors(dims, R, 18, "signed")
        for n in range(len(dims)):
            L = sf.Launch.make(kernel=FRAG, block_threads=1024, chunk_nnz=64, flags=sf.LAUNCH_DETERMINISTIC,
                               hot_kb=hot_kb)
            runs = [G.run(dims, inds, vals, facs, R, modes=[n], launch=L)[0][n] for _ in range(2)]
            G.assert_parity(runs[0], dims, inds, vals, facs, R, n)
            assert np.array_equal(runs[0].view(np.uint32), runs[1].view(np.uint32))
