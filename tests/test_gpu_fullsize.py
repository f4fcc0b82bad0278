"""Full-size parity at BASELINE.json's configs, in the launch configuration the
selector picks (the one bench.py times): sampled output rows against the oracle
computed row by row (oracle.mttkrp_rows streams every nonzero once), plus
properties that hold at any size (empty rows exactly 0, finite output, exact
integer features)."""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_cluster_linwds24_b200 as sf
from tests import gpu_util as G

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def _sample_rows(rng, inds_n, dim, k=48):
    cnt = np.bincount(inds_n, minlength=dim)
    nonempty = np.flatnonzero(cnt)
    empty = np.flatnonzero(cnt == 0)
    rows = {int(np.argmax(cnt)), int(nonempty[0]), int(nonempty[-1])}
    rows |= set(int(x) for x in rng.choice(nonempty, size=min(k, len(nonempty)), replace=False))
    # the rows around the heaviest row and a few light ones
    light = np.flatnonzero(cnt == 1)
    if len(light):
        rows |= set(int(x) for x in rng.choice(light, size=min(4, len(light)), replace=False))
    emp = rng.choice(empty, size=min(4, len(empty)), replace=False) if len(empty) else np.zeros(0, int)
    return np.array(sorted(rows)), emp, cnt


@pytest.mark.parametrize("name", ["nell2", "deli4d", "nell1"])
def test_fullsize_sampled_rows(cuda_device, name):
    cfg = synth.CONFIGS[name]
    inds, vals = synth.config_tensor(cfg)
    facs = synth.config_factors(cfg)
    R = cfg.rank
    rng = np.random.default_rng(cfg.seed)
    h_inds = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    h_vals = torch.from_numpy(vals).pin_memory()
    d_facs = [torch.from_numpy(f).cuda() for f in facs]
    with sf.Tensor(cfg.dims, h_inds, h_vals) as T:
        for n in range(cfg.nmodes):
            T.plan(n, R)
            info = T.plan_info(n, R)
            y = torch.full((cfg.dims[n], R), float("nan"), device="cuda")
            T.mttkrp(n, d_facs, y)
            torch.cuda.synchronize()
            rows, empty, cnt = _sample_rows(rng, inds[n], cfg.dims[n])
            # features at full size (integer-exact)
            f = info["features"]
            assert f["num_slices"] == int(np.count_nonzero(cnt))
            assert f["max_nnz_per_slice"] == int(cnt.max())
            Yr, Sr = oracle.mttkrp_rows(cfg.dims, inds, vals, facs, R, n, rows)
            got = y[torch.from_numpy(rows).cuda()].cpu().numpy()
            rel, zv = oracle.max_rel_err(got, Yr, Sr)
            assert rel <= G.TOL, (name, n, rel, info["launch"])
            if len(empty):
                assert not y[torch.from_numpy(empty).cuda()].any()
            assert torch.isfinite(y).all()


def _streamed_check(dims, inds, vals, facs, R, n, rows, segments=8, streams=4):
    h_inds = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    h_vals = torch.from_numpy(vals).pin_memory()
    d_facs = [torch.from_numpy(f).cuda() for f in facs]
    y = torch.full((dims[n], R), float("nan"), device="cuda")
    sf.mttkrp_streamed(dims, h_inds, h_vals, d_facs, n, y, segments, streams)
    Yr, Sr = oracle.mttkrp_rows(dims, inds, vals, facs, R, n, rows)
    got = y[torch.from_numpy(rows).cuda()].cpu().numpy()
    rel, zv = oracle.max_rel_err(got, Yr, Sr)
    assert torch.isfinite(y).all()
    return rel


def test_streamed_fullsize_nell2(cuda_device):
    """A8 (ii) at BASELINE.json configs[1] size: the sorted-segment streamed path from pinned
    host COO, sampled rows (incl. the heaviest) within the north-star tolerance."""
    cfg = synth.CONFIGS["nell2"]
    inds, vals = synth.config_tensor(cfg)
    facs = synth.config_factors(cfg)
    rng = np.random.default_rng(3)
    for n in range(cfg.nmodes):
        rows, _, _ = _sample_rows(rng, inds[n], cfg.dims[n], k=24)
        rel = _streamed_check(cfg.dims, inds, vals, facs, cfg.rank, n, rows)
        assert rel <= G.TOL, (n, rel)


@pytest.mark.parametrize("name", ["nell2", "deli4d"])
def test_streamed_modes_fullsize(cuda_device, name):
    """sf_mttkrp_streamed_modes at BASELINE.json configs[1] / configs[2] size: every mode from ONE
    upload of the pinned host COO (the bench's one-shot e2e path; 16- and 32-byte segment
    records), sampled rows incl. the heaviest within the north-star tolerance, empty rows exactly 0."""
    cfg = synth.CONFIGS[name]
    inds, vals = synth.config_tensor(cfg)
    facs = synth.config_factors(cfg)
    R = cfg.rank
    rng = np.random.default_rng(5)
    h_inds = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    h_vals = torch.from_numpy(vals).pin_memory()
    d_facs = [torch.from_numpy(f).cuda() for f in facs]
    outs = [torch.full((d, R), float("nan"), device="cuda") for d in cfg.dims]
    sf.mttkrp_streamed_modes(cfg.dims, h_inds, h_vals, d_facs, outs, 16, 4)
    torch.cuda.synchronize()
    for n in range(cfg.nmodes):
        rows, empty, _ = _sample_rows(rng, inds[n], cfg.dims[n], k=24)
        Yr, Sr = oracle.mttkrp_rows(cfg.dims, inds, vals, facs, R, n, rows)
        got = outs[n][torch.from_numpy(rows).cuda()].cpu().numpy()
        rel, _ = oracle.max_rel_err(got, Yr, Sr)
        assert rel <= G.TOL, (n, rel)
        if len(empty):
            assert not outs[n][torch.from_numpy(empty).cuda()].any()
        assert torch.isfinite(outs[n]).all()


def test_streamed_heavy_row(cuda_device):
    """SURVEY C-2: one row holding a large share of 2e7 nonzeros (amazon mode 3 has 1.2e8 in one
    row) -- the sorted-segment kernel pre-reduces it in registers, so the fp32 atomic chain
    stays short and the row meets 1e-4."""
    dims, R, nnz = (50, 4000, 3000), 16, 20_000_000
    inds, vals = synth.gen_coo(dims, nnz, 41, zipf=(2.5, 0.5, 0.5))
    facs = synth.gen_factors(dims, R, 42)
    cnt = np.bincount(inds[0], minlength=dims[0])
    assert cnt.max() > 0.3 * nnz  # a genuinely heavy row
    rows = np.array(sorted({int(np.argmax(cnt)), 0, 1, 2, int(np.argmin(cnt))}))
    for segments, streams in ((8, 4), (3, 2)):
        rel = _streamed_check(dims, inds, vals, facs, R, 0, rows, segments, streams)
        assert rel <= G.TOL, (segments, rel)


def test_streamed_device_footprint(cuda_device):
    """F2 (tensors larger than HBM): the streamed path holds only
    streams x segment buffers on the device (sf_device_bytes), not the tensor."""
    cfg = synth.CONFIGS["nell2"]
    inds, vals = synth.config_tensor(cfg)
    h_inds = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    h_vals = torch.from_numpy(vals).pin_memory()
    d_facs = synth.config_factors_device(cfg)
    y = torch.empty((cfg.dims[0], cfg.rank), device="cuda")
    tensor_bytes = 4 * (cfg.nmodes + 1) * cfg.nnz
    sf.device_bytes(reset_peak=True)
    base, _ = sf.device_bytes()
    sf.mttkrp_streamed(cfg.dims, h_inds, h_vals, d_facs, 0, y, 32, 4)
    torch.cuda.synchronize()
    _, peak = sf.device_bytes()
    # 4 ring slots of one 1/32 segment each (raw arrays + sort scratch ~ 2.5x the raw bytes)
    assert peak - base < 0.5 * tensor_bytes, (peak - base, tensor_bytes)
