"""The device generator (synth/csrc/sfgen_cuda.cu) draws bit-identically to the host one."""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("name", ["tiny", "tiny_skew", "deli4d"])
def test_device_generator_matches_host(cuda_device, name):
    cfg = synth.CONFIGS[name]
    lo = min(12345, cfg.nnz // 3)
    hi = min(cfg.nnz, lo + 300_000)
    hi_ = [a for a in synth.config_tensor(cfg, lo, hi)[0]]
    hv = synth.config_tensor(cfg, lo, hi)[1]
    di, dv = synth.config_tensor_device(cfg, lo=lo, hi=hi)
    for m in range(cfg.nmodes):
        assert np.array_equal(di[m].cpu().numpy().view(np.uint32), hi_[m])
    assert np.array_equal(dv.cpu().numpy(), hv)
    hf = synth.gen_factors(cfg.dims[:1], cfg.rank, cfg.fseed)
    df = synth.gen_factors_device(cfg.dims[:1], cfg.rank, cfg.fseed)
    assert np.array_equal(df[0].cpu().numpy(), hf[0])
