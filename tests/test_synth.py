"""Generator checks: determinism across chunkings, bijective relabel, table
sanity, and the config shapes against the paper's Table III densities."""
import numpy as np
import pytest

import synth


def test_chunk_invariance():
    cfg = synth.CONFIGS["tiny_skew"]
    full_i, full_v = synth.config_tensor(cfg)
    a_i, a_v = synth.config_tensor(cfg, 0, 3333)
    b_i, b_v = synth.config_tensor(cfg, 3333, cfg.nnz)
    for m in range(3):
        assert np.array_equal(full_i[m], np.r_[a_i[m], b_i[m]])
    assert np.array_equal(full_v, np.r_[a_v, b_v])


def test_indices_in_range_and_values():
    for name in ("tiny", "tiny_skew"):
        cfg = synth.CONFIGS[name]
        inds, vals = synth.config_tensor(cfg)
        for m, d in enumerate(cfg.dims):
            assert inds[m].max() < d
        assert vals.min() > 0 and vals.max() <= 1
    i, v = synth.gen_coo((10, 10), 1000, 1, val_kind="int")
    assert set(np.unique(v)) <= {1, 2, 3, 4}
    i, v = synth.gen_coo((10, 10), 1000, 1, val_kind="signed")
    assert v.min() >= -1 and v.max() < 1 and v.min() < 0
    f = synth.gen_factor(50, 8, 3, 0, "int")
    assert set(np.unique(f)) <= {-2, -1, 0, 1, 2}


@pytest.mark.parametrize("I", [1, 2, 3, 5, 100, 1000, 4097, 65536])
def test_relabel_is_bijection(I):
    xs = np.arange(I, dtype=np.uint64)
    ys = synth.permute(I, 12345, 1, xs)
    assert np.array_equal(np.sort(ys), xs)


@pytest.mark.parametrize("I,s", [(100, 1.0), (28818, 0.5), (25495389, 0.8), (1443, 0.3)])
def test_zipf_table(I, s):
    e, t = synth.zipf_table(I, s)
    assert e[0] == 0 and e[-1] == I and np.all(np.diff(e.astype(np.int64)) > 0)
    assert len(t) == len(e) - 2 and np.all(np.diff(t.astype(np.float64)) >= 0)


def test_skew_is_heavy_headed():
    i_u, _ = synth.gen_coo((10000,), 200000, 5, zipf=(0.0,))
    i_z, _ = synth.gen_coo((10000,), 200000, 5, zipf=(1.0,))
    cu = np.bincount(i_u[0], minlength=10000)
    cz = np.bincount(i_z[0], minlength=10000)
    assert cu.max() < 60
    assert cz.max() > 20 * cu.max()


def test_configs_match_table_III_density():
    """PAPER.md Table III (L256-267) densities (reading R13: exponent minus signs restored)."""
    want = {"nell2": 2.4e-5, "nell1": 9.1e-13, "deli4d": 4.3e-15, "vast": 6.9e-3, "flickr3d": 7.8e-12,
            "deli3d": 6.1e-12, "uber": 3.9e-4, "nips": 1.8e-6, "enron": 5.5e-9, "flickr4d": 1.1e-14}
    for name, dens in want.items():
        c = synth.CONFIGS[name]
        d = c.nnz / float(np.prod([float(x) for x in c.dims]))
        assert abs(d - dens) / dens < 0.05, (name, d)
