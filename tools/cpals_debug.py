import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_cluster_linwds24_b200 as sf
from tests import gpu_util as G
from tests.test_gpu_cpals import _lowrank_coo
for R in (32, 64):
    for fused in ("1", "0"):
        os.environ["SF_CPALS_FUSED"] = fused
        rng = np.random.default_rng(R)
        dims = (60, 50, 40)
        inds, vals = _lowrank_coo(rng, dims, 4, 0.3)
        init = [rng.uniform(0.1, 1.0, (d, R)).astype(np.float32) for d in dims]
        facs = [G.dev_f(a) for a in init]
        with sf.Tensor(dims, G.dev_inds(inds), G.dev_f(vals)) as T:
            try:
                fits = T.cp_als(facs, iters=3)
            except Exception as e:
                fits = str(e)
        print(R, fused, fits, float(facs[0].abs().sum()), flush=True)
