import os, sys
sys.path.insert(0, os.getcwd())
import torch, synth, paper_conf_cluster_linwds24_b200 as sf
cfg = synth.CONFIGS["nell1"]
inds, vals = synth.config_tensor_device(cfg)
facs = synth.config_factors_device(cfg)
with sf.Tensor(cfg.dims, inds, vals) as T:
    del inds, vals
    T.cp_als(facs, iters=1)
    torch.cuda.synchronize()
    T.cp_als(facs, iters=1)
    torch.cuda.synchronize()
