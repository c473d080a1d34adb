import numpy as np, torch, sys
sys.path.insert(0, '.')
from paper_conf_icpp_tanlyl024_b200 import arlo, workload as wl
from oracle import encoder as orc
for dtype in (1, 0):
    cfg = wl.TINY
    w = wl.make_weights(cfg)
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, w, dtype), dtype)
    lengths = np.array([32, 17, 1, 2], np.int32)
    ids = wl.sample_token_ids(cfg, lengths, 32, seed=5)
    ref = orc.forward_batch(cfg, w, ids, lengths)
    for rep in range(3):
        rt = arlo.Runtime(W, 32, 4)
        out = np.zeros((4, 2), np.float32)
        rt.infer(ids, lengths, out)
        print(dtype, rep, np.max(np.abs(out - ref)), out.tolist(), flush=True)
        rt.close()
