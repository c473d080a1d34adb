"""Runtimes on several devices of one process (needs >= 2 B200s; skipped otherwise).

Kernel attributes (>48 KB shared memory opt-in) are per device context: a runtime built on
the second device must launch the same kernels, and two host threads building and serving
runtimes on two devices at once must get bitwise the logits of one device."""
import threading

import numpy as np
import pytest
import torch

from paper_conf_icpp_tanlyl024_b200 import workload as wl

pytestmark = pytest.mark.gpu


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs two GPUs")
def test_two_devices_two_threads_bitwise(arlo_lib):
    cfg = wl.BERT_BASE
    w = wl.make_weights(cfg)
    lengths = wl.sample_lengths(8, seed=5, lo=0, hi=128)
    ids = wl.sample_token_ids(cfg, lengths, 128, seed=6)
    out = {}

    def serve(dev):
        with torch.cuda.device(dev):
            W = arlo_lib.Weights(cfg, arlo_lib.upload_weights(cfg, w, arlo_lib.BF16, f"cuda:{dev}"), arlo_lib.BF16,
                                 dev)
            rt = arlo_lib.Runtime(W, 128, 8)
            o = np.zeros((8, 2), np.float32)
            rt.infer(ids, lengths, o)
            out[dev] = o
            rt.close()
            W.close()

    ts = [threading.Thread(target=serve, args=(d,)) for d in (0, 1)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    np.testing.assert_array_equal(out[0], out[1])
