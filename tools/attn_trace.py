"""Per-CTA timeline of one bf16 attention launch (globaltimer + clock64 stamps).

    python tools/attn_trace.py B L heads len
Slots: 0/1 start/end, per 64-key chunk c (c < 8): 3+3c S ready (softmax warp 0),
4+3c exp done, 5+3c P handed over; 32+c S(0,c) issued (c < 16), 48+c PV(0,c) issued (c < 14).
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402

B, L, heads, n = (int(x) for x in sys.argv[1:5])
dev = torch.device("cuda")
qkv = torch.randn(B * L, 3 * 64 * heads, device=dev).to(torch.bfloat16)
lens = torch.full((B,), n, dtype=torch.int32, device=dev)
out = torch.empty(B * L, 64 * heads, device=dev, dtype=torch.bfloat16)
for _ in range(3):
    arlo.op_attention(arlo.BF16, B, L, heads, qkv, lens, out)
buf = torch.zeros(2048 * 64, dtype=torch.int64, device=dev)
arlo.check(arlo.lib.arlo_debug_attn_trace(buf.data_ptr()))
arlo.op_attention(arlo.BF16, B, L, heads, qkv, lens, out)
torch.cuda.synchronize()
arlo.check(arlo.lib.arlo_debug_attn_trace(None))
t = buf.cpu().numpy().reshape(2048, 64).astype(np.float64)
live = t[:, 0] > 0
t = t[live]
gt0, gt1, ck0, ck1 = t[:, 0], t[:, 1], t[:, 62], t[:, 63]
ghz = np.median((ck1 - ck0) / (gt1 - gt0))
t00 = gt0.min()
print(f"B={B} L={L} heads={heads} len={n}: {live.sum()} CTAs traced; span {(gt1.max() - t00) / 1e3:.2f} us; "
      f"SM clock {ghz:.3f} GHz")
dur = (gt1 - gt0) / 1e3
print(f"CTA duration median {np.median(dur):.2f} us  min {dur.min():.2f}  max {dur.max():.2f}")
# within-CTA times from clock64, in us since the CTA's start
d = np.where(t > 0, (t - ck0[:, None]) / ghz / 1e3, np.nan)
d[:, 0] = 0.0
d[:, 1] = dur
names = ["start", "end", "-"] + [f"{k}{j}" for j in range(8) for k in ("S", "exp", "P")]
med = np.nanmedian(d[:, :27], axis=0)
print(" ".join(f"{nm}={m:.2f}" for nm, m in zip(names, med) if not np.isnan(m) and nm != "-"))
starts = np.sort((gt0 - t00) / 1e3)
print("CTA start times (first 10 / every 148th):", np.round(starts[:10], 2), np.round(starts[::148], 2))
mmed = np.nanmedian(d[:, 32:62], axis=0)
print("S(0,c) issued:", " ".join(f"{x:.2f}" for x in mmed[:16] if not np.isnan(x)))
print("PV(0,c) issued:", " ".join(f"{x:.2f}" for x in mmed[16:30] if not np.isnan(x)))
