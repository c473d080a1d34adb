"""Per-CTA timeline of one bf16 attention launch (globaltimer stamps).

    python tools/attn_trace.py B L heads len
Slots: 0 start (after setup), 1 end, 2 S_0 issued (Q/K_0 landed), per key tile j:
3+3j S ready (softmax warp 0), 4+3j max pass done (+ PV_{j-1} wait), 5+3j P written.
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
buf = torch.zeros(2048 * 32, dtype=torch.int64, device=dev)
arlo.check(arlo.lib.arlo_debug_attn_trace(buf.data_ptr()))
arlo.op_attention(arlo.BF16, B, L, heads, qkv, lens, out)
torch.cuda.synchronize()
arlo.check(arlo.lib.arlo_debug_attn_trace(None))
t = buf.cpu().numpy().reshape(2048, 32).astype(np.float64)
live = t[:, 0] > 0
t = t[live]
t0 = t[:, 0].min()
rel = np.where(t > 0, (t - t0) / 1e3, np.nan)
print(f"B={B} L={L} heads={heads} len={n}: {live.sum()} CTAs traced; span {np.nanmax(rel[:, 1]):.2f} us")
dur = rel[:, 1] - rel[:, 0]
print(f"CTA duration median {np.nanmedian(dur):.2f} us  min {np.nanmin(dur):.2f}  max {np.nanmax(dur):.2f}")
d = rel - rel[:, :1]
names = ["start", "end", "S0 issued"] + [f"{k}{j}" for j in range(4) for k in ("S", "max", "P")]
med = np.nanmedian(d, axis=0)
print(" ".join(f"{nm}={m:.2f}" for nm, m in zip(names, med) if not np.isnan(m)))
starts = np.sort(rel[:, 0])
print("CTA start times (first 10 / every 148th):", np.round(starts[:10], 2), np.round(starts[::148], 2))
