"""Per-CTA pipeline timeline of one tcgen05 GEMM launch (globaltimer stamps).

    python tools/gemm_trace.py M N K [BN] [EPI]      BN < 0 = CTA-pair kernel; EPI 0 bias, 1 GELU, 2 residual,
                                                     3 / 4 / 5 LayerNorm fold (arlo_op_gemm_fold)
Slots per CTA: 0 start (after setup), 1 end; per tile i: 2+6i producer starts tile,
3+6i MMA got accumulator, 4+6i first stage landed, 5+6i last MMA issued,
6+6i epilogue got tile, 7+6i epilogue done (warp 0).
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402

M, N, K = (int(x) for x in sys.argv[1:4])
bn = int(sys.argv[4]) if len(sys.argv) > 4 else 256
epi = int(sys.argv[5]) if len(sys.argv) > 5 else 0
dev = torch.device("cuda")
A = torch.randn(M, K, device=dev).to(torch.bfloat16)
W = (0.02 * torch.randn(N, K, device=dev)).to(torch.bfloat16)
b = torch.zeros(N, device=dev)
R = torch.randn(M, N, device=dev).to(torch.bfloat16) if epi in (2, 5) else None
out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
v1, v2 = torch.rand(N, device=dev) + 0.5, torch.rand(N, device=dev)
st_in = torch.rand((N if epi == 5 else K) // 32, M, 2, device=dev) + 1
st_out = torch.zeros(N // 32, M, 2, device=dev)


def launch():
    if epi >= 3:  # LayerNorm-fold epilogues (arlo_op_gemm_fold)
        arlo.op_gemm_fold(A, W, b, out, epi, v1=v1, v2=v2 if epi == 5 else None, st_in=st_in,
                          st_out=st_out if epi == 5 else None, residual=R, force_bn=bn)
    else:
        arlo.op_gemm(arlo.BF16, A, W, b, out, epi=epi, residual=R, force_bn=bn)


for _ in range(3):
    launch()
buf = torch.zeros(148 * 64, dtype=torch.int64, device=dev)
arlo.check(arlo.lib.arlo_debug_gemm_trace(buf.data_ptr()))
launch()
torch.cuda.synchronize()
arlo.check(arlo.lib.arlo_debug_gemm_trace(None))
t = buf.cpu().numpy().reshape(148, 64).astype(np.float64)
grid = int((t[:, 0] > 0).sum())
t = t[:grid]
t0 = t[:, 0].min()
rel = np.where(t > 0, (t - t0) / 1e3, np.nan)  # microseconds
print(f"M={M} N={N} K={K} BN={bn} epi={epi} grid={grid}  kernel span {np.nanmax(rel[:, 1]):.2f} us (from first CTA start)")
print("start spread: min %.2f max %.2f us" % (np.nanmin(rel[:, 0]), np.nanmax(rel[:, 0])))
main, epil, wait = [], [], []
for i in range(10):
    cols = rel[:, 2 + 6 * i: 8 + 6 * i]
    if np.all(np.isnan(cols[:, 1])):
        break
    med = np.nanmedian(cols, axis=0)
    print(f"tile {i}: producer {med[0]:7.2f} | mma acc {med[1]:7.2f} first-stage {med[2]:7.2f} last-mma {med[3]:7.2f}"
          f" | epi start {med[4]:7.2f} done {med[5]:7.2f}   (median over CTAs, us)")
    main.append(np.nanmedian(cols[:, 3] - cols[:, 1]))
    epil.append(np.nanmedian(cols[:, 5] - cols[:, 4]))
    if i > 0:
        prev = rel[:, 2 + 6 * (i - 1): 8 + 6 * (i - 1)]
        wait.append(np.nanmedian(cols[:, 1] - prev[:, 3]))
print("per tile (median): mainloop issue span %s" % " ".join(f"{x:.2f}" for x in main))
print("                   epilogue span       %s" % " ".join(f"{x:.2f}" for x in epil))
print("                   MMA idle before acc %s" % " ".join(f"{x:.2f}" for x in wait))
print("end: median %.2f max %.2f us" % (np.nanmedian(rel[:, 1]), np.nanmax(rel[:, 1])))

# clock64 sub-stamps of warp 0's epilogue on each CTA's first tile (slots 32..63): 32 epi start,
# 33 first TMEM chunk in registers, then per chunk k: 34+5k start, 35+5k math done, 36+5k staging
# buffer free, 37+5k TMA store issued, 38+5k next chunk's TMEM load landed
raw = buf.cpu().numpy().reshape(148, 64)[:grid].astype(np.float64)
if (raw[:, 33] > 0).any():
    d = lambda a, b: np.median(raw[:, b] - raw[:, a])
    print("epilogue warp 0, first tile (median cycles): start->tmem %.0f" % d(32, 33))
    for k in range(6):
        if (raw[:, 34 + 5 * k] > 0).sum() < grid // 2:
            break
        print("  chunk %d: math %.0f  stg-wait %.0f  smem+store %.0f  tmem-wait %.0f  (from start %.0f)" % (
            k, d(34 + 5 * k, 35 + 5 * k), d(35 + 5 * k, 36 + 5 * k), d(36 + 5 * k, 37 + 5 * k), d(37 + 5 * k, 38 + 5 * k),
            d(32, 38 + 5 * k)))
