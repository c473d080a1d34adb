"""Where a single post-flush GEMM launch spends its event-timed duration (bench roofline leg).

    python tools/roofline_ctx.py M N K EPI CODE [reps]

  b2b       `reps` back-to-back launches captured in one CUDA graph (PDL chains them), per launch
  single    bench.py's leg: flush (512 MB write), A / residual rewritten, events around ONE launch
  graphsub  graph of reps x [flush, rewrite, GEMM] minus graph of reps x [flush, rewrite], per rep
  span      one post-flush launch with the globaltimer trace on: first CTA start (after setup)
            to last CTA end, and the event time of the same launch
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402

M, N, K, EPI, CODE = (int(x) for x in sys.argv[1:6])
reps = int(sys.argv[6]) if len(sys.argv) > 6 else 20
dev = torch.device("cuda:0")
s = torch.cuda.Stream(dev)
torch.cuda.set_stream(s)
flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
A = torch.randn(M, K, device=dev).to(torch.bfloat16)
W = (0.02 * torch.randn(N, K, device=dev)).to(torch.bfloat16)
bias = torch.zeros(N, device=dev)
R = torch.randn(M, N, device=dev).to(torch.bfloat16) if EPI == 2 else None
out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
A0, R0 = A.clone(), (R.clone() if R is not None else None)


def gemm():
    arlo.op_gemm(arlo.BF16, A, W, bias, out, epi=EPI, residual=R, force_bn=CODE, stream=s)


def prep():
    flush.zero_()
    A.copy_(A0)
    if R is not None:
        R.copy_(R0)


def graph_time(body, n):
    for _ in range(2):
        body()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(n):
            body()
    ts = []
    for _ in range(5):
        g.replay()
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        g.replay()
        e.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(e) * 1e3 / n)
    return float(np.median(ts))


fl = 2.0 * M * N * K
for _ in range(3):
    gemm()
t_b2b = graph_time(gemm, reps)
ev = []
for _ in range(reps):
    prep()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    gemm()
    e.record(s)
    ev.append((a, e))
torch.cuda.synchronize()
t_single = float(np.mean([a.elapsed_time(e) * 1e3 for a, e in ev]))
t_full = graph_time(lambda: (prep(), gemm()), reps)
t_prep = graph_time(prep, reps)
buf = torch.zeros(148 * 64, dtype=torch.int64, device=dev)
spans, evs = [], []
for _ in range(5):
    prep()
    torch.cuda.synchronize()
    buf.zero_()
    arlo.check(arlo.lib.arlo_debug_gemm_trace(buf.data_ptr()))
    prep()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    gemm()
    e.record(s)
    torch.cuda.synchronize()
    arlo.check(arlo.lib.arlo_debug_gemm_trace(None))
    t = buf.cpu().numpy().reshape(148, 64).astype(np.float64)
    t = t[t[:, 0] > 0]
    spans.append((t[:, 1].max() - t[:, 0].min()) / 1e3)
    evs.append(a.elapsed_time(e) * 1e3)
print(f"M={M} N={N} K={K} epi={EPI} code={CODE}: b2b {t_b2b:.2f} us ({fl / t_b2b / 1e6:.0f} TF) | single {t_single:.2f} us "
      f"({fl / t_single / 1e6:.0f} TF) | graphsub {t_full - t_prep:.2f} us (prep {t_prep:.2f}) | traced span "
      f"{np.median(spans):.2f} us vs its events {np.median(evs):.2f} us", flush=True)
