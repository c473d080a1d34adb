"""Timeline of the fused persistent forward (csrc/encoder_fused.cu) from its task trace.

    python tools/fused_trace.py [bert-base] [L] [b] > gpurun_out/fused_trace.txt

Runs a batch-b forward of the fused runtime with arlo_debug_fused_trace enabled and prints,
per (layer, step), when the step's first task became ready, when its last task finished, and
the spread; then the per-step averages over the layers: the critical path of one layer.
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_tanlyl024_b200 import arlo, workload as wl  # noqa: E402

NAMES = ["embed", "qkv", "attn", "oproj", "ln1", "ffn1", "ffn2", "ln2", "pool", "cls"]


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "bert-base"
    L = int(sys.argv[2]) if len(sys.argv) > 2 else 64
    b = int(sys.argv[3]) if len(sys.argv) > 3 else 1
    cfg = wl.CONFIGS[name]
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16), arlo.BF16)
    rt = arlo.Runtime(W, L, b, arlo.RUNTIME_FUSED)
    lens = np.full(b, L, np.int32)
    ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L, seed=5)).cuda()
    ld = torch.from_numpy(lens).cuda()
    out = torch.empty((b, 2), device="cuda")
    for _ in range(5):
        rt.enqueue(b, ids, ld, out)
    buf = torch.zeros(16 * 200000, dtype=torch.int64, device="cuda")
    arlo.check(arlo.lib.arlo_debug_fused_trace(buf.data_ptr()))
    rt.enqueue(b, ids, ld, out)
    torch.cuda.synchronize()
    arlo.check(arlo.lib.arlo_debug_fused_trace(None))
    tr = buf.cpu().numpy().reshape(-1, 16)
    tr = tr[tr[:, 1] != 0]
    t0 = tr[:, 1].min()
    meta = tr[:, 0]
    typ, layer = meta & 0xFF, (meta >> 8) & 0xFFFF
    cta = (meta >> 52) & 0xFFF
    beg, rdy, end, pdep = (tr[:, 1] - t0) / 1e3, (tr[:, 2] - t0) / 1e3, (tr[:, 3] - t0) / 1e3, tr[:, 4]
    # clock64 slots -> globaltimer ns with each CTA's rate
    rate = {}
    for c in set(((tr[:, 0] >> 52) & 0xFFF).tolist()):
        m = np.where(((tr[:, 0] >> 52) & 0xFFF) == c)[0]
        i0, i1 = m[np.argmin(tr[m, 1])], m[np.argmax(tr[m, 1])]
        dt = tr[i1, 1] - tr[i0, 1]
        rate[c] = (tr[i1, 15] - tr[i0, 15]) / dt if dt > 10000 else 1.93
    r = np.array([rate[c] for c in ((tr[:, 0] >> 52) & 0xFFF).tolist()])
    for k in list(range(5, 15)):
        ok = tr[:, k] > 0
        tr[ok, k] = (tr[ok, 1] + (tr[ok, k] - tr[ok, 15]) / r[ok]).astype(np.int64)
    body = (tr[:, 5] - t0) / 1e3
    pdep = np.where(pdep > 0, (pdep - t0) / 1e3, np.nan)
    print(f"{name} L={L} b={b}: {len(tr)} tasks on {len(set(cta.tolist()))} CTAs, span {end.max():.2f} us")
    print(f"{'layer':>5} {'step':>6} {'n':>4} {'ready0':>8} {'ready1':>8} {'end0':>8} {'end1':>8} {'work':>7} {'body':>6} {'pdep1':>8}")
    steps = {}
    for l in sorted(set(layer.tolist())):
        for ty in range(10):
            m = (layer == l) & (typ == ty)
            if not m.any():
                continue
            r0, r1, e0, e1 = rdy[m].min(), rdy[m].max(), end[m].min(), end[m].max()
            work = float(np.median(end[m] - rdy[m]))
            bw = float(np.median(body[m] - rdy[m]))
            pd = np.nanmax(pdep[m]) if np.isfinite(pdep[m]).any() else float("nan")
            print(f"{l:5d} {NAMES[ty]:>6} {m.sum():4d} {r0:8.2f} {r1:8.2f} {e0:8.2f} {e1:8.2f} {work:7.2f} {bw:6.2f} {pd:8.2f}")
            steps.setdefault(ty, []).append((r1, e1, work, bw))
    print("per-step medians over layers: last ready -> last end, median task work (us)")
    prev_end = {}
    for ty, v in sorted(steps.items()):
        v = np.array(v)
        print(f"  {NAMES[ty]:>6}: ready1->end1 {np.median(v[:, 1] - v[:, 0]):6.2f}  work {np.median(v[:, 2]):6.2f}"
              f"  body {np.median(v[:, 3]):6.2f}")
    # sub-stamps (us): GEMM units: pdep(4) -> A issued(12) -> first stage full(13) -> last MMA
    # committed(14) -> ready(2) -> first chunk in smem(6) -> synced(7) -> epilogue done(8) ->
    # tempty(9) -> bulk done(10) -> proxy fence(11) -> end(3)
    def med(m, x, y):
        a_, b_ = tr[m, x], tr[m, y]
        ok = (a_ > 0) & (b_ > 0)
        return float(np.median((b_[ok] - a_[ok]) / 1e3)) if ok.any() else float("nan")
    rv = np.array(list(rate.values()))
    print(f"SM clock during the forward: median {np.median(rv):.3f} GHz (min {rv.min():.3f}, max {rv.max():.3f})")
    print("sub-stamp medians (us), layers >= 1")
    chain = [(4, 12), (12, 13), (13, 14), (14, 2), (2, 6), (6, 7), (7, 8), (8, 9), (9, 10), (10, 11), (11, 3)]
    for ty in (1, 3, 5, 6):
        m = (typ == ty) & (layer >= 1)
        print(f"  {NAMES[ty]:>6}: " + "  ".join(f"{x}->{y} {med(m, x, y):5.2f}" for x, y in chain))
    for ty in (2, 4, 7):
        m = (typ == ty) & (layer >= 1)
        print(f"  {NAMES[ty]:>6}: ready->6 {med(m, 2, 6):5.2f}  6->7 {med(m, 6, 7):5.2f}  7->5 {med(m, 7, 5):5.2f}"
              f"  6->5 {med(m, 6, 5):5.2f}  5->end {med(m, 5, 3):5.2f}")
    rt.close()


if __name__ == "__main__":
    main()
