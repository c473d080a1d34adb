"""Work accounting for the roofline (SURVEY.md §8(a) totals, §8(d)); no compute.

F(b, L) = layers * (2bLH*3H + 2bLH*H + 2*2bLH*F + 4bL^2H) + b*(2H^2 + 2HC)
(= layers*(24bLH^2 + 4bL^2H) + b(2H^2 + 2HC) when F = 4H): the static-shape
FLOPs one runtime forward at (b, L) executes.  "Useful" work is the same
formula at each request's own length.
"""
from __future__ import annotations


def forward_flops(cfg, b: int, L: int) -> float:
    H, F, C = cfg.hidden, cfg.ffn, cfg.num_labels
    per_layer = 2 * b * L * H * 3 * H + 2 * b * L * H * H + 2 * 2 * b * L * H * F + 4 * b * L * L * H
    return float(cfg.layers * per_layer + b * (2 * H * H + 2 * H * C))


def useful_flops(cfg, lengths) -> float:
    return float(sum(forward_flops(cfg, 1, int(n)) for n in lengths))


def gemm_flops(M: int, N: int, K: int) -> float:
    return 2.0 * M * N * K


def ln_bytes(M: int, H: int, elem: int = 2) -> float:
    """Algorithmic HBM bytes of one LayerNorm launch: read y, write x (gamma/beta L2-resident)."""
    return float(2 * M * H * elem)


def embed_bytes(M: int, H: int, elem: int = 2) -> float:
    """Embedding+LN: gather word row + position row (type row L2-resident), write x, read ids."""
    return float(3 * M * H * elem + 4 * M)
