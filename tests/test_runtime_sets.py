"""derive_set (replay.py, used by tools/runtime_sets.py): the runtime set read off a latency staircase (CPU)."""
from paper_conf_icpp_tanlyl024_b200.replay import derive_runtime_set as derive_set


def test_derive_set_paper_staircase():
    """A TensorRT-like staircase: flat within each 64-token step, +20 % per step -> the paper's
    eight runtimes 64, 128, ..., 512."""
    curve = {L: 1.0 * 1.2 ** ((L - 1) // 64) for L in range(16, 513, 16)}
    assert derive_set(curve) == [64, 128, 192, 256, 320, 384, 448, 512]


def test_derive_set_flat_and_steps():
    assert derive_set({L: 1.0 for L in range(16, 513, 16)}) == [512]  # no step: one runtime (ST)
    curve = {L: (1.0 if L <= 128 else 1.5 if L <= 320 else 2.0) for L in range(16, 513, 16)}
    assert derive_set(curve) == [128, 320, 512]
    # drift within the 5 % tolerance does not open a step
    curve = {L: 1.0 + 0.0009 * (L // 16) for L in range(16, 513, 16)}
    assert derive_set(curve) == [512]
