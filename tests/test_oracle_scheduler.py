"""Pins for oracle/scheduler.py: the paper's worked example (golden fixture)
and hand-derived cases of Algorithm 1 and of the program Eqs. 1-7."""
import json
import os

import numpy as np
import pytest

from oracle import scheduler as osch

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _queue_from(fx):
    q = osch.MultiLevelQueue(fx["max_len"], [len(o) for o in fx["outstanding"]], fx["capacity"])
    q.outstanding = [list(o) for o in fx["outstanding"]]
    return q


def test_fig5_worked_example():
    with open(os.path.join(GOLDEN, "fig5_dispatch.json")) as f:
        fx = json.load(f)
    q = _queue_from(fx)
    assert osch.candidate_runtimes(q, fx["length"]) == [1, 2, 3]  # "(Q2, Q3, and Q4)"
    assert 54 / 60 > fx["lambda"]                                  # Q2 rejected
    assert abs(fx["lambda"] * fx["alpha"] - fx["expected_lambda_at_Q3"]) < 1e-12
    assert 28 / 48 < fx["expected_lambda_at_Q3"]                   # Q3 accepted
    r, i = osch.dispatch(q, fx["length"], fx["lambda"], fx["alpha"], fx["peek"])
    assert (r, i) == (fx["expected_runtime_index"], fx["expected_instance_index"])
    assert q.outstanding[2][0] == 29                               # UPDATE (line 22)


def test_fallback_to_first_candidate_when_all_congested():
    # lines 18-19: every head at P >= lambda -> top candidate's head instance
    q = osch.MultiLevelQueue([64, 128, 256], [2, 1, 1], [10, 10, 10])
    q.outstanding = [[9, 10], [9], [8]]
    assert osch.dispatch(q, 10, 0.85, 0.9, 6) == (0, 0)
    assert q.outstanding[0] == [10, 10]


def test_threshold_decays_per_level():
    # level 0 P=0.9 (>=0.85), level 1 P=0.77 (>=0.765), level 2 P=0.68 (< 0.6885) -> level 2
    q = osch.MultiLevelQueue([64, 128, 256], [1, 1, 1], [100, 100, 100])
    q.outstanding = [[90], [77], [68]]
    assert osch.dispatch(q, 10, 0.85, 0.9, 6) == (2, 0)
    q.outstanding = [[90], [77], [69]]   # 0.69 >= 0.6885 -> all fail -> fallback to level 0
    assert osch.dispatch(q, 10, 0.85, 0.9, 6) == (0, 0)


def test_peek_limit_and_no_candidate():
    # lines 3-4: only the first L candidates are peeked
    q = osch.MultiLevelQueue([64, 128, 256], [1, 1, 1], [10, 10, 10])
    q.outstanding = [[10], [10], [0]]
    assert osch.dispatch(q, 10, 0.85, 0.9, 2) == (0, 0)   # level 2 is beyond the peek limit
    q.outstanding = [[10], [10], [0]]
    assert osch.dispatch(q, 10, 0.85, 0.9, 3) == (2, 0)
    assert osch.dispatch(q, 300, 0.85, 0.9, 3) is None    # no runtime with max_len >= 300
    # a level without instances is not a candidate (reading S16)
    q2 = osch.MultiLevelQueue([64, 128], [0, 1], [10, 10])
    assert osch.dispatch(q2, 10, 0.85, 0.9, 6) == (1, 0)


def test_head_is_least_loaded_lowest_id():
    q = osch.MultiLevelQueue([512], [3], [10])
    q.outstanding = [[2, 1, 1]]
    assert osch.dispatch(q, 5, 0.85, 0.9, 6) == (0, 1)
    assert osch.dispatch(q, 5, 0.85, 0.9, 6) == (0, 2)
    osch.complete(q, 0, 0)
    assert osch.dispatch(q, 5, 0.85, 0.9, 6) == (0, 0)


# ------------------------------------------------------------------ Eqs. 1-7
LAT1 = [float(b) for b in range(1, 33)]        # L_1(b) = b
LAT2 = [2.0 * b for b in range(1, 33)]         # L_2(b) = 2b


def test_ilp_single_gpu_forces_longest_runtime():
    # Eq. 2 + Eq. 7 at G = 1: N = (0, 1); C_2 = Q_1 + Q_2 = 5, B_2 = 5, obj = 2*5*5 = 50
    N, val = osch.allocate(1, [3.0, 2.0], [20.0, 20.0], [LAT1, LAT2])
    assert N == (0, 1) and abs(val - 50.0) < 1e-12


def test_ilp_hand_computed_two_runtimes():
    # (1,1): C1=10,B1=10 -> 10*10; C2=2,B2=2 -> 4*2   => 108
    # (0,2): C1=0; R1=10; C2=12, B2=6 -> 12*12          => 144
    N, val = osch.allocate(2, [10.0, 2.0], [20.0, 20.0], [LAT1, LAT2])
    assert N == (1, 1) and abs(val - 108.0) < 1e-12
    assert abs(osch.objective((0, 2), [10.0, 2.0], [20.0, 20.0], [LAT1, LAT2]) - 144.0) < 1e-12
    assert osch.objective((2, 0), [10.0, 2.0], [20.0, 20.0], [LAT1, LAT2]) is None  # Eq. 7


def test_ilp_eq3_floor_and_spill():
    # Eq. 3: N_1 >= floor(50/20) = 2; G = 3 -> only (2,1).
    # C1 = min(50, 40) = 40, B1 = 20 -> 20*40 = 800; R1 = 10; C2 = 11, B2 = 11 -> 22*11 = 242
    N, val = osch.allocate(3, [50.0, 1.0], [20.0, 20.0], [LAT1, LAT2])
    assert N == (2, 1) and abs(val - 1042.0) < 1e-12
    assert osch.allocate(1, [50.0, 1.0], [20.0, 20.0], [LAT1, LAT2]) is None


def test_ilp_interpolation_and_clamp():
    # B = 2.5 interpolates between L(2) and L(3); B = 0.5 clamps to L(1); B > nb clamps to L(nb)
    assert osch.interp_latency([1.0, 2.0, 4.0], 2.5) == 3.0
    assert osch.interp_latency([1.0, 2.0, 4.0], 0.5) == 1.0
    assert osch.interp_latency([1.0, 2.0, 4.0], 9.0) == 4.0


def test_compositions_count():
    from math import comb
    for G, I in [(8, 8), (5, 3), (1, 4)]:
        comps = list(osch.compositions(G, I))
        assert len(comps) == comb(G + I - 1, I - 1) == len(set(comps))
        assert all(sum(c) == G and len(c) == I for c in comps)


# ------------------------------------------------------------------ instance replacement (L272)
@pytest.mark.parametrize("cur,N_new,expected", [
    ((0, 0, 1, 2), (1, 2, 1), 1),        # GPU 1 leaves runtime 0 (oversubscribed) for runtime 1
    ((0, 1, 1, 2), (1, 2, 1), 0),        # allocation unchanged
    ((-1, -1, -1), (2, 1), 3),           # cold start: every GPU loads an instance
    ((2, 2, 2, 2), (1, 1, 1, 1), 3),     # one GPU keeps runtime 2, three are replaced
    ((0, 1, 2), (0, 0, 2), 2),           # runtimes 0, 1 dropped; GPU 2 keeps runtime 2
    ((0, 1, -1), (1, 1, 0), 0),          # a spare GPU stays spare
])
def test_replace_plan_hand_cases(cur, N_new, expected):
    nxt, changed = osch.replace_plan(list(cur), list(N_new))
    assert changed == expected
    assert all(nxt.count(i) == n for i, n in enumerate(N_new))


def test_replace_plan_matches_matching_bound():
    """The minimum number of changed GPUs equals G minus the largest number of GPUs that can keep
    their state: sum_i min(c_i, N_i) over runtimes plus min(c_-1, spare) idle GPUs (a bipartite
    matching of equal labels), on random tiny cases."""
    rng = np.random.default_rng(7)
    for _ in range(200):
        G, I = int(rng.integers(1, 6)), int(rng.integers(1, 4))
        cur = [int(v) for v in rng.integers(-1, I, size=G)]
        cuts = np.sort(rng.integers(0, G + 1, size=I))
        N_new = [int(v) for v in np.diff(np.concatenate([[0], cuts]))]
        spare = G - sum(N_new)
        keep = sum(min(cur.count(i), N_new[i]) for i in range(I)) + min(cur.count(-1), spare)
        _nxt, changed = osch.replace_plan(cur, N_new)
        assert changed == G - keep
