"""arlo_allocate / arlo_dispatch (C++) against the oracle schedulers (CPU)."""
import json
import os

import numpy as np
import pytest

from oracle import scheduler as osch

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def load_state(arlo_lib, s, max_len, outstanding):
    """Reach an exact per-instance occupancy through the ABI: with a huge lambda and
    peek = 1 every request of length max_len[k] lands on level k's least-loaded
    instance, so filling each level to max(target) and completing the surplus on
    each instance reproduces `outstanding` exactly."""
    s.set_params(1e18, 1.0, 1)
    for lvl, occ in enumerate(outstanding):
        for _ in range(len(occ) * max(occ)):
            r, _i = s.dispatch(max_len[lvl])
            assert r == lvl
        for inst, target in enumerate(occ):
            for _ in range(max(occ) - target):
                s.complete(lvl, inst)
    for lvl, occ in enumerate(outstanding):
        assert [s.outstanding(lvl, i) for i in range(len(occ))] == occ


def test_fig5_worked_example_through_abi(arlo_lib):
    """lambda=0.85, alpha=0.9, L=3, len 200 -> Q2 54/60 rejected, Q3 28/48 chosen."""
    fx = json.load(open(os.path.join(GOLDEN, "fig5_dispatch.json")))
    s = arlo_lib.Scheduler(fx["max_len"], [len(o) for o in fx["outstanding"]], fx["capacity"])
    load_state(arlo_lib, s, fx["max_len"], fx["outstanding"])
    s.set_params(fx["lambda"], fx["alpha"], fx["peek"])
    assert s.dispatch(fx["length"]) == (fx["expected_runtime_index"], fx["expected_instance_index"])
    assert s.outstanding(2, 0) == 29
    s.close()


def _run_both(max_len, n_inst, cap, lam, alpha, peek, events, seed):
    q = osch.MultiLevelQueue(max_len, n_inst, cap)
    s = arlo_lib_global.Scheduler(max_len, n_inst, cap, lam, alpha, peek)
    rng = np.random.default_rng(seed)
    live = []
    for ev in events:
        if ev > 0:
            ref = osch.dispatch(q, ev, lam, alpha, peek)
            if ref is None:
                with pytest.raises(arlo_lib_global.ArloError) as e:
                    s.dispatch(ev)
                assert e.value.code == arlo_lib_global.ENOCAND
                continue
            got = s.dispatch(ev)
            assert got == ref, (ev, got, ref)
            live.append(got)
        elif live:
            r, i = live.pop(int(rng.integers(len(live))))
            osch.complete(q, r, i)
            s.complete(r, i)
    for r in range(len(max_len)):
        for i in range(n_inst[r]):
            assert s.outstanding(r, i) == q.outstanding[r][i]
    s.close()


arlo_lib_global = None


@pytest.mark.parametrize("seed", range(6))
def test_dispatch_matches_algorithm1_oracle(arlo_lib, seed):
    global arlo_lib_global
    arlo_lib_global = arlo_lib
    rng = np.random.default_rng(seed)
    K = int(rng.integers(1, 9))
    max_len = sorted(rng.choice(np.arange(64, 577, 64), size=K, replace=False).tolist())
    n_inst = rng.integers(0, 5, size=K).tolist()
    n_inst[-1] = max(1, n_inst[-1])
    cap = rng.integers(2, 12, size=K).astype(float).tolist()
    peek = int(rng.integers(1, 8))
    events = []
    for _ in range(600):
        if rng.random() < 0.6:
            events.append(int(rng.integers(1, 600)))
        else:
            events.append(0)
    _run_both(max_len, n_inst, cap, 0.85, 0.9, peek, events, seed)


@pytest.mark.parametrize("seed", range(5))
def test_allocate_matches_oracle(arlo_lib, seed):
    rng = np.random.default_rng(100 + seed)
    I = int(rng.integers(1, 6))
    G = int(rng.integers(1, 9))
    nb = int(rng.integers(1, 9))
    M = rng.uniform(5, 40, size=I)
    Q = rng.uniform(0, 30, size=I) * rng.integers(0, 2, size=I)
    base = np.sort(rng.uniform(1, 10, size=I))
    lat = np.array([[b0 * (1 + 0.3 * (k - 1)) for k in range(1, nb + 1)] for b0 in base])
    ref = osch.allocate(G, Q.tolist(), M.tolist(), lat.tolist())
    if ref is None:
        with pytest.raises(arlo_lib.ArloError) as e:
            arlo_lib.allocate(G, Q, M, lat)
        assert e.value.code == arlo_lib.EINFEASIBLE
        return
    N, val = arlo_lib.allocate(G, Q, M, lat)
    assert N == ref[0]
    assert abs(val - ref[1]) <= 1e-9 * max(1.0, abs(ref[1]))


def test_allocate_hand_computed(arlo_lib):
    lat1 = [float(b) for b in range(1, 33)]
    lat2 = [2.0 * b for b in range(1, 33)]
    N, val = arlo_lib.allocate(2, [10.0, 2.0], [20.0, 20.0], [lat1, lat2])
    assert N == (1, 1) and abs(val - 108.0) < 1e-12
    N, val = arlo_lib.allocate(3, [50.0, 1.0], [20.0, 20.0], [lat1, lat2])
    assert N == (2, 1) and abs(val - 1042.0) < 1e-12
    with pytest.raises(arlo_lib.ArloError):
        arlo_lib.allocate(1, [50.0, 1.0], [20.0, 20.0], [lat1, lat2])


def test_allocate_paper_scale_8_runtimes_8_gpus(arlo_lib):
    """8 runtimes on one 8-GPU box (PAPER.md:L299 '8 runtimes'): exact and fast."""
    import time
    rng = np.random.default_rng(7)
    I, G, nb = 8, 8, 32
    M = np.linspace(60, 10, I)
    Q = np.array([30, 40, 15, 5, 2, 1, 0.5, 0.2])
    lat = np.array([[(1 + i) * (1 + 0.05 * (b - 1)) for b in range(1, nb + 1)] for i in range(I)])
    t = time.perf_counter()
    N, val = arlo_lib.allocate(G, Q, M, lat)
    dt = time.perf_counter() - t
    ref = osch.allocate(G, Q.tolist(), M.tolist(), lat.tolist())
    assert N == ref[0] and abs(val - ref[1]) < 1e-9 * abs(ref[1])
    assert sum(N) == G and N[-1] >= 1
    assert dt < 0.5


@pytest.mark.parametrize("policy", ["ilb", "ig", "rs"])
def test_dispatch_policies_match_oracle(arlo_lib, policy):
    """RS (Algorithm 1) and the ILB / IG baselines of PAPER.md:L373 through the ABI, against
    the oracle on a random interleaving of arrivals and completions."""
    rng = np.random.default_rng(17)
    max_len = [64, 128, 192, 256, 512]
    n_inst = [2, 3, 0, 1, 2]
    cap = [6.0, 5.0, 4.0, 3.0, 2.0]
    s = arlo_lib.Scheduler(max_len, n_inst, cap, 0.85, 0.9, 6)
    code = {"rs": arlo_lib.DISPATCH_RS, "ilb": arlo_lib.DISPATCH_ILB, "ig": arlo_lib.DISPATCH_IG}[policy]
    s.set_policy(code)
    q = osch.MultiLevelQueue(max_len, n_inst, cap)
    live = []
    for step in range(600):
        if live and rng.random() < 0.45:
            r, i = live.pop(int(rng.integers(len(live))))
            s.complete(r, i)
            osch.complete(q, r, i)
            continue
        length = int(rng.integers(1, 513))
        if policy == "rs":
            want = osch.dispatch(q, length, 0.85, 0.9, 6)
        elif policy == "ilb":
            want = osch.dispatch_ilb(q, length)
        else:
            want = osch.dispatch_ig(q, length)
        got = s.dispatch(length)
        assert got == want, (step, length, got, want)
        live.append(got)
    s.close()


def test_ilb_ig_hand_cases(arlo_lib):
    """ILB keeps to the ideal runtime however loaded; IG takes the emptiest candidate."""
    s = arlo_lib.Scheduler([128, 256, 512], [1, 1, 1], [2.0, 2.0, 2.0], 0.85, 0.9, 6)
    s.set_policy(arlo_lib.DISPATCH_ILB)
    assert [s.dispatch(100) for _ in range(3)] == [(0, 0)] * 3
    s.set_policy(arlo_lib.DISPATCH_IG)
    assert s.dispatch(100) == (1, 0)   # level 0 has 3 outstanding, levels 1 and 2 none -> smaller max_len
    assert s.dispatch(100) == (2, 0)   # level 1 now 1, level 2 0
    assert s.dispatch(300) == (2, 0)   # only level 2 can run a length-300 request
    with pytest.raises(arlo_lib.ArloError):
        s.set_policy(7)
    s.close()


# ------------------------------------------------------------------ instance replacement (L272)
def test_replace_plan_against_oracle(arlo_lib):
    """arlo_replace_plan: the replaced count is the oracle's minimum; the plan realises N_new and
    only moves a GPU whose runtime is oversubscribed in the new allocation (or that had none)."""
    rng = np.random.default_rng(11)
    for _ in range(300):
        G, I = int(rng.integers(1, 6)), int(rng.integers(1, 4))
        cur = [int(v) for v in rng.integers(-1, I, size=G)]
        cuts = np.sort(rng.integers(0, G + 1, size=I))
        N_new = [int(v) for v in np.diff(np.concatenate([[0], cuts]))]
        nxt, rep = arlo_lib.replace_plan(cur, N_new)
        _o, rep_o = osch.replace_plan(cur, N_new)
        assert rep == rep_o
        assert rep == sum(1 for g in range(G) if nxt[g] != cur[g])
        assert all(nxt.count(i) == n for i, n in enumerate(N_new))
        for g in range(G):
            if nxt[g] != cur[g] and cur[g] >= 0:
                assert cur.count(cur[g]) > N_new[cur[g]]


def test_replace_plan_errors(arlo_lib):
    with pytest.raises(RuntimeError):
        arlo_lib.replace_plan([0, 1], [2, 1])       # sum N_new > G
    with pytest.raises(RuntimeError):
        arlo_lib.replace_plan([0, 5], [1, 1])       # cur out of range
    with pytest.raises(RuntimeError):
        arlo_lib.replace_plan([0, 1], [-1, 1])      # negative N_new
