"""Host logic of the cluster replay (replay.simulate_cluster / plan_cluster): the discrete-event
simulation of G single-instance GPUs, with the C++ Request Scheduler (Algorithm 1) and Runtime
Scheduler (Eqs. 1-7) through the ABI, and a closed-form service time instead of a GPU (CPU)."""
import numpy as np

from paper_conf_icpp_tanlyl024_b200 import replay
from paper_conf_icpp_tanlyl024_b200 import workload as wl


def factory(arlo_lib):
    def f(max_len, n_inst, capacity, lam, alpha, peek):
        return arlo_lib.Scheduler(max_len, n_inst, capacity, lam, alpha, peek)
    return f


def test_single_instance_saturation_is_batch_count(arlo_lib):
    """One L=512 instance, 1 ms per batch of <= 32: n requests at t=0 finish in ceil(n/32) ms."""
    n = 100
    arrivals = np.zeros(n)
    lengths = wl.sample_lengths(n, seed=3)
    done, rof, inst, busy = replay.simulate_cluster(arrivals, lengths, [512], [1], [1e6],
                                                    lambda L, b: 1e-3, 32, factory(arlo_lib))
    assert np.isclose(done.max(), 4e-3)
    assert sorted(np.round(np.unique(done) * 1e3).astype(int)) == [1, 2, 3, 4]
    assert np.all(rof == 0)
    assert np.isclose(sum(busy.values()), 4e-3)


def test_requests_only_run_on_long_enough_runtimes(arlo_lib):
    """a request may only run on a runtime with max_length >= len; every request
    completes after its arrival plus at least one service time; the run is deterministic."""
    Ls = list(wl.RUNTIME_LENGTHS)
    n = 2000
    lengths = wl.sample_lengths(n, seed=4)
    arrivals = wl.poisson_arrivals(n, 20000.0, seed=5)
    n_inst = [1, 2, 1, 0, 0, 0, 0, 1]
    svc = lambda L, b: (0.2 + L / 512.0) * 1e-3  # noqa: E731

    def go():
        return replay.simulate_cluster(arrivals, lengths, Ls, n_inst, [64.0] * len(Ls), svc, 32, factory(arlo_lib))
    done, rof, inst, busy = go()
    assert np.all(np.array(Ls)[rof] >= lengths)
    assert np.all(np.array(n_inst)[rof] > 0)
    assert np.all(done >= arrivals + 0.2e-3 - 1e-12)
    assert np.all(inst < np.array(n_inst)[rof])
    done2, rof2, *_ = go()
    np.testing.assert_array_equal(done, done2)
    np.testing.assert_array_equal(rof, rof2)
    s = replay.summarize(arrivals, lengths, done, rof, Ls, 150.0)
    assert s["requests"] == n and s["p99_ms"] >= s["mean_ms"] > 0


def test_slo_capacity_closed_form():
    # lat(b) = 1 + b ms: b*floor(150/(1+b)) over b = 1..32 -> best at b = 32: 32*4 = 128? check all
    row = [1.0 + b for b in range(1, 33)]
    expect = max(b * np.floor(150.0 / (1.0 + b)) for b in range(1, 33))
    assert replay.slo_capacity(row, 150.0) == expect
    assert replay.slo_capacity([500.0] * 4, 150.0) == 1.0  # nothing fits: capacity floor 1


def test_plan_cluster_satisfies_eqs_2_and_7(arlo_lib):
    Ls = list(wl.RUNTIME_LENGTHS)
    lat = [[0.3 + 0.002 * L * (1 + b / 8.0) for b in range(1, 33)] for L in Ls]
    shares = [0.316, 0.434, 0.163, 0.055, 0.02, 0.008, 0.003, 0.001]
    for G in (1, 2, 4, 8):
        N, Q, M = replay.plan_cluster(arlo_lib, G, Ls, lat, shares, 20000.0 * G, 150.0)
        assert sum(N) == G and N[-1] >= 1  # Eq. 2, Eq. 7
        assert all(n >= np.floor(q / m) for n, q, m in zip(N, Q, M))  # Eq. 3


def test_periodic_plans_track_the_drift_with_minimum_replacement(arlo_lib):
    """SURVEY NEXT-3 host logic: each window deploys the allocation planned on the previous window's
    shares, reached from the current deployment by the minimum number of replaced
    instances (L272): |N_new - N_cur|_1 / 2 when every GPU is used."""
    Ls = [64, 128, 256, 512]
    lat = np.array([[0.2 + 0.01 * b * k for b in range(1, 33)] for k in range(1, 5)])
    shares = [[0.7, 0.2, 0.05, 0.05], [0.7, 0.2, 0.05, 0.05], [0.1, 0.2, 0.3, 0.4], [0.1, 0.2, 0.3, 0.4]]
    G, rate, slo = 8, 2e5, 150.0

    def plan(sh):
        return replay.plan_cluster(arlo_lib, G, Ls, lat, sh, rate, slo)[0]

    N0 = plan(shares[0])
    plans = replay.periodic_plans(arlo_lib, N0, shares, plan)
    assert plans[0] == (list(N0), 0)
    for w in range(1, len(shares)):
        N_w, rep = plans[w]
        assert N_w == list(plan(shares[w - 1]))
        prev = plans[w - 1][0]
        assert rep == sum(abs(a - b) for a, b in zip(N_w, prev)) // 2
        assert sum(N_w) == G and N_w[-1] >= 1          # Eqs. 2 and 7 hold after the replacement
    assert plans[3][0] != plans[2][0] and plans[3][1] > 0  # the drift (window 2) changed the deployment
