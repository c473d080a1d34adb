"""ORACLE — Arlo's host-side schedulers, written from the paper (TEST INFRASTRUCTURE).

Only ``tests/`` (and bench's reference legs) may import this module; the
product path's ``arlo_allocate`` / ``arlo_dispatch`` live in C++ under
``paper_conf_icpp_tanlyl024_b200/csrc/sched.cpp`` and share nothing with it.

* ``dispatch`` — Algorithm 1, Request Scheduler (§3.4),
  step by step in the paper's order and notation: candidate runtimes by
  length (line 2), TOPK to the maximum peeking level L (lines 3-5), congestion
  P = N / M of each candidate's head instance (lines 7-9), dispatch if
  P < lambda (lines 10-13, prose L258 "less than lambda"), otherwise
  lambda <- lambda * alpha (line 15), fall back to Q_e[0] (lines 18-19),
  DISPATCH + UPDATE (lines 21-22).  The multi-level queue (Fig. 5;
  L223, L256) keeps per level a priority queue of instances with the least
  outstanding load at the head.
* ``allocate`` — the Runtime Scheduler program, Eqs. 1-7 (PAPER.md:L181-203
  §3.3), solved by enumerating every composition N_1 + ... + N_I = G.
* ``replace_plan`` — instance replacement (§4): "a replacement
  plan that replaces the minimum number of current runtime instances", as its
  definition: every assignment of the new allocation to the GPUs, the one that
  changes the fewest GPUs (ties: lexicographically smallest), by brute force.

Readings: S13 both sums of Eqs. 1-2 run over i = 1..I; S14 Eq. 3
keeps the printed floor; S15 L_i(B) is the profiled batch->latency table,
linearly interpolated and clamped to [1, nb], and a runtime with N_i = 0
contributes 0; S16 strict ``P < lambda``, lambda restarts at lambda_0 for every
request, candidates are runtimes with max_len >= len that have >= 1 instance;
S17 ties of Eq. 1 go to the first optimum in lexicographic order of
(N_1, ..., N_I); head-of-queue ties go to the lowest instance id.
"""
from __future__ import annotations

import itertools
import math


class MultiLevelQueue:
    """Fig. 5: one level per runtime (ascending max_length); instances carry
    outstanding requests N and max capacity M (Alg. 1 lines 7-8)."""

    def __init__(self, max_len, n_inst, capacity):
        self.max_len = list(max_len)
        self.capacity = list(capacity)
        self.outstanding = [[0] * int(k) for k in n_inst]

    def front(self, i):
        """Head instance of level i: least outstanding, lowest id on ties."""
        occ = self.outstanding[i]
        j = min(range(len(occ)), key=lambda t: (occ[t], t))
        return j, occ[j], self.capacity[i]


def candidate_runtimes(q: MultiLevelQueue, length: int):
    """Alg. 1 line 2: runtimes able to run the request (max_length >= len,
    PAPER.md:L135), in increasing max_length, that have an instance."""
    return [i for i in range(len(q.max_len))
            if q.max_len[i] >= length and len(q.outstanding[i]) > 0]


def dispatch(q: MultiLevelQueue, length: int, lam: float, alpha: float, peek: int):
    """Algorithm 1.  Returns (runtime q, instance) or None when no candidate."""
    Qe, flag = [], False                      # line 1
    Qe = candidate_runtimes(q, length)        # line 2
    if not Qe:
        return None
    if len(Qe) > peek:                        # lines 3-5
        Qe = Qe[:peek]
    chosen = None
    for i in Qe:                              # line 6
        _, N, M = q.front(i)                  # lines 7-8
        P = N / M                             # line 9
        if P < lam:                           # line 10
            chosen = i                        # line 11
            flag = True                       # line 12
            break                             # line 13
        lam = lam * alpha                     # line 15
    if not flag:                              # line 18
        chosen = Qe[0]                        # line 19
    inst, _, _ = q.front(chosen)
    q.outstanding[chosen][inst] += 1          # lines 21-22: DISPATCH + UPDATE
    return chosen, inst


def dispatch_ilb(q: MultiLevelQueue, length: int):
    """ILB, "Intra-group Load Balance" (Table 4 baseline): the runtime
    requiring the least padding, i.e. the first candidate, and its least-loaded instance."""
    Qe = candidate_runtimes(q, length)
    if not Qe:
        return None
    chosen = Qe[0]
    inst, _, _ = q.front(chosen)
    q.outstanding[chosen][inst] += 1
    return chosen, inst


def dispatch_ig(q: MultiLevelQueue, length: int):
    """IG, "Inter-groups Greedy": the least busy instance among all
    candidate runtime queues.  Reading S20: least busy = fewest outstanding requests;
    ties go to the smaller max_length (less padding), then the lower instance id."""
    Qe = candidate_runtimes(q, length)
    if not Qe:
        return None
    best = None
    for i in Qe:                              # every candidate, ascending max_length
        inst, N, _ = q.front(i)
        if best is None or N < best[2]:
            best = (i, inst, N)
    q.outstanding[best[0]][best[1]] += 1
    return best[0], best[1]


def complete(q: MultiLevelQueue, runtime: int, instance: int):
    """A request finished: the instance's outstanding count drops by one."""
    q.outstanding[runtime][instance] -= 1


def interp_latency(lat_row, B: float) -> float:
    """Reading S15: L_i(B) from the profiled table lat_row[b-1] (b = 1..nb),
    linear interpolation, B clamped to [1, nb]."""
    nb = len(lat_row)
    B = min(max(B, 1.0), float(nb))
    lo = int(math.floor(B))
    if lo >= nb:
        return float(lat_row[nb - 1])
    frac = B - lo
    return float(lat_row[lo - 1]) * (1.0 - frac) + float(lat_row[lo]) * frac


def objective(N, Q, M, lat):
    """Eq. 1 value of an allocation N (None if Eq. 3 or 7 is violated).

    Eqs. 4-6: R_0 = 0; C_i = min(R_{i-1}+Q_i, N_i M_i) for i < I and
    R_{I-1}+Q_I for i = I; R_i = max(R_{i-1}+Q_i - N_i M_i, 0); B_i = C_i / N_i.
    """
    I = len(N)
    if N[I - 1] < 1:                                       # Eq. 7
        return None
    for i in range(I):                                     # Eq. 3
        if N[i] < math.floor(Q[i] / M[i]):
            return None
    R_prev, total = 0.0, 0.0
    for i in range(I):
        if i < I - 1:
            C = min(R_prev + Q[i], N[i] * M[i])            # Eq. 5, i < I
        else:
            C = R_prev + Q[i]                              # Eq. 5, i = I
        R = max(R_prev + Q[i] - N[i] * M[i], 0.0)          # Eq. 4
        if N[i] > 0 and C > 0:
            B = C / N[i]                                   # Eq. 6
            total += interp_latency(lat[i], B) * C         # Eq. 1 term
        R_prev = R
    return total


def compositions(G: int, I: int):
    """All (N_1..N_I) of non-negative integers summing to G (Eq. 2), lexicographic."""
    for bars in itertools.combinations(range(G + I - 1), I - 1):
        prev, parts = -1, []
        for b in bars:
            parts.append(b - prev - 1)
            prev = b
        parts.append(G + I - 1 - prev - 1)
        yield tuple(parts)


def allocate(G: int, Q, M, lat):
    """min Eq. 1 s.t. Eqs. 2-7; returns (N tuple, objective) or None if infeasible."""
    best = None
    for N in sorted(compositions(G, len(Q))):
        val = objective(N, Q, M, lat)
        if val is None:
            continue
        if best is None or val < best[1]:
            best = (N, val)
    return best


def replace_plan(cur, N_new):
    """among all per-GPU assignments `nxt` (runtime index or -1) with
    #{g : nxt[g] == i} == N_new[i] for every i, the one minimising #{g : nxt[g] != cur[g]}.
    Brute force (tiny G only).  Returns (nxt tuple, n_replaced)."""
    G, I = len(cur), len(N_new)
    spare = G - sum(N_new)
    assert spare >= 0
    pool = [i for i in range(I) for _ in range(N_new[i])] + [-1] * spare
    best = None
    for nxt in sorted(set(itertools.permutations(pool))):
        changed = sum(1 for g in range(G) if nxt[g] != cur[g])
        if best is None or changed < best[1]:
            best = (nxt, changed)
    return best
