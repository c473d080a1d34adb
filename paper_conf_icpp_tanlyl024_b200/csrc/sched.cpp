// sched.cpp — Arlo's host-side schedulers (plain C++, not an optimisation target).
//
//  * arlo_allocate: the Runtime Scheduler's allocation program
//    (§3.3, Eqs. 1-7), solved exactly by depth-first enumeration of every
//    composition N_1 + ... + N_I = G in lexicographic order, carrying R_{i-1}
//    (Eq. 4) and the partial Eq. 1 sum down the recursion and pruning
//    branches that violate Eq. 3 or cannot leave N_I >= 1 (Eq. 7).
//    The paper uses GUROBI (L153); for the G <= 64 GPUs of one or a few
//    B200 boxes exact enumeration is cheap and has no solver dependency.
//  * arlo_sched_* / arlo_dispatch: the Request Scheduler, Algorithm 1
//    (§3.4) over the multi-level queue of Fig. 5 (L207):
//    one level per runtime in ascending max_length, each level a binary
//    min-heap of instances keyed by (outstanding requests, instance id), so the
//    least loaded instance is at the head (L256).  O(peek + log n) per request,
//    the paper's O(L) + O(log(N/K)) (L262).
// Readings S13-S17 of DESIGN.md apply (sums over i = 1..I, floor in Eq. 3,
// interpolated L_i(B), strict P < lambda, lexicographic tie-break).
#include <cmath>
#include <cstdint>
#include <cstring>
#include <new>
#include <vector>

#include "../../include/arlo.h"
#include "errors.h"

namespace {

double interp_latency(const double* row, int nb, double B) {
  if (B < 1.0) B = 1.0;
  if (B > (double)nb) B = (double)nb;
  const int lo = (int)std::floor(B);
  if (lo >= nb) return row[nb - 1];
  const double frac = B - lo;
  return row[lo - 1] * (1.0 - frac) + row[lo] * frac;
}

struct AllocSearch {
  int G, I, nb;
  const double *Q, *M, *lat;
  std::vector<int> lower;  // Eq. 3 lower bounds
  std::vector<int> cur, best;
  double best_val;
  bool found;

  // Assign N_i for i = idx.. given remaining GPUs, R_{idx-1} = R_prev, partial objective acc.
  void rec(int idx, int remaining, double R_prev, double acc) {
    if (idx == I - 1) {
      const int n = remaining;  // Eq. 2 fixes the last one
      if (n < 1 || n < lower[idx]) return;  // Eq. 7, Eq. 3
      cur[idx] = n;
      const double C = R_prev + Q[idx];     // Eq. 5, i = I
      double total = acc;
      if (C > 0) total += interp_latency(lat + (size_t)idx * nb, nb, C / n) * C;  // Eqs. 6, 1
      if (!found || total < best_val) {
        best_val = total;
        best = cur;
        found = true;
      }
      return;
    }
    // the later runtimes need at least sum(lower[j], j > idx) GPUs and N_I >= 1
    int need_after = 0;
    for (int j = idx + 1; j < I; ++j) need_after += lower[j];
    if (lower[I - 1] < 1) need_after += 1 - lower[I - 1];
    for (int n = lower[idx]; n <= remaining - need_after; ++n) {
      cur[idx] = n;
      const double cap = (double)n * M[idx];
      const double C = std::fmin(R_prev + Q[idx], cap);             // Eq. 5, i < I
      const double R = std::fmax(R_prev + Q[idx] - cap, 0.0);       // Eq. 4
      double a = acc;
      if (n > 0 && C > 0) a += interp_latency(lat + (size_t)idx * nb, nb, C / n) * C;
      rec(idx + 1, remaining - n, R, a);
    }
  }
};

struct Level {
  int max_len;
  double capacity;
  std::vector<int32_t> outstanding;  // by instance id
  std::vector<int32_t> heap;         // instance ids, min-heap by (outstanding, id)
  std::vector<int32_t> pos;          // instance id -> heap index

  bool less(int a, int b) const {
    return outstanding[a] < outstanding[b] || (outstanding[a] == outstanding[b] && a < b);
  }
  void swap_at(int i, int j) {
    std::swap(heap[i], heap[j]);
    pos[heap[i]] = i;
    pos[heap[j]] = j;
  }
  void sift_up(int i) {
    while (i > 0) {
      int p = (i - 1) / 2;
      if (!less(heap[i], heap[p])) break;
      swap_at(i, p);
      i = p;
    }
  }
  void sift_down(int i) {
    const int n = (int)heap.size();
    for (;;) {
      int l = 2 * i + 1, r = l + 1, m = i;
      if (l < n && less(heap[l], heap[m])) m = l;
      if (r < n && less(heap[r], heap[m])) m = r;
      if (m == i) break;
      swap_at(i, m);
      i = m;
    }
  }
};

}  // namespace

struct arlo_sched {
  std::vector<Level> levels;
  double lambda, alpha;
  int peek;
  int policy = ARLO_DISPATCH_RS;
};

extern "C" {

int arlo_allocate(int32_t G, int32_t I, const double* Q, const double* M, const double* lat, int32_t nb,
                  int32_t* N_out, double* objective_out) {
  using namespace arlo;
  if (G < 1 || I < 1 || nb < 1 || !Q || !M || !lat || !N_out)
    return set_error(ARLO_EINVAL, "arlo_allocate: need G >= 1, I >= 1, nb >= 1 and non-null arrays");
  // number of compositions C(G+I-1, I-1)
  double comps = 1.0;
  for (int k = 1; k <= I - 1; ++k) comps = comps * (double)(G + k) / (double)k;
  if (comps > 5e7) return set_error(ARLO_EINVAL, "arlo_allocate: %.3g compositions exceed the 5e7 limit", comps);
  AllocSearch s;
  s.G = G; s.I = I; s.nb = nb; s.Q = Q; s.M = M; s.lat = lat;
  s.lower.resize(I);
  int need = 0;
  for (int i = 0; i < I; ++i) {
    if (!(M[i] > 0) || !(Q[i] >= 0)) return set_error(ARLO_EINVAL, "arlo_allocate: need M[i] > 0, Q[i] >= 0");
    s.lower[i] = (int)std::floor(Q[i] / M[i]);  // Eq. 3 (reading S14: floor as printed)
    need += s.lower[i];
  }
  if (s.lower[I - 1] < 1) need += 1 - s.lower[I - 1];
  if (need > G) return set_error(ARLO_EINFEASIBLE, "arlo_allocate: Eqs. 3 and 7 need %d GPUs, G = %d", need, G);
  s.cur.assign(I, 0);
  s.found = false;
  s.best_val = 0;
  s.rec(0, G, 0.0, 0.0);
  if (!s.found) return set_error(ARLO_EINFEASIBLE, "arlo_allocate: no feasible allocation");
  for (int i = 0; i < I; ++i) N_out[i] = s.best[i];
  if (objective_out) *objective_out = s.best_val;
  return ARLO_OK;
}

int arlo_sched_create(int32_t K, const int32_t* max_len, const int32_t* n_inst, const double* capacity,
                      double lambda, double alpha, int32_t peek, arlo_sched** out) {
  using namespace arlo;
  if (!out || K < 1 || !max_len || !n_inst || !capacity || peek < 1)
    return set_error(ARLO_EINVAL, "arlo_sched_create: bad arguments");
  for (int k = 0; k < K; ++k) {
    if (n_inst[k] < 0 || !(capacity[k] > 0)) return set_error(ARLO_EINVAL, "arlo_sched_create: level %d", k);
    if (k > 0 && max_len[k] <= max_len[k - 1])
      return set_error(ARLO_EINVAL, "arlo_sched_create: max_len must be strictly ascending");
  }
  arlo_sched* s = new (std::nothrow) arlo_sched;
  if (!s) return set_error(ARLO_ENOMEM, "arlo_sched_create: out of memory");
  s->lambda = lambda;
  s->alpha = alpha;
  s->peek = peek;
  s->levels.resize(K);
  for (int k = 0; k < K; ++k) {
    Level& l = s->levels[k];
    l.max_len = max_len[k];
    l.capacity = capacity[k];
    l.outstanding.assign(n_inst[k], 0);
    l.heap.resize(n_inst[k]);
    l.pos.resize(n_inst[k]);
    for (int j = 0; j < n_inst[k]; ++j) l.heap[j] = l.pos[j] = j;
  }
  *out = s;
  return ARLO_OK;
}

void arlo_sched_destroy(arlo_sched* s) { delete s; }

int arlo_dispatch(arlo_sched* s, int32_t length, int32_t* runtime_out, int32_t* instance_out) {
  using namespace arlo;
  if (!s || !runtime_out || !instance_out || length < 1) return set_error(ARLO_EINVAL, "arlo_dispatch: bad arguments");
  // line 2: candidate runtimes, ascending max_length; lines 3-5: at most `peek`
  int cand[64];
  int nc = 0;
  const int K = (int)s->levels.size();
  for (int k = 0; k < K && nc < s->peek && nc < 64; ++k)
    if (s->levels[k].max_len >= length && !s->levels[k].heap.empty()) cand[nc++] = k;
  if (nc == 0) return set_error(ARLO_ENOCAND, "arlo_dispatch: no runtime with max_length >= %d", length);
  if (s->policy == ARLO_DISPATCH_ILB || s->policy == ARLO_DISPATCH_IG) {
    // baselines of PAPER.md:L373 (Table 4): ILB = ideal runtime (least padding), its
    // least-loaded instance; IG = least busy instance over ALL candidate runtimes
    // (reading S20: fewest outstanding requests, ties to the smaller max_length)
    int q = -1;
    if (s->policy == ARLO_DISPATCH_ILB) {
      q = cand[0];
    } else {
      int best = 0x7fffffff;
      for (int k = 0; k < K; ++k) {
        const Level& l = s->levels[k];
        if (l.max_len < length || l.heap.empty()) continue;
        const int n = l.outstanding[l.heap[0]];
        if (n < best) { best = n; q = k; }
      }
    }
    Level& l = s->levels[q];
    const int inst = l.heap[0];
    l.outstanding[inst] += 1;
    l.sift_down(0);
    *runtime_out = q;
    *instance_out = inst;
    return ARLO_OK;
  }
  double lam = s->lambda;
  int q = -1;
  for (int c = 0; c < nc; ++c) {  // line 6
    const Level& l = s->levels[cand[c]];
    const double N = l.outstanding[l.heap[0]];  // line 7
    const double P = N / l.capacity;            // lines 8-9
    if (P < lam) {                              // line 10
      q = cand[c];                              // lines 11-13
      break;
    }
    lam = lam * s->alpha;                       // line 15
  }
  if (q < 0) q = cand[0];                       // lines 18-19
  Level& l = s->levels[q];
  const int inst = l.heap[0];
  l.outstanding[inst] += 1;                     // line 21 DISPATCH
  l.sift_down(0);                               // line 22 UPDATE
  *runtime_out = q;
  *instance_out = inst;
  return ARLO_OK;
}

int arlo_sched_set_policy(arlo_sched* s, int32_t policy) {
  using namespace arlo;
  if (!s || policy < ARLO_DISPATCH_RS || policy > ARLO_DISPATCH_IG)
    return set_error(ARLO_EINVAL, "arlo_sched_set_policy: bad arguments");
  s->policy = policy;
  return ARLO_OK;
}

int arlo_sched_set_params(arlo_sched* s, double lambda, double alpha, int32_t peek) {
  using namespace arlo;
  if (!s || peek < 1) return set_error(ARLO_EINVAL, "arlo_sched_set_params: bad arguments");
  s->lambda = lambda;
  s->alpha = alpha;
  s->peek = peek;
  return ARLO_OK;
}

int arlo_complete(arlo_sched* s, int32_t runtime, int32_t instance) {
  using namespace arlo;
  if (!s || runtime < 0 || runtime >= (int)s->levels.size())
    return set_error(ARLO_EINVAL, "arlo_complete: bad runtime");
  Level& l = s->levels[runtime];
  if (instance < 0 || instance >= (int)l.outstanding.size() || l.outstanding[instance] <= 0)
    return set_error(ARLO_EINVAL, "arlo_complete: bad instance or nothing outstanding");
  l.outstanding[instance] -= 1;
  l.sift_up(l.pos[instance]);
  return ARLO_OK;
}

// Instance replacement plan (§4): after a new allocation N_new, replace the
// minimum number of current runtime instances.  GPU g keeps its runtime cur[g] while fewer than
// N_new[cur[g]] GPUs (lowest indices first) have claimed it; the runtimes still missing go, in
// ascending runtime order, first to the GPUs freed from an oversubscribed runtime, then to idle
// ones.  GPUs kept = sum_i min(count_i(cur), N_new[i]) + min(#idle, #spare), the most any plan can
// keep (a matching of equal labels), so the number replaced is minimal.  Deterministic, O(G + I).
int arlo_replace_plan(int32_t G, int32_t I, const int32_t* cur, const int32_t* N_new, int32_t* next,
                      int32_t* n_replaced) {
  using namespace arlo;
  if (G < 1 || I < 1 || !cur || !N_new || !next)
    return set_error(ARLO_EINVAL, "arlo_replace_plan: need G >= 1, I >= 1 and non-null arrays");
  long total = 0;
  for (int i = 0; i < I; ++i) {
    if (N_new[i] < 0) return set_error(ARLO_EINVAL, "arlo_replace_plan: N_new[%d] < 0", i);
    total += N_new[i];
  }
  if (total > G) return set_error(ARLO_EINVAL, "arlo_replace_plan: sum N_new = %ld > G = %d", total, G);
  std::vector<int32_t> kept(I, 0);
  for (int g = 0; g < G; ++g) {
    const int32_t r = cur[g];
    if (r < -1 || r >= I) return set_error(ARLO_EINVAL, "arlo_replace_plan: cur[%d] = %d out of range", g, r);
    if (r >= 0 && kept[r] < N_new[r]) {
      next[g] = r;
      ++kept[r];
    } else {
      next[g] = -1;
    }
  }
  // missing runtimes go first to GPUs freed from an oversubscribed runtime (they change in any
  // case), then to idle GPUs (cur = -1), each group by ascending GPU index; an idle GPU left
  // without a runtime stays idle (unchanged)
  int i = 0;
  for (int pass = 0; pass < 2; ++pass) {
    for (int g = 0; g < G; ++g) {
      if (next[g] >= 0 || (pass == 0) != (cur[g] >= 0)) continue;
      while (i < I && kept[i] >= N_new[i]) ++i;
      if (i == I) break;
      next[g] = i;
      ++kept[i];
    }
  }
  int32_t replaced = 0;
  for (int g = 0; g < G; ++g) replaced += next[g] != cur[g];
  if (n_replaced) *n_replaced = replaced;
  return ARLO_OK;
}

int32_t arlo_sched_outstanding(const arlo_sched* s, int32_t runtime, int32_t instance) {
  if (!s || runtime < 0 || runtime >= (int)s->levels.size()) return ARLO_EINVAL;
  const Level& l = s->levels[runtime];
  if (instance < 0 || instance >= (int)l.outstanding.size()) return ARLO_EINVAL;
  return l.outstanding[instance];
}

}  // extern "C"
