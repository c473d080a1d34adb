// Host dispatch-overhead microbenchmark (PAPER.md:L347 5.1.4 reports
// 0.737 ms for 2400 concurrent requests over 1200 instances).  Builds an arlo_sched with K
// levels x I instances, keeps `live` requests outstanding, and times arlo_dispatch +
// arlo_complete pairs for each dispatch policy.  Host code only: runs without a GPU.
//   g++ -O2 -std=c++17 -I include tools/sched_bench.cpp -o tools/sched_bench \
//       -L paper_conf_icpp_tanlyl024_b200 -larlo -Wl,-rpath,$PWD/paper_conf_icpp_tanlyl024_b200
//   ./tools/sched_bench [K] [instances_per_level] [live] [ops]
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <random>
#include <vector>

#include "arlo.h"

int main(int argc, char** argv) {
  const int K = argc > 1 ? atoi(argv[1]) : 8;
  const int I = argc > 2 ? atoi(argv[2]) : 150;  // 8 x 150 = 1200 instances
  const int live = argc > 3 ? atoi(argv[3]) : 2400;
  const int ops = argc > 4 ? atoi(argv[4]) : 1000000;
  std::vector<int32_t> max_len(K), n_inst(K, I);
  std::vector<double> cap(K);
  for (int k = 0; k < K; ++k) {
    max_len[k] = 512 * (k + 1) / K;
    cap[k] = 64.0;
  }
  const char* names[3] = {"RS (Algorithm 1)", "ILB", "IG"};
  std::mt19937 rng(7);
  std::uniform_int_distribution<int> len(2, 512);
  for (int policy = 0; policy < 3; ++policy) {
    arlo_sched* s = nullptr;
    if (arlo_sched_create(K, max_len.data(), n_inst.data(), cap.data(), 0.85, 0.9, 6, &s) != 0) {
      printf("create failed: %s\n", arlo_last_error());
      return 1;
    }
    arlo_sched_set_policy(s, policy);
    std::vector<std::pair<int32_t, int32_t>> out;
    out.reserve(live);
    for (int i = 0; i < live; ++i) {
      int32_t r, j;
      arlo_dispatch(s, len(rng), &r, &j);
      out.push_back({r, j});
    }
    std::uniform_int_distribution<int> pick(0, live - 1);
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < ops; ++i) {
      const int v = pick(rng);
      arlo_complete(s, out[v].first, out[v].second);
      int32_t r, j;
      arlo_dispatch(s, len(rng), &r, &j);
      out[v] = {r, j};
    }
    auto t1 = std::chrono::steady_clock::now();
    const double ns = std::chrono::duration<double, std::nano>(t1 - t0).count() / ops;
    printf("%-17s K=%d instances=%d live=%d: %.1f ns per dispatch+complete (%.2f M dispatches/s; "
           "%d dispatches = %.3f ms)\n",
           names[policy], K, K * I, live, ns, 1e3 / ns, live, live * ns / 1e6);
    arlo_sched_destroy(s);
  }
  return 0;
}
