// core_bench.cpp -- speed of the scheduler decision core alone (SURVEY.md §8(d)
// "host decision <= 1 us/job"; "report DES speed (decisions/s) separately").
//
// Drives strings::Core in virtual time with injected durations, exactly as the
// runtime's DECISIONS_ONLY mode does, but with no-op hooks and no runtime
// locking, on C2/C5-shaped synthetic workloads (same class sizes and nominal
// durations as strings_workload).  Prints ns per job and decisions per second.
//
//   g++ -O3 -std=c++17 -I paper_conf_sc_senguptagsp14_b200/csrc tools/core_bench.cpp \
//       paper_conf_sc_senguptagsp14_b200/csrc/core.cpp -o /tmp/core_bench && /tmp/core_bench
#include <chrono>
#include <cstdio>
#include <cstring>
#include <memory>
#include <queue>
#include <vector>

#include "core.hpp"

using namespace strings;

namespace {
using Ev = std::pair<uint64_t, Completion>;
struct EvLater {
  bool operator()(const Ev& a, const Ev& b) const {
    if (a.first != b.first) return a.first > b.first;
    return b.second < a.second;
  }
};
using Heap = std::priority_queue<Ev, std::vector<Ev>, EvLater>;
struct VHooks : Hooks {
  Heap* heap;
  void on_wake(Job&, int, uint64_t) override {}
  void on_start(Job& j, int e, int slot, uint64_t t) override {
    heap->push({t + j.dur[e], Completion{t + j.dur[e], j.gid, e, slot, j.id}});
  }
  void on_job_done(Job&, uint64_t) override {}
};
}  // namespace

struct Shape {
  const char* name;
  int G, tenants, jobs_per_tenant, balancer, joint;
  bool rotate;   // C5: class rotates every 4 jobs
};

static void fill_job(Job& j, int kclass) {
  j.kclass = kclass;
  if (kclass == K_VSCALE) {
    j.h2d_bytes = j.d2h_bytes = 4ull << 20;
    class_bytes_flop(K_VSCALE, 1 << 20, 0, 0, 1, &j.hbm_bytes, &j.flop);
  } else if (kclass == K_GEMM) {
    j.h2d_bytes = 2 * 2 * 256 * 256;
    j.d2h_bytes = 4 * 256 * 256;
    class_bytes_flop(K_GEMM, 256, 256, 256, 64, &j.hbm_bytes, &j.flop);
  } else {
    j.h2d_bytes = j.d2h_bytes = 64ull << 20;
    class_bytes_flop(K_XFER, 1 << 24, 0, 0, 1, &j.hbm_bytes, &j.flop);
  }
  j.dur[0] = (j.h2d_bytes + 49) / 50;
  j.dur[2] = (j.d2h_bytes + 49) / 50;
  j.dur[1] = std::max((j.hbm_bytes + 5999) / 6000, (j.flop + 699999) / 700000);
}

static double run(const Shape& s, bool trace, uint64_t* decisions) {
  CoreConfig cfg;
  cfg.G = s.G;
  cfg.P = 2;
  cfg.A = 4;
  cfg.M = 8;
  cfg.balancer = s.balancer;
  cfg.joint = s.joint;
  cfg.device_policy = P_PS;
  cfg.record_trace = trace;
  Heap heap;
  VHooks hk;
  hk.heap = &heap;
  Core core(cfg, &hk);
  const int T = s.tenants, J = s.jobs_per_tenant;
  std::vector<Job> jobs((size_t)T * J);
  for (int t = 0; t < T; ++t) core.add_tenant(1, 1);
  uint64_t id = 0;
  for (int q = 0; q < J; ++q)
    for (int t = 0; t < T; ++t) {
      Job& j = jobs[id];
      j.id = id++;
      j.tenant = t;
      j.seq = q;
      const int cls = s.rotate ? ((q / 4 + t) % 3) : (t < T / 2 ? K_GEMM : K_XFER);
      fill_job(j, cls == 0 ? K_VSCALE : cls == 1 ? K_GEMM : K_XFER);
    }
  for (auto& j : jobs) core.add_job(&j);
  auto t0 = std::chrono::steady_clock::now();
  while (core.unfinished()) {
    uint64_t t = heap.empty() ? UINT64_MAX : heap.top().first;
    if (core.has_pending_arrival()) t = std::min(t, core.next_arrival());
    t = std::min(t, core.next_epoch());
    bool first = true;
    for (;;) {
      std::vector<Completion> batch;
      while (!heap.empty() && heap.top().first == t) {
        batch.push_back(heap.top().second);
        heap.pop();
      }
      core.step(t, std::move(batch), first);
      first = false;
      if (heap.empty() || heap.top().first != t) break;
    }
  }
  auto t1 = std::chrono::steady_clock::now();
  *decisions = core.decisions();
  return std::chrono::duration<double, std::nano>(t1 - t0).count() / jobs.size();
}

int main(int argc, char** argv) {
  const int reps = argc > 1 ? atoi(argv[1]) : 5;
  const Shape shapes[] = {
      {"C2 (G=1, 16 tenants x 8, DTF joint)", 1, 16, 8, B_DTF, 1, false},
      {"C5 (G=8, 128 tenants x 24, DYNAMIC)", 8, 128, 24, B_DYNAMIC, 0, true},
      {"C5x8 (G=8, 1024 tenants x 24, DYNAMIC)", 8, 1024, 24, B_DYNAMIC, 0, true},
  };
  for (const auto& s : shapes)
    for (int tr = 0; tr < 2; ++tr) {
      double best = 1e30;
      uint64_t dec = 0;
      for (int r = 0; r < reps; ++r) best = std::min(best, run(s, tr, &dec));
      const double jobs = (double)s.tenants * s.jobs_per_tenant;
      printf("{\"workload\": \"%s\", \"trace\": %s, \"ns_per_job\": %.0f, \"decisions_per_s\": %.3g}\n", s.name,
             tr ? "true" : "false", best, dec / (best * jobs * 1e-9));
    }
  return 0;
}
