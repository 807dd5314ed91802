// core.hpp -- the Strings two-level scheduler decision core (host, no CUDA).
//
// Implements DESIGN.md §4 (the contract shared with the independent CPU
// oracle): balancer admission + GPU choice (level 1, PAPER.md L683-689,
// L823-831), per-device wake decisions FIFO / LAS / PS (level 2, L669, L693,
// L819), epochs with the decayed service of Eq. (1) (L695), the feedback
// table SFT (L311, L671-673) and the canonical decision trace (§4.9).
//
// The core never touches a GPU.  It talks to the outside through Hooks:
//   on_wake(job, engine)       -- the op entered its engine FIFO: issue it
//   on_start(job, engine, t)   -- the op started (virtual modes: schedule DONE)
//   on_job_done(job)           -- D2H finished: release the slot, wake syncers
// and is driven by a caller that feeds it timestamps and completions
// (engine.cpp), so the same code serves MEASURED, INJECTED and DECISIONS_ONLY.
#pragma once

#include <cstdint>
#include <deque>
#include <map>
#include <set>
#include <unordered_map>
#include <string>
#include <vector>

namespace strings {

enum Engine : int { ENG_H2D = 0, ENG_KL = 1, ENG_D2H = 2 };
enum KClass : int { K_VSCALE = 0, K_GEMM = 1, K_XFER = 2, K_HIST = 3, K_SCAN = 4, K_SORT = 5, K_NCLASS = 6 };
enum Balancer : int { B_GRR = 0, B_GMIN, B_GWTMIN, B_RTF, B_GUF, B_DTF, B_MBF, B_DYNAMIC };
enum DevPolicy : int { P_FIFO = 0, P_LAS = 1, P_PS = 2, P_TFS = 3 };

struct CoreConfig {
  int G = 1, P = 2, A = 4, M = 8;
  int balancer = B_GMIN, las_admission = 0, device_policy = P_PS, joint = 0;
  uint64_t Q = 1000000;
  uint64_t tfs_slice = 500000;        // TFS base slice S (R-28)
  std::vector<uint32_t> weights;      // DST device weights; empty = all 1
  bool record_trace = true;           // keep the decision trace
};

// One job's scheduling record (the RCB view of a request).
struct Job {
  uint64_t id = 0;
  uint32_t tenant = 0, seq = 0, prio = 1;
  int kclass = 0;
  uint64_t arrival = 0;
  uint64_t h2d_bytes = 0, d2h_bytes = 0, hbm_bytes = 0, flop = 0;
  uint64_t dur[3] = {0, 0, 0};        // injected durations
  // MEASURED mode: a phase's busy time measured on the device (KL: the
  // dispatcher's %globaltimer claim -> last CTA), fed to the SFT instead of the
  // host-observed DONE - START, which adds the publish and completion-observation
  // latency; 0 = not measured (the host-observed time is used)
  uint64_t measured[3] = {0, 0, 0};
  // decision state
  bool arrived = false, placed = false;
  int gid = -1;
  uint64_t t_place = 0, place_order = 0;
  int phase = 0;                      // phases completed (3 = done)
  bool woken = false;
  uint64_t start[3] = {0, 0, 0}, done[3] = {0, 0, 0};
  int slot[3] = {-1, -1, -1};
  uint64_t t_done = 0;
  bool finished = false;
  void* user = nullptr;               // execution-side payload (engine.cpp)
};

struct SftRow {                        // Scheduler Feedback Table row (Fig 6)
  uint64_t count = 0, h2d = 0, kl = 0, d2h = 0, util = 0;
};

struct Hooks {
  virtual ~Hooks() {}
  virtual void on_wake(Job& j, int engine, uint64_t t) = 0;
  virtual void on_start(Job& j, int engine, int slot, uint64_t t) = 0;
  virtual void on_job_done(Job& j, uint64_t t) = 0;
};

struct Completion {                    // DONE event key (§4.2 order)
  uint64_t t;
  int gid, engine, slot;
  uint64_t job;
  bool operator<(const Completion& o) const;
};

class Core {
 public:
  Core(const CoreConfig& cfg, Hooks* hooks);

  int add_tenant(uint32_t weight, uint32_t max_inflight);
  // Registers a submitted job (arrival time already set).  The core keeps the
  // pointer; it must stay valid until the job finished.
  void add_job(Job* j);

  // One iteration of process(t) (§4.2): complete `dones` (any order; sorted
  // here), then on the first iteration the epoch and the arrivals at t, then
  // admission and the dispatch/start passes of every device.
  void step(uint64_t t, std::vector<Completion> dones, bool first);
  // Close every epoch boundary < t that has not been closed (measured mode).
  void close_epochs_before(uint64_t t);

  uint64_t next_epoch() const { return next_epoch_; }
  bool has_pending_arrival() const { return !arr_.empty(); }
  uint64_t next_arrival() const;
  uint64_t unfinished() const { return jobs_total_ - jobs_done_; }
  uint64_t jobs_done() const { return jobs_done_; }
  uint64_t current_time() const { return now_; }

  std::string& trace() { return trace_; }
  uint64_t trace_records() const { return trace_records_; }
  uint64_t decisions() const { return decisions_; }
  uint64_t busy_ns(int gid, int eng) const { return busy_ns_[gid][eng]; }
  const CoreConfig& config() const { return cfg_; }

 private:
  struct Tenant {
    uint32_t weight = 1, c = 1;
    std::deque<Job*> pending;         // submitted, not yet placed (seq order)
    uint32_t inflight = 0;
    uint64_t cgs = 0;                 // Q48.16 ns (Eq. 1)
    uint64_t gs_acc = 0;              // completed service in the current epoch
  };
  struct Device {
    int gid = 0;
    uint32_t weight = 1;
    std::vector<Job*> resident;       // placement order
    std::deque<Job*> fifo[3];
    std::vector<Job*> busy[3];        // H2D: 1 slot, KL: P slots, D2H: 1 slot
    int woken_unfinished = 0;
    // True Fair-Share (R-28)
    long awake = -1;                  // tenant awake on this device, -1 = none
    uint64_t awake_used = 0;          // its service here since it woke
    std::vector<uint64_t> svc;        // cumulative service per tenant on this device
  };
  struct Pred { uint64_t h2d, kl, d2h, util; };
  // Per-device sums over resident jobs' remaining predicted work (every balancer
  // score is such a sum plus the new job's term; integer sums, so computing them
  // once per admission round gives the same values as summing per candidate).
  struct Agg {
    uint64_t n = 0, rem_total = 0, util = 0, copy = 0, kl = 0, h2d = 0, d2h = 0, hbm = 0, sm = 0;
  };
  Agg aggregate(const Device& d) const;
  uint64_t score_from(int policy, const Agg& a, const Job* j) const;

  void rec(uint64_t t, const char* kind, int gid, int eng, int slot, long tenant, long seq,
           long job, uint64_t a1, uint64_t a2);
  // LAS (R-7): a before b iff CGS_a * p_b < CGS_b * p_a, then tenant, seq.
  bool las_before(const Job* a, const Job* b) const;
  bool las_key_less(const Job* a, const Job* b) const;
  bool admission_before(const Job* a, const Job* b) const;
  Pred pred(const Job* j) const;
  bool has_sample(const Job* j) const;
  int effective_policy(const Job* j) const;
  uint64_t score(int policy, const Job* j, const Device& d) const;
  int select_device(int policy, const Job* j, const std::vector<int>& adm, const std::vector<Agg>& aggs,
                    uint64_t* score_out);

  void admission(uint64_t t);
  void place(uint64_t t, Job* j, int gid, int policy, uint64_t score);
  void dispatch(uint64_t t, Device& d);
  void tfs_dispatch(uint64_t t, Device& d, const std::vector<Job*>& cand, int budget);
  void wake(uint64_t t, Device& d, Job* j);
  void start_pass(uint64_t t, Device& d);
  void complete(const Completion& c);
  void feedback(uint64_t t, Job* j);
  void epoch(uint64_t t);

  CoreConfig cfg_;
  Hooks* hooks_;
  std::vector<Tenant> tenants_;
  std::vector<Device> devs_;
  std::vector<SftRow> sft_;           // [tenant * K_NCLASS + class]
  struct ArrLess {
    bool operator()(const Job* a, const Job* b) const {
      if (a->arrival != b->arrival) return a->arrival < b->arrival;
      if (a->tenant != b->tenant) return a->tenant < b->tenant;
      return a->seq < b->seq;
    }
  };
  std::set<Job*, ArrLess> arr_;       // submitted, not yet arrived
  std::unordered_map<uint64_t, Job*> jobs_;   // id -> job (unfinished)
  uint64_t jobs_total_ = 0, jobs_done_ = 0;
  uint64_t epoch_start_ = 0, next_epoch_;
  int grr_cursor_ = 0;
  uint64_t place_counter_ = 0;
  uint64_t now_ = 0;
  std::string trace_;
  uint64_t trace_records_ = 0, decisions_ = 0;
  std::vector<std::vector<uint64_t>> busy_ns_;
  // scratch buffers reused by the hot paths (no per-call heap allocation)
  std::vector<Job*> scratch_cand_, scratch_ph_[3], scratch_copies_, scratch_elig_;
  std::vector<int> scratch_adm_;
  std::vector<Agg> scratch_aggs_;
  // Work-skipping: a dispatch pass on a device whose state did not change since
  // its last pass, or an admission pass with no job arrival/completion since the
  // last one, is a no-op (each pass runs to its fixed point), so it is skipped.
  bool adm_dirty_ = false;
  std::vector<char> dev_dirty_;
};

// Algorithmic kernel bytes and tensor FLOP of a job.
void class_bytes_flop(int kclass, uint64_t n, uint64_t m, uint64_t k, uint64_t reps,
                      uint64_t* hbm_bytes, uint64_t* flop);

}  // namespace strings
