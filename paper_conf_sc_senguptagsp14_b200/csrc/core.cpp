// core.cpp -- Strings scheduler decision core.  See core.hpp and DESIGN.md §4.
#include "core.hpp"

#include <algorithm>
#include <cstdio>
#include <stdexcept>

namespace strings {

namespace {
constexpr uint64_t kPriorLinkBytesPerNs = 50;     // nominal integer peaks (R-13)
constexpr uint64_t kPriorHbmBytesPerNs = 6000;
constexpr uint64_t kPriorKlFlopPerNs = 700000;
constexpr const char* kEngName[3] = {"H2D", "KL", "D2H"};

inline uint64_t cdiv(uint64_t a, uint64_t b) { return (a + b - 1) / b; }
inline bool is_feedback_policy(int b) {
  return b == B_RTF || b == B_GUF || b == B_DTF || b == B_MBF || b == B_DYNAMIC;
}
}  // namespace

void class_bytes_flop(int kclass, uint64_t n, uint64_t m, uint64_t k, uint64_t reps,
                      uint64_t* hbm_bytes, uint64_t* flop) {
  switch (kclass) {
    case K_VSCALE:   // read x (fp32), write y (fp32)
    case K_XFER:     // read x (u32), write y (u32)
      *hbm_bytes = 8 * n;
      *flop = 0;
      return;
    case K_GEMM:     // compulsory: A, B (bf16) in, C (fp32) out; 2mnk FLOP per repetition
      *hbm_bytes = 2 * m * k + 2 * k * n + 4 * m * n;
      *flop = 2 * m * n * k * reps;
      return;
    case K_HIST:     // read x (u8), write 256 u32 bins
      *hbm_bytes = n + 1024;
      *flop = 0;
      return;
    case K_SCAN:     // read x, write y (u32)
    case K_SORT:
      *hbm_bytes = 8 * n;
      *flop = 0;
      return;
  }
  throw std::invalid_argument("kernel class");
}

bool Completion::operator<(const Completion& o) const {
  if (gid != o.gid) return gid < o.gid;
  if (engine != o.engine) return engine < o.engine;
  if (slot != o.slot) return slot < o.slot;
  return job < o.job;
}

Core::Core(const CoreConfig& cfg, Hooks* hooks) : cfg_(cfg), hooks_(hooks), next_epoch_(cfg.Q) {
  devs_.resize(cfg_.G);
  dev_dirty_.assign(cfg_.G, 0);
  busy_ns_.assign(cfg_.G, std::vector<uint64_t>(3, 0));
  for (int g = 0; g < cfg_.G; ++g) {
    devs_[g].gid = g;
    devs_[g].weight = g < (int)cfg_.weights.size() ? cfg_.weights[g] : 1;
    devs_[g].busy[ENG_H2D].assign(1, nullptr);
    devs_[g].busy[ENG_KL].assign(cfg_.P, nullptr);
    devs_[g].busy[ENG_D2H].assign(1, nullptr);
  }
}

int Core::add_tenant(uint32_t weight, uint32_t max_inflight) {
  Tenant t;
  t.weight = weight;
  t.c = max_inflight;
  tenants_.push_back(t);
  sft_.resize(tenants_.size() * K_NCLASS);
  return static_cast<int>(tenants_.size()) - 1;
}

void Core::add_job(Job* j) {
  if (j->prio == 0) j->prio = tenants_.at(j->tenant).weight;
  tenants_[j->tenant].pending.push_back(j);
  jobs_[j->id] = j;
  arr_.insert(j);
  ++jobs_total_;
}

uint64_t Core::next_arrival() const { return arr_.empty() ? UINT64_MAX : (*arr_.begin())->arrival; }

// ---------------------------------------------------------------- trace
namespace {
inline char* put_u64(char* p, uint64_t v) {
  char tmp[24];
  int n = 0;
  do {
    tmp[n++] = char('0' + v % 10);
    v /= 10;
  } while (v);
  while (n) *p++ = tmp[--n];
  return p;
}
inline char* put_opt(char* p, long v) {
  if (v < 0) {
    *p++ = '-';
    return p;
  }
  return put_u64(p, (uint64_t)v);
}
inline char* put_str(char* p, const char* s) {
  while (*s) *p++ = *s++;
  return p;
}
}  // namespace

void Core::rec(uint64_t t, const char* kind, int gid, int eng, int slot, long tenant, long seq,
               long job, uint64_t a1, uint64_t a2) {
  ++trace_records_;
  if (!cfg_.record_trace) return;
  char buf[256];
  char* p = put_u64(buf, t);
  *p++ = ' ';
  p = put_str(p, kind);
  *p++ = ' ';
  p = put_opt(p, gid);
  *p++ = ' ';
  p = put_str(p, eng < 0 ? "-" : kEngName[eng]);
  *p++ = ' ';
  p = put_opt(p, slot);
  *p++ = ' ';
  p = put_opt(p, tenant);
  *p++ = ' ';
  p = put_opt(p, seq);
  *p++ = ' ';
  p = put_opt(p, job);
  *p++ = ' ';
  p = put_u64(p, a1);
  *p++ = ' ';
  p = put_u64(p, a2);
  *p++ = '\n';
  trace_.append(buf, p - buf);
}

// ---------------------------------------------------------------- orders
bool Core::las_key_less(const Job* a, const Job* b) const {
  unsigned __int128 lhs = (unsigned __int128)tenants_[a->tenant].cgs * b->prio;
  unsigned __int128 rhs = (unsigned __int128)tenants_[b->tenant].cgs * a->prio;
  return lhs < rhs;
}

bool Core::las_before(const Job* a, const Job* b) const {
  if (las_key_less(a, b)) return true;
  if (las_key_less(b, a)) return false;
  if (a->tenant != b->tenant) return a->tenant < b->tenant;
  return a->seq < b->seq;
}

bool Core::admission_before(const Job* a, const Job* b) const {
  if (cfg_.las_admission) return las_before(a, b);
  if (a->arrival != b->arrival) return a->arrival < b->arrival;
  if (a->tenant != b->tenant) return a->tenant < b->tenant;
  return a->seq < b->seq;
}

// ---------------------------------------------------------- predictions
bool Core::has_sample(const Job* j) const { return sft_[j->tenant * K_NCLASS + j->kclass].count > 0; }

Core::Pred Core::pred(const Job* j) const {
  const SftRow& r = sft_[j->tenant * K_NCLASS + j->kclass];
  if (r.count > 0) return {r.h2d, r.kl, r.d2h, r.util};
  Pred p;
  p.h2d = cdiv(j->h2d_bytes, kPriorLinkBytesPerNs);
  p.d2h = cdiv(j->d2h_bytes, kPriorLinkBytesPerNs);
  p.kl = std::max(cdiv(j->hbm_bytes, kPriorHbmBytesPerNs), cdiv(j->flop, kPriorKlFlopPerNs));
  uint64_t tot = p.h2d + p.kl + p.d2h;
  p.util = tot ? (p.kl * 65536) / tot : 0;
  return p;
}

int Core::effective_policy(const Job* j) const {
  int b = cfg_.balancer;
  if (is_feedback_policy(b) && !has_sample(j)) return B_GMIN;   // arbiter (R-15)
  return b == B_DYNAMIC ? B_MBF : b;
}

Core::Agg Core::aggregate(const Device& d) const {
  Agg a;
  a.n = d.resident.size();
  for (const Job* r : d.resident) {
    Pred q = pred(r);
    const uint64_t h = r->phase <= ENG_H2D ? q.h2d : 0;
    const uint64_t k = r->phase <= ENG_KL ? q.kl : 0;
    const uint64_t dd = r->phase <= ENG_D2H ? q.d2h : 0;
    a.rem_total += h + k + dd;                   // RTF: predicted remaining runtime
    a.util += q.util;                            // GUF: summed utilisation
    a.copy += h + dd;                            // DTF: remaining transfer time
    a.kl += k;                                   //      and remaining kernel time
    a.h2d += h;                                  // MBF: per-resource busy time
    a.d2h += dd;
    if (r->phase <= ENG_KL) {
      const uint64_t hb = std::min(q.kl, cdiv(r->hbm_bytes, kPriorHbmBytesPerNs));
      a.hbm += hb;
      a.sm += q.kl - hb;
    }
  }
  return a;
}

// Balancer score of placing j on a device with aggregates a (minimised; R-13).
uint64_t Core::score_from(int policy, const Agg& a, const Job* j) const {
  switch (policy) {
    case B_GMIN:
    case B_GWTMIN:
      return a.n;
    case B_RTF: {
      Pred p = pred(j);
      return a.rem_total + p.h2d + p.kl + p.d2h;
    }
    case B_GUF:                         // L827
      return a.util + pred(j).util;
    case B_DTF: {                       // L829
      Pred p = pred(j);
      return std::max(a.copy + p.h2d + p.d2h, a.kl + p.kl);
    }
    case B_MBF: {                       // L831
      Pred p = pred(j);
      const uint64_t hb = std::min(p.kl, cdiv(j->hbm_bytes, kPriorHbmBytesPerNs));
      return std::max(std::max(a.h2d + p.h2d, a.d2h + p.d2h), std::max(a.hbm + hb, a.sm + p.kl - hb));
    }
  }
  throw std::logic_error("score: policy");
}

uint64_t Core::score(int policy, const Job* j, const Device& d) const {
  return score_from(policy, aggregate(d), j);
}

int Core::select_device(int policy, const Job* j, const std::vector<int>& adm,
                        const std::vector<Agg>& aggs, uint64_t* score_out) {
  if (policy == B_GRR) {
    for (int k = 0; k < cfg_.G; ++k) {
      int g = (grr_cursor_ + k) % cfg_.G;
      if (std::find(adm.begin(), adm.end(), g) != adm.end()) {
        grr_cursor_ = (g + 1) % cfg_.G;
        *score_out = 0;
        return g;
      }
    }
    throw std::logic_error("GRR: no admissible device");
  }
  if (policy == B_GWTMIN) {             // L689: min load / weight (cross-multiplied)
    int best = adm[0];
    for (int g : adm) {
      const Device& d = devs_[g];
      const Device& b = devs_[best];
      if ((uint64_t)d.resident.size() * b.weight < (uint64_t)b.resident.size() * d.weight) best = g;
    }
    *score_out = devs_[best].resident.size();
    return best;
  }
  int best = -1;
  uint64_t bs = 0;
  for (int g : adm) {                   // ties -> lowest GID (L687)
    uint64_t s = score_from(policy, aggs[g], j);
    if (best < 0 || s < bs) {
      best = g;
      bs = s;
    }
  }
  *score_out = bs;
  return best;
}

// ------------------------------------------------------------ admission
void Core::admission(uint64_t t) {
  const bool joint = cfg_.joint &&
                     (cfg_.balancer == B_DTF || cfg_.balancer == B_MBF || cfg_.balancer == B_DYNAMIC);
  std::vector<Job*>& elig = scratch_elig_;
  std::vector<int>& adm = scratch_adm_;
  std::vector<Agg>& aggs = scratch_aggs_;
  // Cheap exits first: most calls (a completion that freed no resident slot
  // the pending jobs can use) find no device with room or no eligible job.
  adm.clear();
  for (auto& d : devs_)
    if ((int)d.resident.size() < cfg_.M) adm.push_back(d.gid);
  if (adm.empty()) return;
  // Eligible jobs: each tenant's oldest pending job while the tenant is below c_t.
  // Built once per call; a placement changes only the placed job's tenant.
  elig.clear();
  for (auto& tn : tenants_)
    if (!tn.pending.empty() && tn.inflight < tn.c && tn.pending.front()->arrived)
      elig.push_back(tn.pending.front());
  if (elig.empty()) return;
  aggs.resize(devs_.size());
  const bool need_aggs = cfg_.balancer != B_GRR && cfg_.balancer != B_GMIN && cfg_.balancer != B_GWTMIN;
  // Aggregates depend only on the resident jobs' phases and the SFT, neither of
  // which changes during admission: compute them once, then refresh only the
  // device that received a job.  Every selection below is a linear min scan in
  // admission order (no sort): O(T + T*G) per placement.
  for (auto& d : devs_) {
    if (need_aggs) aggs[d.gid] = aggregate(d);
    else aggs[d.gid].n = d.resident.size();
  }
  for (;;) {
    Job* pick = nullptr;
    int gid = -1, pol = B_GMIN;
    uint64_t sc = 0;
    if (joint) {
      // first job in admission order still placed by GMin (no sample yet) ...
      for (Job* j : elig)
        if (effective_policy(j) == B_GMIN && (!pick || admission_before(j, pick))) pick = j;
      if (pick) {
        pol = B_GMIN;
        gid = select_device(pol, pick, adm, aggs, &sc);
      } else {
        // ... else the lexicographic min of (score, admission order, GID)
        for (Job* j : elig) {
          int p = effective_policy(j);
          for (int g : adm) {
            uint64_t s = score_from(p, aggs[g], j);
            if (!pick || s < sc || (s == sc && j != pick && admission_before(j, pick))) {
              sc = s;
              pick = j;
              gid = g;
              pol = p;
            }
          }
        }
      }
    } else {
      for (Job* j : elig)
        if (!pick || admission_before(j, pick)) pick = j;
      pol = effective_policy(pick);
      gid = select_device(pol, pick, adm, aggs, &sc);
    }
    place(t, pick, gid, pol, sc);
    if (need_aggs) aggs[gid] = aggregate(devs_[gid]);
    else aggs[gid].n = devs_[gid].resident.size();
    if ((int)devs_[gid].resident.size() >= cfg_.M) {
      adm.erase(std::find(adm.begin(), adm.end(), gid));
      if (adm.empty()) return;
    }
    // the placed job's tenant: its next pending job replaces it if the tenant
    // is still below c_t (elig keeps no particular order: every scan is a min)
    Tenant& tn = tenants_[pick->tenant];
    auto pos = std::find(elig.begin(), elig.end(), pick);
    if (!tn.pending.empty() && tn.inflight < tn.c && tn.pending.front()->arrived) {
      *pos = tn.pending.front();
    } else {
      *pos = elig.back();
      elig.pop_back();
      if (elig.empty()) return;
    }
  }
}

void Core::place(uint64_t t, Job* j, int gid, int policy, uint64_t score) {
  Tenant& tn = tenants_[j->tenant];
  if (tn.pending.empty() || tn.pending.front() != j) throw std::logic_error("place: order");
  tn.pending.pop_front();
  ++tn.inflight;
  j->placed = true;
  j->gid = gid;
  j->t_place = t;
  j->place_order = place_counter_++;
  devs_[gid].resident.push_back(j);
  dev_dirty_[gid] = 1;
  ++decisions_;
  rec(t, "PLACE", gid, -1, -1, j->tenant, j->seq, (long)j->id, policy, score);
}

// ------------------------------------------------------------- dispatch
void Core::wake(uint64_t t, Device& d, Job* j) {
  j->woken = true;
  d.fifo[j->phase].push_back(j);
  ++d.woken_unfinished;
  ++decisions_;
  rec(t, "WAKE", d.gid, j->phase, -1, j->tenant, j->seq, (long)j->id, 0, 0);
  hooks_->on_wake(*j, j->phase, t);
}

void Core::dispatch(uint64_t t, Device& d) {
  std::vector<Job*>& cand = scratch_cand_;
  cand.clear();
  for (Job* j : d.resident)
    if (j->phase < 3 && !j->woken) cand.push_back(j);
  int budget = cfg_.A - d.woken_unfinished;
  auto by_key = [this](const Job* a, const Job* b) { return las_before(a, b); };
  if (cfg_.device_policy == P_TFS) {
    tfs_dispatch(t, d, cand, budget);
  } else if (!cand.empty() && budget > 0) {
    if (cfg_.device_policy == P_FIFO) {
      for (size_t i = 0; i < cand.size() && budget > 0; ++i, --budget) wake(t, d, cand[i]);
    } else if (cfg_.device_policy == P_LAS) {       // phase-blind
      std::sort(cand.begin(), cand.end(), by_key);
      for (size_t i = 0; i < cand.size() && budget > 0; ++i, --budget) wake(t, d, cand[i]);
    } else {                                        // Phase Selection, L819 (R-11)
      std::vector<Job*>* ph = scratch_ph_;
      for (int x = 0; x < 3; ++x) ph[x].clear();
      for (Job* j : cand) ph[j->phase].push_back(j);
      for (int x = 0; x < 3; ++x) std::sort(ph[x].begin(), ph[x].end(), by_key);
      int active[3];
      for (int x = 0; x < 3; ++x) {
        active[x] = (int)d.fifo[x].size();
        for (Job* b : d.busy[x]) active[x] += b != nullptr;
      }
      size_t head[3] = {0, 0, 0};
      // (i) diversity: one woken op per phase, KL first
      if (active[ENG_KL] == 0 && !ph[ENG_KL].empty() && budget > 0) {
        wake(t, d, ph[ENG_KL][head[ENG_KL]++]);
        --budget;
      }
      int order[2] = {ENG_H2D, ENG_D2H};
      bool h_ok = active[ENG_H2D] == 0 && !ph[ENG_H2D].empty();
      bool d_ok = active[ENG_D2H] == 0 && !ph[ENG_D2H].empty();
      if (h_ok && d_ok && las_key_less(ph[ENG_D2H][0], ph[ENG_H2D][0])) {
        order[0] = ENG_D2H;
        order[1] = ENG_H2D;
      }
      for (int x : order) {
        bool ok = (x == ENG_H2D) ? h_ok : d_ok;
        if (ok && budget > 0) {
          wake(t, d, ph[x][head[x]++]);
          --budget;
        }
      }
      // (ii) fill: KL > H2D = D2H
      while (head[ENG_KL] < ph[ENG_KL].size() && budget > 0) {
        wake(t, d, ph[ENG_KL][head[ENG_KL]++]);
        --budget;
      }
      std::vector<Job*>& copies = scratch_copies_;
      copies.clear();
      for (size_t i = head[ENG_H2D]; i < ph[ENG_H2D].size(); ++i) copies.push_back(ph[ENG_H2D][i]);
      for (size_t i = head[ENG_D2H]; i < ph[ENG_D2H].size(); ++i) copies.push_back(ph[ENG_D2H][i]);
      std::sort(copies.begin(), copies.end(), by_key);
      for (size_t i = 0; i < copies.size() && budget > 0; ++i, --budget) wake(t, d, copies[i]);
    }
  }
  start_pass(t, d);
}

// True Fair-Share (R-28).  At most one tenant is awake on
// a device; it keeps the device for w_t * S of service (ops are not preempted),
// or until it has nothing left to run (work conserving), and is released only
// once its woken ops have finished.  The next tenant is the one with the least
// cumulative service / weight on this device, which pays back any overshoot.
void Core::tfs_dispatch(uint64_t t, Device& d, const std::vector<Job*>& cand, int budget) {
  if (d.svc.size() < tenants_.size()) d.svc.resize(tenants_.size(), 0);
  if (d.awake >= 0) {
    const uint64_t slice = (uint64_t)tenants_[d.awake].weight * cfg_.tfs_slice;
    bool has_work = false;
    for (const Job* j : cand) has_work |= (long)j->tenant == d.awake;
    if (d.woken_unfinished == 0 && (d.awake_used >= slice || !has_work)) d.awake = -1;
  }
  if (d.awake < 0) {
    long best = -1;
    for (const Job* j : cand) {
      const long tid = j->tenant;
      if (best < 0) {
        best = tid;
        continue;
      }
      const unsigned __int128 lhs = (unsigned __int128)d.svc[tid] * tenants_[best].weight;
      const unsigned __int128 rhs = (unsigned __int128)d.svc[best] * tenants_[tid].weight;
      if (lhs < rhs || (lhs == rhs && tid < best)) best = tid;
    }
    if (best >= 0) {
      d.awake = best;
      d.awake_used = 0;
    }
  }
  if (d.awake < 0 || d.awake_used >= (uint64_t)tenants_[d.awake].weight * cfg_.tfs_slice) return;
  for (Job* j : cand) {                         // placement order
    if (budget <= 0) break;
    if ((long)j->tenant != d.awake) continue;
    wake(t, d, j);
    --budget;
  }
}

void Core::start_pass(uint64_t t, Device& d) {
  for (int x = 0; x < 3; ++x) {
    for (size_t s = 0; s < d.busy[x].size(); ++s) {
      if (d.busy[x][s] == nullptr && !d.fifo[x].empty()) {
        Job* j = d.fifo[x].front();
        d.fifo[x].pop_front();
        d.busy[x][s] = j;
        j->start[x] = t;
        j->slot[x] = (int)s;
        rec(t, "START", d.gid, x, (int)s, j->tenant, j->seq, (long)j->id, 0, 0);
        hooks_->on_start(*j, x, (int)s, t);
      }
    }
  }
}

// ----------------------------------------------------------- completion
void Core::complete(const Completion& c) {
  auto it = jobs_.find(c.job);
  if (it == jobs_.end()) throw std::logic_error("complete: unknown job");
  Job* j = it->second;
  Device& d = devs_.at(c.gid);
  if (d.busy[c.engine].at(c.slot) != j) throw std::logic_error("complete: engine not running job");
  const uint64_t t = c.t;
  d.busy[c.engine][c.slot] = nullptr;
  dev_dirty_[c.gid] = 1;
  --d.woken_unfinished;
  j->done[c.engine] = t;
  j->phase += 1;
  j->woken = false;
  busy_ns_[c.gid][c.engine] += t - j->start[c.engine];
  if (d.svc.size() < tenants_.size()) d.svc.resize(tenants_.size(), 0);
  d.svc[j->tenant] += t - j->start[c.engine];
  if (d.awake == (long)j->tenant) d.awake_used += t - j->start[c.engine];
  Tenant& tn = tenants_[j->tenant];
  tn.gs_acc += t - std::max(j->start[c.engine], epoch_start_);
  rec(t, "DONE", c.gid, c.engine, c.slot, j->tenant, j->seq, (long)j->id, t - j->start[c.engine], 0);
  if (c.engine == ENG_D2H) {
    j->t_done = t;
    j->finished = true;
    ++jobs_done_;
    rec(t, "JOB_DONE", c.gid, -1, -1, j->tenant, j->seq, (long)j->id, t - j->arrival, 0);
    feedback(t, j);
    adm_dirty_ = true;
    d.resident.erase(std::find(d.resident.begin(), d.resident.end(), j));
    --tn.inflight;
    jobs_.erase(it);
    hooks_->on_job_done(*j, t);
  }
}

void Core::feedback(uint64_t t, Job* j) {
  // Request Monitor -> Feedback Engine -> SFT (R-14)
  uint64_t smp[3];
  for (int x = 0; x < 3; ++x) smp[x] = j->measured[x] ? j->measured[x] : j->done[x] - j->start[x];
  uint64_t span = t - j->t_place;
  uint64_t util = span ? (smp[ENG_KL] * 65536) / span : 0;
  SftRow& r = sft_[j->tenant * K_NCLASS + j->kclass];
  if (r.count == 0) {
    r.h2d = smp[0];
    r.kl = smp[1];
    r.d2h = smp[2];
    r.util = util;
  } else {
    r.h2d = (4 * smp[0] + r.h2d) / 5;
    r.kl = (4 * smp[1] + r.kl) / 5;
    r.d2h = (4 * smp[2] + r.d2h) / 5;
    r.util = (4 * util + r.util) / 5;
  }
  ++r.count;
  rec(t, "FEEDBACK", j->gid, -1, -1, j->tenant, j->seq, (long)j->id, r.h2d + r.d2h, r.kl);
}

void Core::epoch(uint64_t t) {
  // GS_n and Eq. (1) with k = 4/5 in Q48.16 (R-4, R-6)
  std::vector<uint64_t> inprog(tenants_.size(), 0);
  for (auto& d : devs_)
    for (int x = 0; x < 3; ++x)
      for (Job* j : d.busy[x])
        if (j) inprog[j->tenant] += t - std::max(j->start[x], epoch_start_);
  for (size_t i = 0; i < tenants_.size(); ++i) {
    Tenant& tn = tenants_[i];
    uint64_t gs = tn.gs_acc + inprog[i];
    uint64_t old = tn.cgs;
    tn.cgs = (4 * (gs << 16) + old) / 5;
    tn.gs_acc = 0;
    if (gs > 0 || old > 0) rec(t, "EPOCH", -1, -1, -1, (long)i, -1, -1, gs, tn.cgs);
  }
  epoch_start_ = t;
  next_epoch_ = t + cfg_.Q;
}

// ------------------------------------------------------------ the step
void Core::step(uint64_t t, std::vector<Completion> dones, bool first) {
  now_ = t;
  std::sort(dones.begin(), dones.end());
  for (const Completion& c : dones) complete(c);
  if (first) {
    if (next_epoch_ == t) epoch(t);
    while (!arr_.empty() && (*arr_.begin())->arrival <= t) {
      Job* j = *arr_.begin();
      arr_.erase(arr_.begin());
      j->arrived = true;
      adm_dirty_ = true;
      rec(t, "ARRIVE", -1, -1, -1, j->tenant, j->seq, (long)j->id, j->prio, 0);
    }
  }
  if (adm_dirty_) {
    adm_dirty_ = false;
    admission(t);
  }
  for (auto& d : devs_)
    if (dev_dirty_[d.gid]) {
      dev_dirty_[d.gid] = 0;
      dispatch(t, d);
    }
}

void Core::close_epochs_before(uint64_t t) {
  while (next_epoch_ < t) step(next_epoch_, {}, true);
}

}  // namespace strings
