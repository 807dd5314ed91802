// ctrl.hpp -- host <-> persistent-kernel control block (host-mapped pinned memory).
//
// One block per physical GPU.  The device-resident request queue of KL work
// items (the paper's Dispatcher -> GPU path, replacing the
// RT-signal wake-up of L697 with a doorbell the GPU polls in device memory) and
// the completion words the GPU writes back to host memory (Request Monitor
// input, L671).
#pragma once
#include <cstdint>

#include "tenant_kernels.cuh"

namespace strings_dev {

constexpr int kRing = 256;            // entries per KL ring
// KL rings per logical device: 0 = entries the host publishes when the scheduler
// wakes a KL (queue stream), 1 = entries chained on the H2D stream behind the
// job's input copy when the KL's wake is certain (eager chaining, runtime.cu)
constexpr int kRings = 2;
constexpr uint32_t kStop = 0xFFFFFFFFu;

struct __align__(32) KlDone {
  volatile uint32_t seq;              // = item.seq when the item has finished
  uint32_t partition;
  uint64_t t_start, t_end;            // %globaltimer ns: leader claim, last CTA done
  uint64_t t_exec;                    // %globaltimer ns: leader CTA starts the body
};

// Host-mapped part (cudaHostAlloc mapped): the completion words the GPU writes.
struct HostCtrl {
  uint32_t pad[16];
  // followed by KlDone[L][kRings][kRing], then the copy partition's KlDone[kRing] and CopyItem[kRing]
};

// Device-memory part: claim counters and per-partition mailboxes.
struct __align__(128) PartState {
  uint64_t gen;                       // lo: item generation published by the leader (kStop = exit),
                                      // hi: resident slot of the item (its entry in the item table)
  uint32_t done_gen;                  // last generation fully finished by all CTAs
  uint32_t done_cnt;                  // CTAs finished with the current generation
  uint32_t ring_idx;
  uint32_t seq;                       // claim number of the current item (ring entry)
  uint64_t t_start;
  uint64_t t_exec;
  // Lending an idle KL partition to its sibling's streaming item (DispatchParams::help):
  uint32_t lock;                      // 0 free, kLockOwn = running its own item, q+1 = lent to partition q
  uint32_t total;                     // CTAs working on this partition's current item (own + lent);
                                      // 0 until the leader has decided on lending, which it does only
                                      // after releasing its own CTAs (they read it when they finish)
  uint64_t help;                      // (kHelpGen | owner << 16 | slot) << 32 when lent, published by the owner
  GroupSync sync;                     // barrier + partials for group-wide bodies (SCAN, HIST)
};
constexpr uint32_t kLockOwn = 0xFFFFFFFEu;
constexpr uint32_t kHelpGen = 0x80000000u;     // generation slot word: this is a lent share of another item

// The KL request queue lives in DEVICE memory: the host never makes the GPU
// read host memory on the dispatch path (16 leaders polling host memory cut the
// copy engines' throughput 4x, and under a saturated host link one 512-B PCIe
// read of a work item took ~20 us; profiles/r01_doorbell.md):
//   items[ld][slot]  work item of the job holding resident slot `slot`, DMA'd at
//                    the job's H2D issue on the queue stream;
//   ring[ld][i]      (seq << 32) | (kclass << 16) | slot, one 64-bit stream
//                    memory op per KL on the same stream (so after the item
//                    copy; slot < 2^16 since M <= 0xFFFF).  Entry i is
//                    published when its seq == i + 1 (mod kRing reuse: seq is
//                    monotone and the host never overwrites an unclaimed entry);
//   stop             shutdown word, stream memory op at teardown.
// Small host-link copies on SMs (the copy partition).  The copy engines serve
// mixed-size traffic badly: a 128-256 KiB copy queued among 4-64 MiB copies
// waits for them and costs ~14 us of engine time more than alone
// (tools/mix_probe.cu, profiles/r01_mix_probe.jsonl).  So H2D/D2H ops of up to
// STRINGS_SM_COPY_MAX bytes whose host buffers are mapped pinned memory run on
// a partition of the persistent dispatcher instead: 16-B zero-copy loads and
// stores over PCIe, concurrent with the engines' large copies.  The host
// writes a CopyItem into a host-mapped table and publishes (seq, index) into a
// device-memory ring with one stream memory op (no copy-engine operation on
// this path); the partition leader claims it, the item is read once from host
// memory, and the last CTA writes a KlDone word into host memory.
struct CopySeg {
  uint64_t src, dst, bytes;           // device-visible addresses; 16-B aligned, bytes % 16 == 0
};
constexpr int kCopySegs = 4;
struct __align__(128) CopyItem {
  uint64_t job;
  uint32_t nseg;
  uint32_t to_host;                   // 1: destinations are host memory (D2H): system-scope fence
  CopySeg seg[kCopySegs];
};
static_assert(sizeof(CopyItem) == 128, "CopyItem layout");

__device__ __forceinline__ uint4 ld_cv_v4(const uint4* p) {     // host memory: never a stale cached line
  uint4 r;
  asm volatile("ld.global.cv.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p) : "memory");
  return r;
}
__device__ __forceinline__ uint4 ld_cg_v4(const uint4* p) {     // device memory another SM wrote
  uint4 r;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p) : "memory");
  return r;
}

// One copy item on the partition's S CTAs: every segment cut into 16-B words
// dealt round-robin over S*256 threads, 8 independent loads in flight per
// thread (32 KB per CTA) to cover the PCIe round trip.
__device__ __forceinline__ void copy_body(const CopyItem& c, int rank, int S) {
  const uint64_t tid = (uint64_t)rank * kThreads + threadIdx.x;
  const uint64_t nthr = (uint64_t)S * kThreads;
  constexpr int U = 8;
  for (uint32_t g = 0; g < c.nseg; ++g) {
    const uint4* src = reinterpret_cast<const uint4*>(c.seg[g].src);
    uint4* dst = reinterpret_cast<uint4*>(c.seg[g].dst);
    const uint64_t n16 = c.seg[g].bytes / 16;
    uint64_t i = tid;
    for (; i + (U - 1) * nthr < n16; i += U * nthr) {
      uint4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = c.to_host ? ld_cg_v4(src + i + u * nthr) : ld_cv_v4(src + i + u * nthr);
#pragma unroll
      for (int u = 0; u < U; ++u) dst[i + u * nthr] = v[u];
    }
    for (; i < n16; i += nthr) dst[i] = c.to_host ? ld_cg_v4(src + i) : ld_cv_v4(src + i);
  }
  // every thread orders its own host-memory stores before the CTA counts in (the
  // last CTA's completion word must not overtake any of them over PCIe)
  if (c.to_host) __threadfence_system();
}

struct DispatchParams {
  KlDone* done;                       // [L][kRings][kRing] host-mapped completion words
  uint32_t* done_dev;                 // [L][kRings][kRing] device copies of the completion seq
                                      // (an eager D2H waits on them: cuStreamWaitValue32)
  uint32_t* heads;                    // [L][kRings] device-memory claim counters, [L*kRings] = copy ring
  PartState* parts;                   // [L * P]
  const int* part_start;              // [L * P + 1] first CTA of each partition (device memory)
  const uint32_t* stop;
  const uint64_t* ring;               // [L][kRings][kRing]
  const KlItem* items;                // [L * M]
  int L, P, M;                        // logical devices hosted, partitions per device, slots per device
  uint32_t flags;                     // experiment knobs (STRINGS_DISPATCH_FLAGS): bit0 no poll back-off
  uint32_t poll_max_ns;               // idle-poll back-off cap (STRINGS_POLL_MAX_NS)
  uint64_t fault_job;                 // fault injection (STRINGS_FAULT_JOB): trap on this job id
  uint32_t help;                      // 1: an idle sibling KL partition joins VSCALE/XFER items
  // copy partition (partition index L*P, CTAs [part_start[L*P], part_start[L*P+1])) when copy_ctas > 0;
  // its claim counter is heads[L * kRings] and its PartState parts[L*P]
  int copy_ctas;
  uint32_t* progress;                 // [gridDim.x] per-CTA (generation << 4 | step) for stall dumps
  const uint64_t* cring;              // [kRing] device ring entries (seq << 32) | index
  const CopyItem* citems;             // [kRing] host-mapped copy items (device view)
  KlDone* cdone;                      // [kRing] host-mapped completion words
};

inline size_t host_ctrl_bytes(int L) {
  return sizeof(HostCtrl) + sizeof(KlDone) * kRing * (L * kRings + 1) + sizeof(CopyItem) * kRing + 128;
}

}  // namespace strings_dev
