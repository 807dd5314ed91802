// ctrl.hpp -- host <-> persistent-kernel control block (host-mapped pinned memory).
//
// One block per physical GPU.  It carries, per hosted logical device, the
// device-resident request queue of KL work items (the paper's Dispatcher ->
// GPU path, replacing the RT-signal wake-up of L697 with a
// doorbell the GPU polls) and the completion words the GPU writes back
// (Request Monitor input, L671).
#pragma once
#include <cstdint>

#include "tenant_kernels.cuh"

namespace strings_dev {

constexpr int kRing = 256;            // KL ring entries per logical device
constexpr uint32_t kStop = 0xFFFFFFFFu;

struct __align__(64) KlRing {
  volatile uint32_t tail;             // number of items published (host writes, GPU reads)
  uint32_t pad[15];
  KlItem items[kRing];
};

struct __align__(32) KlDone {
  volatile uint32_t seq;              // = item.seq when the item has finished
  uint32_t partition;
  uint64_t t_start, t_end;            // %globaltimer ns: leader claim, last CTA done
  uint64_t t_exec;                    // %globaltimer ns: leader CTA starts the body
};

// Host-mapped part (cudaHostAlloc mapped): rings + completions + shutdown flag.
struct HostCtrl {
  volatile uint32_t shutdown;
  uint32_t pad[15];
  // followed by KlRing[L] and KlDone[L][kRing] (sizes depend on L)
};

// Device-memory part: claim counters and per-partition mailboxes.
struct __align__(128) PartState {
  uint32_t gen;                       // item generation published by the leader (kStop = exit)
  uint32_t done_gen;                  // last generation fully finished by all CTAs
  uint32_t done_cnt;                  // CTAs finished with the current generation
  uint32_t ring_idx;
  uint64_t t_start;
  uint64_t t_exec;
  KlItem item;
  GroupSync sync;                     // barrier + partials for group-wide bodies (SCAN, HIST)
};

struct DispatchParams {
  HostCtrl* ctrl;                     // device view of the host-mapped block
  KlRing* rings;                      // [L]
  KlDone* done;                       // [L * kRing]
  uint32_t* heads;                    // [L] device-memory claim counters
  PartState* parts;                   // [L * P]
  const int* part_start;              // [L * P + 1] first CTA of each partition (device memory)
  int L, P;                           // logical devices hosted, partitions per logical device
  uint32_t flags;                     // experiment knobs (STRINGS_DISPATCH_FLAGS): bit0 no poll back-off,
                                      // bit1 host doorbell
  uint64_t fault_job;                 // fault injection (STRINGS_FAULT_JOB): trap on this job id
  uint32_t poll_max_ns;               // idle-poll back-off cap (STRINGS_POLL_MAX_NS)
  // Device-memory doorbells (default): word 32*ld = ring tail of logical device
  // ld, word 32*L = shutdown; written by the host through cuStreamWriteValue32.
  // flags bit1 (STRINGS_DOORBELL=host): poll the host-mapped ring tail instead.
  uint32_t* doorbells;
};

inline size_t host_ctrl_bytes(int L) {
  return sizeof(HostCtrl) + sizeof(KlRing) * L + sizeof(KlDone) * kRing * L;
}

}  // namespace strings_dev
