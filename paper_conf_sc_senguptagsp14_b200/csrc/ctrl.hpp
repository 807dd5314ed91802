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

constexpr int kRing = 256;            // KL ring entries per logical device
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
  // followed by KlDone[L][kRing]
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
  GroupSync sync;                     // barrier + partials for group-wide bodies (SCAN, HIST)
};

// The KL request queue lives in DEVICE memory: the host never makes the GPU
// read host memory on the dispatch path (16 leaders polling host memory cut the
// copy engines' throughput 4x, and under a saturated host link one 512-B PCIe
// read of a work item took ~20 us; profiles/r01_doorbell.md):
//   items[ld][slot]  work item of the job holding resident slot `slot`, DMA'd at
//                    the job's H2D issue on the queue stream;
//   ring[ld][i]      (seq << 32) | slot, one 64-bit stream memory op per KL on
//                    the same stream (so after the item copy).  Entry i is
//                    published when its seq == i + 1 (mod kRing reuse: seq is
//                    monotone and the host never overwrites an unclaimed entry);
//   stop             shutdown word, stream memory op at teardown.
struct DispatchParams {
  KlDone* done;                       // [L * kRing] host-mapped completion words
  uint32_t* heads;                    // [L] device-memory claim counters
  PartState* parts;                   // [L * P]
  const int* part_start;              // [L * P + 1] first CTA of each partition (device memory)
  const uint32_t* stop;
  const uint64_t* ring;               // [L * kRing]
  const KlItem* items;                // [L * M]
  int L, P, M;                        // logical devices hosted, partitions per device, slots per device
  uint32_t flags;                     // experiment knobs (STRINGS_DISPATCH_FLAGS): bit0 no poll back-off
  uint32_t poll_max_ns;               // idle-poll back-off cap (STRINGS_POLL_MAX_NS)
  uint64_t fault_job;                 // fault injection (STRINGS_FAULT_JOB): trap on this job id
};

inline size_t host_ctrl_bytes(int L) { return sizeof(HostCtrl) + sizeof(KlDone) * kRing * L; }

}  // namespace strings_dev
