// dispatcher.cu -- persistent sm_100a dispatcher kernel and stand-alone launcher.
//
// The persistent kernel is the device half of the per-device GPU scheduler
// (PAPER.md L331-333, L667-673): it pulls KL work items from the
// device-resident request queue (KL ring, ctrl.hpp) and runs tenant kernel
// bodies on SM partitions, so tenants' kernels co-run on disjoint SMs while
// the copy engines stream other tenants' buffers (PS, L819; MBF, L831).
//
// Geometry: one CTA per SM (grid = #SMs, 256 threads, ~196 KB smem so GEMM
// operands fit), split into NP = L*P partitions of contiguous CTAs.  Partition
// q serves logical device q / P.  Its leader (CTA rank 0, thread 0):
//   1. waits until the previous item is finished by every CTA (done_gen),
//   2. polls the next entry of its logical device's KL ring in device memory
//      (ld.acquire.gpu, nanosleep back-off; the host publishes (seq, slot) with
//      one cuStreamWriteValue64) and claims it with a CAS on the device claim
//      counter.  The dispatch path never reads host memory (ctrl.hpp),
//   3. publishes (slot, gen+1) in one 64-bit st.release.gpu.
// Every CTA of the partition waits for the new generation, reads the job's item
// from the device item table, runs its share of the item, and the last CTA to
// finish writes the completion word and the %globaltimer stamps back to host
// memory (gpu-scope fence + plain store).
// With copy_ctas > 0 the last partition serves small H2D/D2H copies instead
// (ctrl.hpp, CopyItem): same claim/broadcast/completion protocol on its own
// ring, the item read from host memory, the body a zero-copy PCIe copy.
#include <atomic>
#include <cstdio>

#include "ctrl.hpp"

namespace strings_dev {

#ifndef STRINGS_GEN_POLL_NS
#define STRINGS_GEN_POLL_NS 32                    // CTAs' back-off between polls of their generation word
#endif


__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const volatile uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_acquire_gpu_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release_gpu(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}

// Partition q owns CTAs [part_start[q], part_start[q+1]) (sized on the host by
// logical-device weight, then split evenly into P KL slots).
__device__ __forceinline__ void partition_of(int b, int NP, const int* part_start, int* q, int* start, int* S) {
  int p = 0;
  while (p + 1 < NP && part_start[p + 1] <= b) ++p;
  *q = p;
  *start = part_start[p];
  *S = part_start[p + 1] - part_start[p];
}

__global__ void __launch_bounds__(kThreads, 1) dispatcher_kernel(DispatchParams p) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ KlItem s_item;
  __shared__ CopyItem s_citem;
  __shared__ uint32_t s_gen, s_slot, s_owner;
  GemmSmem sm = carve_smem(smem);
  if ((smem_u32(smem) & 1023u) != 0) __trap();   // SWIZZLE_128B tiles need a 1 KB-aligned base
  const int NK = p.L * p.P;                       // KL partitions; the copy partition (if any) is NK
  const int NP = NK + (p.copy_ctas > 0 ? 1 : 0);
  int q, start, S;
  partition_of(blockIdx.x, NP, p.part_start, &q, &start, &S);
  const int rank = blockIdx.x - start;
  const bool cpart = q == NK;
  const int ld = cpart ? p.L : q / p.P;           // logical device (copy partition: L)
  const int nrings = cpart ? 1 : kRings;         // KL rings of the device (host-published, eager)
  PartState* ps = p.parts + q;
  const KlItem* table = p.items + (size_t)(cpart ? 0 : ld) * p.M;
  uint32_t* const heads = cpart ? p.heads + (size_t)p.L * kRings : p.heads + (size_t)ld * kRings;
  const uint64_t* const rings = cpart ? p.cring : p.ring + (size_t)ld * kRings * kRing;
  // the sibling KL slot of the same logical device that may lend its CTAs (P >= 2)
  const int sib = (!cpart && p.help && (q ^ 1) < NK && (q ^ 1) / p.P == ld) ? (q ^ 1) : -1;
  PartState* sps = sib >= 0 ? p.parts + sib : nullptr;
  const int S_sib = sib >= 0 ? p.part_start[sib + 1] - p.part_start[sib] : 0;
  const uint32_t tmem = cta_setup(sm);
  uint32_t mma_phase = 0;
  uint32_t seen = 0;
  for (;;) {
    if (threadIdx.x < 32) {                       // warp 0
      const unsigned lane = threadIdx.x;
      if (rank == 0 && lane == 0) {               // the partition leader
        while (ld_acquire_gpu(&ps->done_gen) != seen) __nanosleep(32);
        uint32_t backoff = 32;
        uint64_t pub;
        uint32_t kc = 0xFFu, slot = 0;            // class and slot of an item claimed by this partition
        bool claimed = false;
        for (;;) {
          if (sib >= 0) {                         // lent to the sibling's item?
            const uint64_t hw = ld_acquire_gpu_u64(&ps->help);
            if (hw) {
              pub = (hw & 0xFFFFFFFF00000000ull) | (seen + 1);
              break;
            }
          }
          bool retry = false;
          // ring 0 (entries the host published at the model's wake) first, then the
          // eager ring: an eager entry waits at most one extra L2 read, ring 0 none
          for (int r = 0; r < nrings && !claimed; ++r) {
            const uint32_t h = *reinterpret_cast<volatile uint32_t*>(&heads[r]);
            const uint64_t e = ld_acquire_gpu_u64(&rings[(size_t)r * kRing + h % kRing]);
            if ((uint32_t)(e >> 32) != h + 1) continue;            // entry h of ring r not published
            if (sib >= 0 && atomicCAS(&ps->lock, 0u, kLockOwn) != 0u) {  // being lent: help first
              retry = true;
              break;
            }
            const uint64_t t_seen = globaltimer();
            if (atomicCAS(&heads[r], h, h + 1) == h) {
              ps->ring_idx = (uint32_t)r * kRing + h % kRing;
              ps->seq = h + 1;
#ifdef STRINGS_TSTART_AFTER_CAS
              ps->t_start = globaltimer();      // experiment: how long the claim CAS takes
#else
              ps->t_start = t_seen;
#endif
              ps->total = 0;                      // decided below, after the CTAs are released
              slot = cpart ? (uint32_t)e : ((uint32_t)e & 0xFFFFu);
              kc = cpart ? 0xFFu : (((uint32_t)e >> 16) & 0xFFu);
              claimed = true;
              pub = ((uint64_t)slot << 32) | (seen + 1);
            } else {
              if (sib >= 0) st_release_gpu(&ps->lock, 0u);
              retry = true;                       // the other KL slot took it
              break;
            }
          }
          if (claimed) break;
          if (retry) continue;
          if (ld_acquire_gpu(p.stop)) {
            pub = kStop;
            break;
          }
          if (p.flags & 1u) continue;
          __nanosleep(backoff);
          if (backoff < p.poll_max_ns) backoff <<= 1;
        }
        st_release_gpu_u64(&ps->gen, pub);        // the partition's CTAs start now
        if (claimed) {
          // an item of this partition (own claim): a streaming item borrows the
          // sibling slot's CTAs if that slot is idle.  Decided after the release:
          // the own CTAs claim chunks dynamically, so lent CTAs may join late
          uint32_t total = (uint32_t)S;
          if (sib >= 0 && (kc == 0 || kc == 2) && atomicCAS(&sps->lock, 0u, (uint32_t)q + 1) == 0u) {
            total += (uint32_t)S_sib;
            const uint64_t hw = (uint64_t)(kHelpGen | ((uint32_t)q << 16) | slot) << 32;
            st_release_gpu_u64(&sps->help, hw);
            // Start the sibling's CTAs at once rather than through its leader's
            // back-off poll of `help` (item 24.0 -> 23.7 us on C2, tools/item_ab.sh):
            // only when the sibling is fully idle -- its last item's done_gen
            // published (its completion step reads its gen word, and it releases the
            // lock before done_gen) -- which stays so while we hold its lock.  Its
            // leader, on seeing `help`, writes the same gen word again.
            const uint64_t sg = ld_acquire_gpu_u64(&sps->gen);
            if ((uint32_t)sg != kStop && ld_acquire_gpu(&sps->done_gen) == (uint32_t)sg)
              st_release_gpu_u64(&sps->gen, hw | (uint32_t)((uint32_t)sg + 1));
          }
          st_release_gpu(&ps->total, total);
        }
      }
      uint64_t gw = 0;
      if (lane == 0)                              // one poller per CTA
        while ((uint32_t)(gw = ld_acquire_gpu_u64(&ps->gen)) == seen) {
#ifndef STRINGS_GEN_SPIN
          __nanosleep(STRINGS_GEN_POLL_NS);
#endif
        }
      __syncwarp();                               // orders lane 0's acquire before the item loads
      gw = __shfl_sync(0xffffffffu, gw, 0);
      const uint32_t g = (uint32_t)gw, slot_word = (uint32_t)(gw >> 32);
      const bool lent = !cpart && g != kStop && (slot_word & kHelpGen);
      const uint32_t slot = lent ? (slot_word & 0xFFFFu) : slot_word;
      if (g != kStop && cpart) {
        // the 128-B copy item from the host-mapped table: one PCIe read by 8 lanes
        if (lane < sizeof(CopyItem) / 16)
          reinterpret_cast<uint4*>(&s_citem)[lane] = ld_cv_v4(reinterpret_cast<const uint4*>(p.citems + slot) + lane);
      } else if (g != kStop) {
        // the 512-B item straight from the device item table: one warp-wide L2 read
        // (.cg: the copy engine wrote it, no stale L1 line)
        uint4 v;
        asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                     : "l"(reinterpret_cast<const uint4*>(table + slot) + lane) : "memory");
        reinterpret_cast<uint4*>(&s_item)[lane] = v;
      }
      if (lane == 0) {
        s_gen = g;
        s_slot = slot;
        s_owner = lent ? ((slot_word >> 16) & 0x7FFFu) : (uint32_t)q;
      }
    }
    __syncthreads();
    const uint32_t g = s_gen;
    if (g == kStop) break;
    seen = g;
    if (threadIdx.x == 0) p.progress[blockIdx.x] = (g << 12) | (s_item.kclass << 8) | 1u;     // item read
    const bool lent = s_owner != (uint32_t)q;
    PartState* ops = p.parts + s_owner;          // the partition whose item this is
    // the owner partition's CTAs come first in the item's rank order
    const int S_owner = lent ? p.part_start[s_owner + 1] - p.part_start[s_owner] : S;
#ifdef STRINGS_TEXEC_FIRST
    // experiment: t_exec = the FIRST CTA (own or lent) to start the body
    if (!cpart && threadIdx.x == 0) atomicMin(reinterpret_cast<unsigned long long*>(&ops->t_exec), globaltimer());
#else
    if (!lent && rank == 0 && threadIdx.x == 0) ps->t_exec = globaltimer();
#endif
    if (cpart) {
      copy_body(s_citem, rank, S);
    } else {
      const KlItem it = s_item;
      if (it.job == p.fault_job) __trap();        // fault injection (tests the watchdog)
      // a lent CTA takes rank S_owner + rank; it claims the owner's streaming chunks
      // (the owner's GroupSync) and leaves a ragged tail to the owner's CTAs
      run_item(it, table + s_slot, true, lent ? S_owner + rank : rank, S_owner, sm, tmem, mma_phase, &ops->sync,
               &ops->total);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      p.progress[blockIdx.x] = (seen << 12) | 2u;                     // body done
      // CTAs on this item (own + lent), published by the owner's leader after it
      // released its CTAs (long ago by now: the load overlaps the fence below)
      uint32_t total = ld_acquire_gpu(&ops->total);
      // D2H copy items wrote host memory: their stores must be visible system-wide
      // before the completion word; everything else only needs gpu scope
      if (cpart && s_citem.to_host)
        __threadfence_system();
      else
        __threadfence();
      while (total == 0u) {
        __nanosleep(32);
        total = ld_acquire_gpu(&ops->total);
      }
      const uint32_t old = atomicAdd(&ops->done_cnt, 1u);
      p.progress[blockIdx.x] = (seen << 12) | 3u;                     // counted in
      if (old == total - 1) {                     // last CTA of the item (own or lent)
        ops->done_cnt = 0;
        ops->sync.chunk_next = 0;                 // streaming chunk counter for the next item
        const size_t di = (size_t)ld * kRings * kRing + ops->ring_idx;
        KlDone* d = cpart ? &p.cdone[ops->ring_idx] : &p.done[di];
        d->partition = s_owner;
        d->t_start = ops->t_start;
        d->t_exec = ops->t_exec;
#ifdef STRINGS_TEXEC_FIRST
        ops->t_exec = ~0ull;
#endif
        d->t_end = globaltimer();
        // Every CTA fenced its output writes at gpu scope before counting in, so the
        // outputs are in L2/HBM; the host reacts to this word only by issuing a D2H
        // DMA from device memory, so a gpu-scope fence + plain store is sufficient
        // (a sys-scope release costs ~3 us more per item, PCIe-fence round trip).
        __threadfence();
        d->seq = ops->seq;
        // the device copy an eager D2H's stream waits on (gpu scope: the copy engine
        // reads the outputs through L2, which every CTA's fence already ordered)
        if (!cpart) st_release_gpu(&p.done_dev[di], ops->seq);
        const uint32_t og = (uint32_t)*reinterpret_cast<volatile uint64_t*>(&ops->gen);
        if (sib >= 0 || lent) st_release_gpu(&ops->lock, 0u);   // the owner may claim / lend again
        st_release_gpu(&ops->done_gen, og);
      }
      if (lent) {                                  // this partition's own bookkeeping for the lent share
        const uint32_t o2 = atomicAdd(&ps->done_cnt, 1u);
        if (o2 == (uint32_t)S - 1) {
          ps->done_cnt = 0;
          st_release_gpu_u64(&ps->help, 0ull);     // before done_gen: the leader must not help twice
          st_release_gpu(&ps->lock, 0u);
          st_release_gpu(&ps->done_gen, seen);
        }
      }
    }
  }
  cta_teardown(tmem);
}

// Barrier/partials for stand-alone launches (one group-wide launch at a time
// per device; the counter returns to zero after every barrier).
__device__ GroupSync g_oneshot_sync;

// Stand-alone launch of one tenant body on `gridDim.x` CTAs (kernel-level
// checks outside the scheduler, and KL_MODE_LAUNCH).  One instantiation per
// kernel class, so each contains only its own body: the register allocation of
// one body no longer depends on the others (with every body in one kernel the
// SORT network ran 29% slower after an unrelated streaming-body change).
template <int KC>
__global__ void __launch_bounds__(kThreads, 1) oneshot_kernel(const __grid_constant__ KlItem it) {
  extern __shared__ __align__(1024) uint8_t smem[];
  GemmSmem sm = carve_smem(smem);
  uint32_t tmem = 0, mma_phase = 0;
  GroupSync* gs = it.sync ? reinterpret_cast<GroupSync*>(it.sync) : &g_oneshot_sync;
  const int rank = blockIdx.x, S = gridDim.x;
  if constexpr (KC != 1) mbar_setup(sm);          // (GEMM: cta_setup below)
  if constexpr (KC == 0) {
    stream_body<0>(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n,
                   it.alpha, it.seed, rank, S, sm.stage, sm.sbar, sm.scratch, sm.sphase, gs, nullptr);
  } else if constexpr (KC == 1) {
    tmem = cta_setup(sm);
    gemm_body(it.tmap_a, it.tmap_b, it.tmap_c, false, reinterpret_cast<float*>(it.out0), it.m, it.n, it.k, it.reps,
              rank, S, sm, tmem, mma_phase);
    cta_teardown(tmem);
  } else if constexpr (KC == 2) {
    stream_body<2>(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n,
                   it.alpha, it.seed, rank, S, sm.stage, sm.sbar, sm.scratch, sm.sphase, gs, nullptr);
  } else if constexpr (KC == 3) {
    hist_body(reinterpret_cast<const uint8_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n, rank, S, gs,
              sm.stage, sm.sbar, sm.sphase);
  } else if constexpr (KC == 4) {
    scan_body(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n, rank, S, gs,
              sm.stage, sm.sbar, sm.scratch, sm.sphase);
  } else {
    sort_body(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n, rank, S,
              sm.stage);
  }
}

// Clock calibration ping-pong: sample i is taken when the host raises flag to
// i+1; the kernel answers with %globaltimer (host-mapped memory both ways).
__global__ void clock_probe_kernel(const uint32_t* flag, uint64_t* out, int n) {
  for (int i = 0; i < n; ++i) {
    while (ld_acquire_sys(flag) != (uint32_t)(i + 1)) {
    }
    const uint64_t t = globaltimer();
    *reinterpret_cast<volatile uint64_t*>(out + i) = t;
    __threadfence_system();
  }
}

}  // namespace strings_dev

// ----------------------------------------------------------------- host side
namespace strings {

cudaError_t launch_dispatcher(const strings_dev::DispatchParams& p, int grid, cudaStream_t s) {
  cudaError_t e = cudaFuncSetAttribute(strings_dev::dispatcher_kernel,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)strings_dev::kSmemGemm);
  if (e != cudaSuccess) return e;
  // Every CTA must be resident at once (partition leaders and followers poll each
  // other, and the last CTA of a partition completes its item): a cooperative
  // launch guarantees co-residency or fails, instead of hanging when other work
  // holds some SMs at launch time.
  strings_dev::DispatchParams arg = p;
  void* args[] = {&arg};
  return cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(strings_dev::dispatcher_kernel), dim3(grid),
                                     dim3(strings_dev::kThreads), args, strings_dev::kSmemGemm, s);
}

cudaError_t launch_clock_probe(const uint32_t* flag, uint64_t* out, int n, cudaStream_t s) {
  strings_dev::clock_probe_kernel<<<1, 1, 0, s>>>(flag, out, n);
  return cudaGetLastError();
}

cudaError_t launch_oneshot(const strings_dev::KlItem& it, int ctas, cudaStream_t s) {
  // the smem opt-in is a per-device (per-context) function attribute: one flag per device
  if (it.kclass > 5) return cudaErrorInvalidValue;
  using K = void (*)(strings_dev::KlItem);
  static const K kernels[6] = {strings_dev::oneshot_kernel<0>, strings_dev::oneshot_kernel<1>,
                               strings_dev::oneshot_kernel<2>, strings_dev::oneshot_kernel<3>,
                               strings_dev::oneshot_kernel<4>, strings_dev::oneshot_kernel<5>};
  const K k = kernels[it.kclass];
  static std::atomic<bool> attr_set[64][6];
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64 || !attr_set[dev][it.kclass].load(std::memory_order_acquire)) {
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)strings_dev::kSmemGemm);
    if (e != cudaSuccess) return e;
    if (dev >= 0 && dev < 64) attr_set[dev][it.kclass].store(true, std::memory_order_release);
  }
  k<<<ctas, strings_dev::kThreads, strings_dev::kSmemGemm, s>>>(it);
  return cudaGetLastError();
}

}  // namespace strings
