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
//   2. polls its logical device's doorbell word in device memory (ld.acquire.gpu,
//      nanosleep back-off; the host writes the ring tail there with
//      cuStreamWriteValue32) and claims the next item with a CAS on the device
//      claim counter, then reads the item from the host-mapped ring.  Polling
//      L2 instead of host memory keeps the PCIe link free for the tenants'
//      DMA: with 16 leaders polling host memory the copy engines lost 4x
//      throughput (profiles/r01_doorbell.md),
//   3. copies the item into the partition mailbox and publishes gen+1
//      (st.release.gpu).
// Every CTA of the partition waits for the new generation, runs its share of
// the item, and the last CTA to finish writes the completion word and the
// %globaltimer stamps back to host memory (st.release.sys).
#include <cstdio>

#include "ctrl.hpp"

namespace strings_dev {

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
  __shared__ uint32_t s_gen;
  GemmSmem sm = carve_smem(smem);
  if ((smem_u32(smem) & 1023u) != 0) __trap();   // SWIZZLE_128B tiles need a 1 KB-aligned base
  const int NP = p.L * p.P;
  int q, start, S;
  partition_of(blockIdx.x, NP, p.part_start, &q, &start, &S);
  const int rank = blockIdx.x - start;
  const int ld = q / p.P;
  PartState* ps = p.parts + q;
  const uint32_t tmem = cta_setup(sm);
  uint32_t mma_phase = 0;
  uint32_t seen = 0;
  for (;;) {
    if (threadIdx.x == 0) {
      if (rank == 0) {
        while (ld_acquire_gpu(&ps->done_gen) != seen) __nanosleep(32);
        uint32_t g;
        uint32_t backoff = 32;
        const bool host_db = p.flags & 2u;
        for (;;) {
          const uint32_t tail = host_db ? ld_acquire_sys(&p.rings[ld].tail) : ld_acquire_gpu(&p.doorbells[32 * ld]);
          const uint32_t h = *reinterpret_cast<volatile uint32_t*>(&p.heads[ld]);
          if (h < tail) {
            if (atomicCAS(&p.heads[ld], h, h + 1) == h) {
              const KlItem* src = &p.rings[ld].items[h % kRing];
              // 16-B loads that bypass stale cached lines (.cv), issued back to back: one
              // PCIe round trip for the whole item instead of one per 32-bit field
              uint4 v[sizeof(KlItem) / 16];
#pragma unroll
              for (int w = 0; w < (int)(sizeof(KlItem) / 16); ++w)
                asm volatile("ld.global.cv.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(v[w].x), "=r"(v[w].y), "=r"(v[w].z), "=r"(v[w].w)
                             : "l"(reinterpret_cast<const uint4*>(src) + w));
              uint4* d4 = reinterpret_cast<uint4*>(&ps->item);
#pragma unroll
              for (int w = 0; w < (int)(sizeof(KlItem) / 16); ++w) d4[w] = v[w];
              ps->ring_idx = h % kRing;
              ps->t_start = globaltimer();
              g = seen + 1;
              break;
            }
            continue;
          }
          if (host_db ? ld_acquire_sys(&p.ctrl->shutdown) : ld_acquire_gpu(&p.doorbells[32 * p.L])) {
            g = kStop;
            break;
          }
          if (p.flags & 1u) continue;
          __nanosleep(backoff);
          if (backoff < p.poll_max_ns) backoff <<= 1;
        }
        st_release_gpu(&ps->gen, g);
      }
      uint32_t g;
      while ((g = ld_acquire_gpu(&ps->gen)) == seen) __nanosleep(32);
      s_gen = g;
      if (g != kStop) s_item = ps->item;
    }
    __syncthreads();
    const uint32_t g = s_gen;
    if (g == kStop) break;
    seen = g;
    const KlItem it = s_item;
    if (it.job == p.fault_job) __trap();          // fault injection (tests the watchdog)
    if (rank == 0 && threadIdx.x == 0) ps->t_exec = globaltimer();
    run_item(it, &ps->item, true, rank, S, sm, tmem, mma_phase, &ps->sync);
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      const uint32_t old = atomicAdd(&ps->done_cnt, 1u);
      if (old == (uint32_t)S - 1) {
        ps->done_cnt = 0;
        KlDone* d = &p.done[ld * kRing + ps->ring_idx];
        d->partition = (uint32_t)q;
        d->t_start = ps->t_start;
        d->t_exec = ps->t_exec;
        d->t_end = globaltimer();
        // Every CTA fenced its output writes at gpu scope before counting in, so the
        // outputs are in L2/HBM; the host reacts to this word only by issuing a D2H
        // DMA from device memory, so a gpu-scope fence + plain store is sufficient
        // (a sys-scope release costs ~3 us more per item, PCIe-fence round trip).
        __threadfence();
        d->seq = it.seq;
        st_release_gpu(&ps->done_gen, seen);
      }
    }
  }
  cta_teardown(tmem);
}

// Barrier/partials for stand-alone launches (one group-wide launch at a time
// per device; the counter returns to zero after every barrier).
__device__ GroupSync g_oneshot_sync;

// Stand-alone launch of one tenant body on `gridDim.x` CTAs (kernel-level
// checks outside the scheduler, and KL_MODE_LAUNCH).
__global__ void __launch_bounds__(kThreads, 1) oneshot_kernel(const __grid_constant__ KlItem it) {
  extern __shared__ __align__(1024) uint8_t smem[];
  GemmSmem sm = carve_smem(smem);
  uint32_t tmem = 0, mma_phase = 0;
  const bool gemm = it.kclass == 1;
  if (gemm) tmem = cta_setup(sm);
  GroupSync* gs = it.sync ? reinterpret_cast<GroupSync*>(it.sync) : &g_oneshot_sync;
  run_item(it, &it, false, blockIdx.x, gridDim.x, sm, tmem, mma_phase, gs);
  if (gemm) cta_teardown(tmem);
}

}  // namespace strings_dev

// ----------------------------------------------------------------- host side
namespace strings {

cudaError_t launch_dispatcher(const strings_dev::DispatchParams& p, int grid, cudaStream_t s) {
  cudaError_t e = cudaFuncSetAttribute(strings_dev::dispatcher_kernel,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)strings_dev::kSmemGemm);
  if (e != cudaSuccess) return e;
  strings_dev::dispatcher_kernel<<<grid, strings_dev::kThreads, strings_dev::kSmemGemm, s>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_oneshot(const strings_dev::KlItem& it, int ctas, cudaStream_t s) {
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(strings_dev::oneshot_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)strings_dev::kSmemGemm);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  strings_dev::oneshot_kernel<<<ctas, strings_dev::kThreads, strings_dev::kSmemGemm, s>>>(it);
  return cudaGetLastError();
}

}  // namespace strings
