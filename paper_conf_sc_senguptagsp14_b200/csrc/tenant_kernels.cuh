// tenant_kernels.cuh -- the three tenant kernel classes as device functions.
//
// Each body runs on a group of S CTAs (one SM partition of the persistent
// dispatcher, or a stand-alone grid); `rank` is this CTA's index in the group.
// Block = 256 threads.  Classes follow the paper's workload classes (Table I,
// PAPER.md L767-815) as made concrete in SURVEY.md §8(d):
//   VSCALE  y = alpha * x            fp32, one __fmul_rn per element (R-23)
//   XFER    y = fmix32(x ^ seed)     u32 (MurmurHash3 finaliser)
//   GEMM    C = A . B, R repetitions bf16 -> fp32, tcgen05 + TMEM (R-17, R-22)
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace strings_dev {

constexpr int kThreads = 256;

// One KL work item: built by the host at the job's H2D issue and DMA'd into the
// device item table with the job's inputs (ctrl.hpp).  GEMM items carry the TMA
// tensor maps of A, B and C (encoded on the host per job).
struct __align__(64) KlItem {
  uint32_t seq;          // claim number (1-based, monotone per ring); set by the claiming leader
  uint32_t kclass;
  uint64_t job;
  uint64_t in0, in1, out0;   // device pointers
  uint64_t n, m, k;
  uint32_t reps;
  float alpha;
  uint32_t seed;
  uint32_t pad;
  uint64_t t_issue;      // unused (telemetry is kept on the host)
  uint64_t sync;         // stand-alone launches: GroupSync* to use (0 = the default one)
  uint64_t pad3[4];
  uint8_t tmap_a[128];   // CUtensorMap of A (bf16 M x K, K-major, box 64 x 128, SWIZZLE_128B)
  uint8_t tmap_b[128];   // CUtensorMap of B (bf16 K x N, N-major, box 64 x 64,  SWIZZLE_128B)
  uint8_t tmap_c[128];   // CUtensorMap of C (fp32 M x N, N-major, box 32 x 128, SWIZZLE_128B)
};
static_assert(sizeof(KlItem) == 512, "KlItem layout");
static_assert(offsetof(KlItem, tmap_a) % 64 == 0, "tensor maps must be 64-B aligned");

// ---------------------------------------------------------- smem / mbarrier
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// Every mbarrier is initialised ONCE per kernel (mbar_setup at the kernel's
// start); items that re-use one track its phase parity across items (the stage
// and fill parities in GemmSmem::sphase, the MMA barrier's in mma_phase).
// Re-initialising a barrier per item, as round 1 did, was not reliable on
// sm_100a: the persistent dispatcher's second streaming item on a CTA could
// wait forever on its first stage (the new phase accounted an arrival twice).
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
constexpr int kTailBarriers = 14;    // stream/SCAN pipeline stages [0, kStreamStages), GEMM fill [kFillBar0, +4)
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t a = smem_u32(bar);
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n\t}"
      :: "r"(a), "r"(parity) : "memory");
}

// A "group" is the S CTAs running one item (an SM partition of the dispatcher,
// or a stand-alone grid).  All of them are co-resident (one CTA per SM), so a
// counter/generation barrier in global memory is safe.
constexpr int kScanRing = 8;          // SCAN: rows of GroupSync::wave (wave k uses row k mod 8)
struct __align__(128) GroupSync {
  uint32_t bar_cnt;
  uint32_t bar_gen;
  uint32_t chunk_next;                 // streaming items: next unclaimed 32 KB chunk (dynamic claiming)
  uint32_t chunk_done;                 // streaming items: CTAs finished claiming (the last one resets both)
  uint32_t scan_epoch;                 // SCAN items finished on this group (tags the wave table)
  uint32_t scan_done;                  // CTAs finished with the current SCAN item (the last one bumps the epoch)
  uint32_t pad[26];
  uint32_t partial[256];               // per-CTA partial results (S <= 256)
  uint64_t wave[kScanRing * 256];      // SCAN: (tag << 32) | sum of rank r's part of wave k, at [(k % 8) * 256 + r]
};

// ---------------------------------------------------------------- streaming
__device__ __forceinline__ uint32_t fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6Bu;
  h ^= h >> 13;
  h *= 0xC2B2AE35u;
  h ^= h >> 16;
  return h;
}

__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ void st_stream(uint4* p, uint4 v) {
  asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};"
               :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

template <int KCLASS>
__device__ __forceinline__ uint32_t elem_op(uint32_t x, float alpha, uint32_t seed) {
  if constexpr (KCLASS == 0) return __float_as_uint(__fmul_rn(__uint_as_float(x), alpha));
  else return fmix32(x ^ seed);
}

// Vectorised grid-stride stream over the group's CTAs: 8 independent 16-B
// loads in flight per thread (32 KB per CTA) to cover HBM latency.
// LDG/STG fallback: vectorised grid-stride over elements [e0, e1) of the group
// (used for unaligned buffers and for the tail after the bulk-copy chunks).
template <int KCLASS>
__device__ void stream_ldg(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t e0, uint64_t e1,
                           float alpha, uint32_t seed, int rank, int S) {
  constexpr int U = 8;
  const uint64_t tid = (uint64_t)rank * kThreads + threadIdx.x;
  const uint64_t nthreads = (uint64_t)S * kThreads;
  const bool aligned = ((reinterpret_cast<uintptr_t>(x + e0) | reinterpret_cast<uintptr_t>(y + e0)) & 15) == 0;
  const uint64_t nvec = aligned ? (e1 - e0) / 4 : 0;
  const uint4* xv = reinterpret_cast<const uint4*>(x + e0);
  uint4* yv = reinterpret_cast<uint4*>(y + e0);
  uint64_t i = tid;
  for (; i + (U - 1) * nthreads < nvec; i += U * nthreads) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ld_stream(xv + i + u * nthreads);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      v[u].x = elem_op<KCLASS>(v[u].x, alpha, seed);
      v[u].y = elem_op<KCLASS>(v[u].y, alpha, seed);
      v[u].z = elem_op<KCLASS>(v[u].z, alpha, seed);
      v[u].w = elem_op<KCLASS>(v[u].w, alpha, seed);
      st_stream(yv + i + u * nthreads, v[u]);
    }
  }
  for (; i < nvec; i += nthreads) {
    uint4 v = ld_stream(xv + i);
    v.x = elem_op<KCLASS>(v.x, alpha, seed);
    v.y = elem_op<KCLASS>(v.y, alpha, seed);
    v.z = elem_op<KCLASS>(v.z, alpha, seed);
    v.w = elem_op<KCLASS>(v.w, alpha, seed);
    st_stream(yv + i, v);
  }
  for (uint64_t e = e0 + nvec * 4 + tid; e < e1; e += nthreads) y[e] = elem_op<KCLASS>(x[e], alpha, seed);
}

// 6 x 32 KB stages, loads 4 chunks ahead, one bulk store allowed in flight
// while its stage is refilled two iterations later (profiles/r01_stream_lead.jsonl:
// the fastest race-free shape, XFER 2^24 on 74 SMs 29.2 us, 2^28 on 148 SMs 0.95
// of peak; 4 x 48 KB with a 3-chunk lead must wait for every store to read out
// (34.8 us)).
#ifndef STRINGS_STREAM_STAGES
#define STRINGS_STREAM_STAGES 6
#endif
#ifndef STRINGS_STREAM_CHUNK_KB
#define STRINGS_STREAM_CHUNK_KB 32
#endif
#ifndef STRINGS_STREAM_LEAD
#define STRINGS_STREAM_LEAD (STRINGS_STREAM_STAGES - 2)
#endif
constexpr int kStreamStages = STRINGS_STREAM_STAGES;                 // stage count (<= 12 mbarriers in the tail)
constexpr uint32_t kStreamChunk = STRINGS_STREAM_CHUNK_KB * 1024;    // bytes per stage (6 x 32 KB = 192 KB)
// Loads run kStreamLead chunks ahead of the chunk being processed.  The stage a
// new load refills was last stored by the chunk kStreamStages - kStreamLead
// iterations back; before the load overwrites it, that bulk store must have
// finished READING shared memory, i.e. at most kStreamStages - kStreamLead - 1
// newer store groups may still be pending (cp.async.bulk.wait_group.read N).
// Minimum chunks per CTA for the pipeline (below: LDG path).  0 = always the
// pipeline: at 4 MiB on 18-72 CTAs the two paths are within +-10% either way, only
// 16 MiB on 72 CTAs gains from the LDG path (profiles/r01_small_item.jsonl).
#ifndef STRINGS_STREAM_MIN_CHUNKS
#define STRINGS_STREAM_MIN_CHUNKS 0
#endif
#ifndef STRINGS_STREAM_TAIL_SPLIT
#define STRINGS_STREAM_TAIL_SPLIT 1
#endif
constexpr int kStreamTailSplit = STRINGS_STREAM_TAIL_SPLIT;
constexpr int kStreamLead = STRINGS_STREAM_LEAD;
constexpr int kStreamMinChunks = STRINGS_STREAM_MIN_CHUNKS;
constexpr int kStreamStoreSlack = kStreamStages - kStreamLead - 1;
static_assert(kStreamStages >= 3 && kStreamStages <= 12, "stream stages");
constexpr int kFillBar0 = kStreamStages;   // first GEMM fill barrier in the smem tail (after the stages)
static_assert(kFillBar0 + 4 <= kTailBarriers, "tail barriers: stages + 4 GEMM fill barriers");
static_assert(kStreamLead >= 1 && kStreamLead < kStreamStages, "stream lead");

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(
                   static_cast<uint32_t>(__cvta_generic_to_shared(bar))), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(dst))), "l"(src), "r"(bytes),
                  "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
               :: "l"(dst), "r"(static_cast<uint32_t>(__cvta_generic_to_shared(src))), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

// Streaming body: the buffer is cut into 32 KB chunks.  The first kStreamLead
// rounds go statically to the group's own CTAs (no atomic before the first
// loads); the rest are CLAIMED dynamically from a per-item counter
// (GroupSync::chunk_next): CTAs that
// start late (an idle sibling partition lending its SMs joins a microsecond or
// two after the owner's) or run slower simply take fewer chunks, so the item
// ends when the bytes are done rather than when the slowest CTA's static share
// is.  Each CTA runs a 6-stage TMA bulk-copy pipeline through shared memory
// (cp.async.bulk global->smem with mbarrier completion, the element op in smem,
// cp.async.bulk smem->global), keeping 4 chunks (128 KB) of loads in flight per
// SM while the previous chunk's store drains; thread 0 claims the chunk of a
// load one iteration before it issues it (so the atomic's round trip is off the
// pipeline's critical path) and records it for the stage in smem (`cid`).
// A stage whose claim came back empty gets an arrive without bytes and the id
// kNoChunk, which ends the CTA's loop.  The last CTA to finish claiming resets
// the counter for the group's next item (inside the dispatcher, total_word set,
// the item's last CTA does, in its completion step).  Unaligned buffers and the tail (the last
// partial chunk) use the LDG path with a static split over ranks < S (a lent
// CTA has rank >= S and skips it).
constexpr uint32_t kNoChunk = 0xFFFFFFFFu;
// Stage phase parities after `used` more pipeline positions (position i uses
// stage i mod kStreamStages once).
__device__ __forceinline__ uint32_t stage_phases_after(uint32_t bits, uint64_t used) {
  for (int st = 0; st < kStreamStages; ++st) {
    const uint64_t uses = used > (uint64_t)st ? (used - 1 - st) / kStreamStages + 1 : 0;
    bits ^= (uint32_t)(uses & 1) << st;
  }
  return bits;
}

template <int KCLASS>
__device__ void stream_body(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t n,
                            float alpha, uint32_t seed, int rank, int S, uint8_t* stage, uint64_t* sbar,
                            uint32_t* cid, uint32_t* sphase, GroupSync* gs, const uint32_t* total_word) {
  const bool aligned = ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(y)) & 15) == 0;
  const uint64_t bytes = n * 4;
  // items too small to fill the pipeline (fewer than kStreamMinChunks chunks per CTA)
  // take the LDG path, whose first loads go out without a pipeline fill
  const uint64_t nchunks =
      aligned && bytes / kStreamChunk >= (uint64_t)S * kStreamMinChunks ? bytes / kStreamChunk : 0;
  if (nchunks) {
    const uint8_t* xb = reinterpret_cast<const uint8_t*>(x);
    uint8_t* yb = reinterpret_cast<uint8_t*>(y);
    uint32_t next = kNoChunk;                     // thread 0: the claim for the next load
    bool claiming = true;                         // thread 0: the counter may still hold chunks
    // The first kStreamLead rounds are dealt statically to the group's own CTAs
    // (chunk r + j*D over D dealt ranks): their loads go out at once, with no atomic
    // round trip on the item's start-up path; the counter hands out the chunks after
    // them.  Inside the dispatcher (total_word set) rank 0 hosts the partition
    // leader, which starts its own share last (claim, release, lending decision), so
    // it takes counter chunks only.
    const int d0 = total_word ? 1 : 0;            // first dealt rank
    const int D = S - d0;                         // dealt ranks
    // The last `split` whole chunks are handed out as half chunks, so the CTAs
    // (own and lent) run out of work closer together at the item's end.  Units
    // [0, nfull) are whole chunks, [nfull, nunits) halves of the rest.
    const uint64_t split = kStreamTailSplit ? (nchunks / 4 < 2ull * S ? nchunks / 4 : 2ull * S) : 0;
    const uint64_t nfull = nchunks - split, nunits = nfull + 2 * split;
    auto unit_off = [&](uint32_t u) -> uint64_t {
      return u < nfull ? (uint64_t)u * kStreamChunk : nfull * kStreamChunk + (u - nfull) * (uint64_t)(kStreamChunk / 2);
    };
    auto unit_bytes = [&](uint32_t u) -> uint32_t { return u < nfull ? kStreamChunk : kStreamChunk / 2; };
    const uint64_t dealt = D <= 0 ? 0 : (nunits < (uint64_t)kStreamLead * D ? nunits : (uint64_t)kStreamLead * D);
    int pre = 0;                                  // thread 0: statically dealt chunks used so far
    auto claim = [&]() -> uint32_t {
      if (rank >= d0 && rank < S && pre < kStreamLead) {
        const uint64_t c = (uint64_t)(rank - d0) + (uint64_t)(pre++) * D;
        if (c < dealt) return (uint32_t)c;
        pre = kStreamLead;                        // this CTA's static share is used up
      }
      const uint64_t c = dealt + atomicAdd(&gs->chunk_next, 1u);
      return c < nunits ? (uint32_t)c : kNoChunk;
    };
    // thread 0: fill stage st with the chunk claimed earlier (or end the CTA's loop there)
    auto issue = [&](int st) {
      const uint32_t c = claiming ? next : kNoChunk;
      cid[st] = c;
      if (c == kNoChunk) {
        claiming = false;
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(&sbar[st])) : "memory");
        return;
      }
      mbar_expect_tx(&sbar[st], unit_bytes(c));
      bulk_g2s(stage + st * kStreamChunk, xb + unit_off(c), unit_bytes(c), &sbar[st]);
      next = claim();                             // consumed at the next issue
    };
    // the stage barriers live for the whole kernel (mbar_setup); their phase
    // parities carry over from item to item in *sphase (bit st = stage st)
    const uint32_t ph0 = *reinterpret_cast<volatile uint32_t*>(sphase);
    if (threadIdx.x == 0) {
      next = claim();
      for (int st = 0; st < kStreamLead && claiming; ++st) issue(st);
    }
    __syncthreads();
    uint64_t i = 0;
    for (;; ++i) {
      const int st = (int)(i % kStreamStages);
      const uint32_t ph = ((ph0 >> st) & 1u) ^ (uint32_t)((i / kStreamStages) & 1);
      if (threadIdx.x == 0 && claiming) {
        const int s2 = (int)((i + kStreamLead) % kStreamStages);
        // stage s2 was last stored at iteration i + kStreamLead - kStreamStages: that
        // store must have finished reading smem before the load overwrites it
        if (i + kStreamLead >= (uint64_t)kStreamStages)
          asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(kStreamStoreSlack) : "memory");
        issue(s2);
      }
      mbar_wait(&sbar[st], ph);
      const uint32_t c = *reinterpret_cast<volatile uint32_t*>(&cid[st]);
      if (c == kNoChunk) break;                   // every thread sees the same end stage
      uint4* buf = reinterpret_cast<uint4*>(stage + st * kStreamChunk);
      const int nv = (int)(unit_bytes(c) / 16);
#pragma unroll 4
      for (int j = threadIdx.x; j < nv; j += kThreads) {
        uint4 v = buf[j];
        v.x = elem_op<KCLASS>(v.x, alpha, seed);
        v.y = elem_op<KCLASS>(v.y, alpha, seed);
        v.z = elem_op<KCLASS>(v.z, alpha, seed);
        v.w = elem_op<KCLASS>(v.w, alpha, seed);
        buf[j] = v;
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // smem writes -> async proxy
      __syncthreads();
      if (threadIdx.x == 0) bulk_s2g(yb + unit_off(c), stage + st * kStreamChunk, unit_bytes(c));
    }
    if (threadIdx.x == 0) {
      *sphase = stage_phases_after(ph0, i + 1);   // positions 0..i (the end marker's included) used a phase
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");                   // writes done
      asm volatile("fence.proxy.async.global;" ::: "memory");                     // async -> generic
      // every claim of this CTA has returned (the last one came back empty and was
      // consumed): count out; the last CTA of a stand-alone group resets the
      // counter.  Inside the dispatcher (total_word set) the item's last CTA
      // resets it instead, in the completion step it runs anyway.
      if (!total_word) {
        __threadfence();
        if (atomicAdd(&gs->chunk_done, 1u) == (uint32_t)S - 1) {
          atomicExch(&gs->chunk_next, 0u);
          atomicExch(&gs->chunk_done, 0u);
          __threadfence();
        }
      }
    }
    __syncthreads();                              // cid / stages free for the next item
  }
  if (rank < S) stream_ldg<KCLASS>(x, y, nchunks * (kStreamChunk / 4), n, alpha, seed, rank, S);
}

// --------------------------------------------------------------------- GEMM
// Tile 128 x 256 (M x N) per CTA, whole K (<= 256) resident in shared memory in
// the UMMA canonical SWIZZLE_128B layouts that TMA tensor loads produce:
//   A (K-major, M x K row-major): 4 K-slabs of 64 elements; slab c = 128 rows x
//     128 B (16 KB) at c*16 KB, 16-B chunks XOR-swizzled by row%8 inside each
//     1 KB atom of 8 rows.  UMMA desc: SBO = 1024 (8-row atom), LBO unused (16);
//     a K=16 step inside a slab advances the start address by 32 B.
//   B (MN-major, K x N row-major): 4 N-slabs of 64 elements; slab j = 256 k-rows x
//     128 B (32 KB) at 64 KB + j*32 KB.  UMMA desc: LBO = 32 KB (next N-slab),
//     SBO = 1024 (8 k-rows); a K=16 step advances the start by 16 rows = 2 KB.
// The fill is split into four K-chunks (A slab c + the 64 k-rows c of every B
// slab, 48 KB), each completing its own mbarrier, so the first repetition's MMAs
// start as soon as their chunk has landed.
constexpr int kTileM = 128, kTileN = 256, kMaxK = 256;
constexpr uint32_t kSmemA = kTileM * kMaxK * 2;          // 64 KB
constexpr uint32_t kSmemB = kTileN * kMaxK * 2;          // 128 KB
// The streaming stages alias the GEMM operand smem (and may extend past it); the
// 128-B tail of mbarriers / TMEM slot sits after the larger of the two.
constexpr uint32_t kSmemMain = (kStreamStages * kStreamChunk > kSmemA + kSmemB) ? kStreamStages * kStreamChunk
                                                                                 : kSmemA + kSmemB;
constexpr uint32_t kSmemGemm = kSmemMain + 256;          // dynamic smem of the dispatcher / one-shot kernels
                                                         // (tail: 128 B mbarriers / TMEM slot + 128 B scratch)
static_assert(kSmemGemm + 2048 <= 227 * 1024, "dynamic + static smem must fit one CTA per SM");
constexpr uint32_t kTmemCols = 256;                      // fp32 accumulator 128 x 256
constexpr uint32_t kSlabA = 128 * 128;                   // 16 KB
constexpr uint32_t kSlabB = 256 * 128;                   // 32 KB
constexpr uint32_t kChunkB = 64 * 128;                   // 64 k-rows of one B slab: 8 KB

// Shared-memory matrix descriptor (sm_100 UMMA): start>>4 [0,14), LBO>>4 [16,30),
// SBO>>4 [32,46), version=1 [46,48), base offset 0, layout [61,64) (2 = SWIZZLE_128B).
__device__ __forceinline__ uint64_t umma_desc_sw128(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

// Instruction descriptor kind::f16: D=f32 [4,6)=1, A=bf16 [7,10)=1, B=bf16 [10,13)=1,
// A K-major (bit 15 = 0), B MN-major (bit 16 = 1), N>>3 at [17,23), M>>4 at [24,29).
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int M, int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(N >> 3) << 17) |
         ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void tmem_alloc(uint32_t* slot_smem, uint32_t cols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
               :: "r"(smem_u32(slot_smem)), "r"(cols) : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t cols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(taddr), "r"(cols) : "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

__device__ __forceinline__ void umma_bf16(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc,
                                          uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
      :: "r"(tmem_d), "l"(da), "l"(db), "r"(idesc), "r"(accumulate) : "memory");
}
__device__ __forceinline__ void umma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
               :: "r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]),
        "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]),
        "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// TMA 2D tile store from shared memory (bulk async-group completion).
__device__ __forceinline__ void tma_store_2d(const void* tmap, const void* src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];"
               :: "l"(tmap), "r"(smem_u32(src)), "r"(c0), "r"(c1) : "memory");
}

// TMA 2D tile load (tensor map in global or param space) completing on `bar`.
__device__ __forceinline__ void tma_load_2d(void* dst, const void* tmap, int c0, int c1, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
      :: "r"(smem_u32(dst)), "l"(tmap), "r"(c0), "r"(c1), "r"(smem_u32(bar)) : "memory");
}

struct GemmSmem {
  uint8_t* a;          // kSmemA bytes, 1024-B aligned
  uint8_t* b;          // kSmemB bytes
  uint64_t* bar;       // MMA-completion mbarrier
  uint32_t* tmem_slot; // TMEM base written by tcgen05.alloc
  uint8_t* stage;      // streaming stages (aliases a/b: a CTA runs one item at a time)
  uint64_t* sbar;      // streaming stage mbarriers / GEMM fill mbarriers [4]
  uint32_t* scratch;   // 32 words outside the stages (SCAN warp totals)
  uint32_t* sphase;    // phase parities of the pipeline stage barriers (bit per stage), kept across items
};

// Units u = tile * R + rep, tile = (mt, nt); this CTA takes the contiguous
// chunk [rank*U/S, (rank+1)*U/S).  Each repetition is a full 16-MMA chain into
// the TMEM accumulator; C is written from repetition R-1 (R-17).  tmap_a/tmap_b
// point to the job's tensor maps (global memory: tmap_global = true, each
// consumer fences the tensormap proxy; kernel-parameter space otherwise).
__device__ inline void gemm_body(const void* tmap_a, const void* tmap_b, const void* tmap_c, bool tmap_global,
                                 float* __restrict__ C, uint64_t M, uint64_t N, uint64_t K, uint32_t R,
                                 int rank, int S, const GemmSmem& sm, uint32_t tmem_base, uint32_t& mma_phase) {
  const uint64_t tiles_n = N / kTileN, tiles = (M / kTileM) * tiles_n;
  const uint64_t U = tiles * R;
  const uint64_t u0 = (U * rank) / S, u1 = (U * (rank + 1)) / S;
  const uint32_t idesc = umma_idesc_bf16(kTileM, kTileN);
  const uint32_t a_base = smem_u32(sm.a), b_base = smem_u32(sm.b);
  const int kchunks = (int)(K / 64);
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0 && tmap_global && u0 < u1) {
    asm volatile("fence.proxy.tensormap::generic.acquire.gpu [%0], 128;" :: "l"(tmap_a) : "memory");
    asm volatile("fence.proxy.tensormap::generic.acquire.gpu [%0], 128;" :: "l"(tmap_b) : "memory");
    asm volatile("fence.proxy.tensormap::generic.acquire.gpu [%0], 128;" :: "l"(tmap_c) : "memory");
  }
  // fill barrier c's phase parity: bit 8 + c of *sm.sphase (only thread 0 uses them)
  uint32_t fph = threadIdx.x == 0 ? (*sm.sphase >> 8) & 0xFu : 0u;
  uint64_t u = u0;
  while (u < u1) {
    const uint64_t tile = u / R;
    const uint64_t last = min(u1, (tile + 1) * R);        // exclusive end of this tile's run
    const uint64_t mt = tile / tiles_n, nt = tile % tiles_n;
    if (threadIdx.x == 0) {
      for (int c = 0; c < kchunks; ++c) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
                     :: "r"(smem_u32(&sm.sbar[kFillBar0 + c])), "r"(kSlabA + 4 * kChunkB) : "memory");
        tma_load_2d(sm.a + c * kSlabA, tmap_a, 64 * c, (int)(mt * kTileM), &sm.sbar[kFillBar0 + c]);
#pragma unroll
        for (int j = 0; j < 4; ++j)
          tma_load_2d(sm.b + j * kSlabB + c * kChunkB, tmap_b, (int)(nt * kTileN) + 64 * j, 64 * c,
                      &sm.sbar[kFillBar0 + c]);
      }
      for (uint64_t v = u; v < last; ++v) {
        for (int c = 0; c < kchunks; ++c) {
          if (v == u) {
            mbar_wait(&sm.sbar[kFillBar0 + c], (fph >> c) & 1u);
            tc_fence_after();
          }
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            const int ks = 4 * c + kk;
            const uint64_t da = umma_desc_sw128(a_base + c * kSlabA + kk * 32, 16, 1024);
            const uint64_t db = umma_desc_sw128(b_base + ks * 2048, kSlabB, 1024);
            umma_bf16(tmem_base, da, db, idesc, ks > 0 ? 1u : 0u);
          }
        }
      }
      umma_commit(sm.bar);            // arrives when every MMA above has completed
      fph ^= (1u << kchunks) - 1u;    // each fill barrier completed one phase in this run
    }
    __syncwarp();
    mbar_wait(sm.bar, mma_phase);
    mma_phase ^= 1;
    tc_fence_after();
    if ((last - 1) % R == R - 1) {    // this run contains the final repetition: epilogue
      // TMEM -> registers -> smem staging in the TMA SWIZZLE_128B layout of a
      // 32-column x 128-row fp32 box (row r at r*128 B, 16-B chunk q at q ^ (r%8):
      // the 8 lanes of a store phase hit 8 different chunks, no bank conflicts)
      // -> eight TMA tensor stores of the 128 x 256 tile.  A/B smem is free: every
      // MMA has completed (sm.bar).
      const int lane_base = (warp & 3) * 32;
      const int col0 = (warp >> 2) * 128;
      const int r = lane_base + lane;
#pragma unroll 1
      for (int cc = 0; cc < 128; cc += 32) {
        uint32_t v[32];
        tmem_ld32(tmem_base + ((uint32_t)lane_base << 16) + (uint32_t)(col0 + cc), v);
        uint8_t* box = sm.a + ((col0 + cc) / 32) * (128 * 128);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          uint4 w = make_uint4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
          *reinterpret_cast<uint4*>(box + r * 128 + ((q ^ (r & 7)) << 4)) = w;
        }
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // smem writes -> async proxy
      __syncthreads();
      if (threadIdx.x == 0) {
#pragma unroll
        for (int g = 0; g < 8; ++g)
          tma_store_2d(tmap_c, sm.a + g * (128 * 128), (int)(nt * kTileN) + 32 * g, (int)(mt * kTileM));
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");    // C written before the item ends
        asm volatile("fence.proxy.async.global;" ::: "memory");
      }
    }
    tc_fence_before();
    __syncthreads();                  // smem and TMEM free for the next run
    u = last;
  }
  if (threadIdx.x == 0 && u0 < u1) *sm.sphase = (*sm.sphase & ~0xF00u) | (fph << 8);
  __syncthreads();
}

// ------------------------------------------------------- group coordination
// A "group" is the S CTAs running one item (an SM partition of the dispatcher,
// or a stand-alone grid).  All of them are co-resident (one CTA per SM), so a
// counter/generation barrier in global memory is safe.

__device__ __forceinline__ void group_barrier(GroupSync* gs, int S) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t gen = *reinterpret_cast<volatile uint32_t*>(&gs->bar_gen);
    if (atomicAdd(&gs->bar_cnt, 1u) == (uint32_t)S - 1) {
      *reinterpret_cast<volatile uint32_t*>(&gs->bar_cnt) = 0;
      __threadfence();
      atomicAdd(&gs->bar_gen, 1u);
    } else {
      while (*reinterpret_cast<volatile uint32_t*>(&gs->bar_gen) == gen) __nanosleep(20);
    }
    __threadfence();
  }
  __syncthreads();
}

// ---------------------------------------------------- HIST (Table I: HI)
// bins[256] (u32) = byte histogram of x[n].  Counting is bound by the SM's
// shared-memory atomic rate, not by HBM (one ATOMS per byte;
// tools/hist_probe.cu, profiles/r02_hist.md).  Counters are lane-private,
// [bin][lane] u32, so a warp's 32 atomics hit 32 different banks whatever
// the bytes are, and there are two copies (even / odd warps) so fewer warps
// contend for one word; each copy is 32 KB at the front of the stage area.
// Whole 32 KB chunks stream through a 4-stage TMA bulk pipeline (chunks dealt
// statically, chunk c to rank c mod S) once there is at least
// kHistBulkMinChunks per CTA; the rest (the tail, or buffers too small for
// one chunk per CTA) use 16-B LDGs, 8 in flight per thread, and unaligned
// buffers byte loads.  From cold L2 the pipeline wins at every size measured
// (2^26 bytes on 148 / 72 CTAs: 0.40 / 0.25 of the HBM peak vs 0.31 / 0.21
// with LDGs; tools/hist_ab.sh).  Then each
// thread sums one bin over both copies and the 32 lanes, rank 0 zeroes the
// output before the group barrier, and one global atomicAdd per non-zero bin.
constexpr int kHistCopies = 2;
constexpr uint32_t kHistCounterBytes = kHistCopies * 256 * 32 * 4;      // 64 KB
constexpr int kHistStages = 4;
constexpr uint32_t kHistChunk = 32768;
#ifndef STRINGS_HIST_BULK_MIN_CHUNKS
#define STRINGS_HIST_BULK_MIN_CHUNKS 1
#endif
constexpr uint64_t kHistBulkMinChunks = STRINGS_HIST_BULK_MIN_CHUNKS;
static_assert(kHistCounterBytes + kHistStages * kHistChunk <= kSmemMain, "HIST smem");
static_assert(kHistStages <= kStreamStages, "HIST uses the first stage barriers");

__device__ __forceinline__ void hist_word(uint32_t* mine, uint32_t w) {
#pragma unroll
  for (int b = 0; b < 4; ++b) atomicAdd(&mine[((w >> (8 * b)) & 0xFF) * 32], 1u);
}
__device__ __forceinline__ void hist_vec(uint32_t* mine, uint4 q) {
  hist_word(mine, q.x);
  hist_word(mine, q.y);
  hist_word(mine, q.z);
  hist_word(mine, q.w);
}

__device__ inline void hist_body(const uint8_t* __restrict__ x, uint32_t* __restrict__ bins, uint64_t n,
                                 int rank, int S, GroupSync* gs, uint8_t* stage, uint64_t* sbar, uint32_t* sphase) {
  uint32_t* sh = reinterpret_cast<uint32_t*>(stage);            // [kHistCopies][256 bins][32 lanes]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < (int)(kHistCounterBytes / 16); i += kThreads)
    reinterpret_cast<uint4*>(sh)[i] = make_uint4(0, 0, 0, 0);
  if (rank == 0)
    for (int i = threadIdx.x; i < 256; i += kThreads) bins[i] = 0;
  __syncthreads();
  uint32_t* mine = sh + (warp % kHistCopies) * (256 * 32) + lane;
  const bool aligned = (reinterpret_cast<uintptr_t>(x) & 15) == 0;
  const uint64_t nch = aligned ? n / kHistChunk : 0;
  const uint64_t my_ch = nch > (uint64_t)rank ? (nch - 1 - rank) / S + 1 : 0;
  uint64_t done_bytes = 0;                                      // bytes [0, done_bytes) counted by the bulk path
  if (nch >= (uint64_t)S * kHistBulkMinChunks) {
    uint8_t* st = stage + kHistCounterBytes;
    const uint32_t ph0 = *reinterpret_cast<volatile uint32_t*>(sphase);
    if (threadIdx.x == 0)
      for (int s = 0; s < kHistStages && (uint64_t)s < my_ch; ++s) {
        mbar_expect_tx(&sbar[s], kHistChunk);
        bulk_g2s(st + s * kHistChunk, x + (rank + (uint64_t)s * S) * kHistChunk, kHistChunk, &sbar[s]);
      }
    for (uint64_t i = 0; i < my_ch; ++i) {
      const int s = (int)(i % kHistStages);
      mbar_wait(&sbar[s], ((ph0 >> s) & 1u) ^ (uint32_t)((i / kHistStages) & 1));
      const uint4* b4 = reinterpret_cast<const uint4*>(st + s * kHistChunk);
#pragma unroll 4
      for (int j = threadIdx.x; j < (int)(kHistChunk / 16); j += kThreads) hist_vec(mine, b4[j]);
      __syncthreads();                                          // stage s read by every thread
      if (threadIdx.x == 0 && i + kHistStages < my_ch) {
        mbar_expect_tx(&sbar[s], kHistChunk);
        bulk_g2s(st + s * kHistChunk, x + (rank + (i + kHistStages) * S) * kHistChunk, kHistChunk, &sbar[s]);
      }
    }
    if (threadIdx.x == 0) {                                     // barrier s completed ceil((my_ch - s) / 4) phases
      uint32_t bits = ph0;
      for (int s = 0; s < kHistStages; ++s) {
        const uint64_t uses = my_ch > (uint64_t)s ? (my_ch - 1 - s) / kHistStages + 1 : 0;
        bits ^= (uint32_t)(uses & 1) << s;
      }
      *sphase = bits;
    }
    done_bytes = nch * kHistChunk;
  }
  // LDG path over [done_bytes, n): 16-B vectors (8 in flight per thread), then bytes
  const uint64_t tid = (uint64_t)rank * kThreads + threadIdx.x, nt = (uint64_t)S * kThreads;
  const uint64_t nv = aligned ? (n - done_bytes) / 16 : 0;
  const uint4* x4 = reinterpret_cast<const uint4*>(x + done_bytes);
  constexpr int U = 8;
  uint64_t v = tid;
  for (; v + (U - 1) * nt < nv; v += U * nt) {
    uint4 q[U];
#pragma unroll
    for (int u = 0; u < U; ++u) q[u] = ld_stream(x4 + v + u * nt);
#pragma unroll
    for (int u = 0; u < U; ++u) hist_vec(mine, q[u]);
  }
  for (; v < nv; v += nt) hist_vec(mine, ld_stream(x4 + v));
  for (uint64_t e = done_bytes + nv * 16 + tid; e < n; e += nt) atomicAdd(&mine[(uint32_t)x[e] * 32], 1u);
  __syncthreads();
  uint32_t total = 0;                                           // thread t owns bin t
#pragma unroll
  for (int c = 0; c < kHistCopies; ++c)
    for (int l = 0; l < 32; ++l) total += sh[c * (256 * 32) + threadIdx.x * 32 + ((l + threadIdx.x) & 31)];
  group_barrier(gs, S);                                         // output zeroed by rank 0
  if (total) atomicAdd(&bins[threadIdx.x], total);
}

// ---------------------------------------------------- SCAN (Table I: SC)
// y = inclusive prefix sum of x (u32, mod 2^32) over the whole group:
// per-CTA chunk sums -> group barrier -> chunk offset -> tiled block scan.
template <int O>
__device__ __forceinline__ void shfl_up_add(uint32_t& v) {
  asm("{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
      "shfl.sync.up.b32 t|p, %0, %1, 0, 0xffffffff;\n\t"
      "@p add.u32 %0, %0, t;\n\t}"
      : "+r"(v) : "n"(O));
}
// shfl.up's predicate output says whether the source lane exists: one SHFL and
// one predicated add per step (the C form compiled to SHFL + SEL + IADD)
__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v) {
  shfl_up_add<1>(v);
  shfl_up_add<2>(v);
  shfl_up_add<4>(v);
  shfl_up_add<8>(v);
  shfl_up_add<16>(v);
  return v;
}

// Tiles of 256 threads x 32 consecutive elements (32 KB): each thread loads its
// 32 with eight 16-B loads (all in flight at once), scans them in registers,
// and the warp / CTA totals give its offset; chunks are whole tiles, so every
// CTA's loads stay 16-B aligned when the buffers are.
constexpr int kScanPT = 32;
// One 32 KB chunk (8192 u32) scanned in place in shared memory: warp w owns
// elements [1024w, 1024w + 1024) as 256 16-B vectors; lane l takes vector
// 32m + l in round m = 0..7 (consecutive lanes, consecutive 16 B: conflict-free
// 128-bit shared loads).  A round scans its 128 elements as four in-thread adds
// plus one 5-step warp scan over the lanes' vector sums, so a chunk costs 8 x 6
// shuffles per warp (a scan per 32 words cost 32 x 6).  The eight vectors stay
// in registers between the warp-total pass and the scan pass; the warps'
// offsets come from their totals.  Returns the chunk total; `carry` is the sum
// of everything before the chunk.
__device__ __forceinline__ uint32_t scan_chunk_smem(uint32_t* c, uint32_t carry, uint32_t* wtot) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint4* mine = reinterpret_cast<uint4*>(c) + warp * 256;
  uint4 q[8];
  uint32_t s = 0;
#pragma unroll
  for (int m = 0; m < 8; ++m) {
    q[m] = mine[32 * m + lane];
    s += q[m].x + q[m].y + q[m].z + q[m].w;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) wtot[warp] = s;
  __syncthreads();
  uint32_t run = carry, total = 0;
  for (int w = 0; w < 8; ++w) {
    const uint32_t t = wtot[w];
    if (w < warp) run += t;
    total += t;
  }
#pragma unroll
  for (int m = 0; m < 8; ++m) {
    const uint32_t a = q[m].x, b = a + q[m].y, d3 = b + q[m].z, d = d3 + q[m].w;
    const uint32_t incl = warp_incl_scan(d);
    const uint32_t e = run + incl - d;                             // sum before this lane's vector
    mine[32 * m + lane] = make_uint4(e + a, e + b, e + d3, e + d);
    run += __shfl_sync(0xffffffffu, incl, 31);
  }
  return total;
}

// Reduce-then-scan over the whole group (unaligned buffers; STRINGS_SCAN_TWOPASS=1
// for every buffer): per-CTA chunk sums -> group barrier -> chunk offsets -> the
// chunk again through the pipeline.  Reads the input twice (12n bytes).
__device__ inline void scan_body_twopass(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t n,
                                         int rank, int S, GroupSync* gs, uint8_t* stage, uint64_t* sbar,
                                         uint32_t* wsum, uint32_t* sphase) {
  // wsum: 16 words outside the stages ([8] warp totals + [8] broadcast / second buffer)
  constexpr uint64_t kTile = (uint64_t)kThreads * kScanPT;
  const uint64_t chunk = ((n + S - 1) / S + kTile - 1) / kTile * kTile;
  const uint64_t b0 = min(n, (uint64_t)rank * chunk), b1 = min(n, b0 + chunk);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const bool vec = ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(y)) & 15) == 0;
  // 1. chunk sum (8 independent 16-B loads in flight per thread)
  uint32_t s = 0;
  uint64_t tail = b0;
  if (vec) {
    const uint4* x4 = reinterpret_cast<const uint4*>(x + b0);
    const uint64_t n4 = (b1 - b0) / 4;
    uint64_t i = threadIdx.x;
    for (; i + 7 * kThreads < n4; i += 8 * kThreads) {
      uint4 q[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) q[u] = ld_stream(x4 + i + u * kThreads);
#pragma unroll
      for (int u = 0; u < 8; ++u) s += q[u].x + q[u].y + q[u].z + q[u].w;
    }
    for (; i < n4; i += kThreads) {
      const uint4 q = ld_stream(x4 + i);
      s += q.x + q.y + q.z + q.w;
    }
    tail = b0 + n4 * 4;
  }
  for (uint64_t e = tail + threadIdx.x; e < b1; e += kThreads) s += x[e];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) wsum[warp] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < 8; ++w) t += wsum[w];
    gs->partial[rank] = t;
  }
  group_barrier(gs, S);
  // 2. offset of this chunk
  if (threadIdx.x == 0) {
    uint32_t off = 0;
    for (int r = 0; r < rank; ++r) off += *reinterpret_cast<volatile uint32_t*>(&gs->partial[r]);
    wsum[8] = off;
  }
  __syncthreads();
  uint32_t carry = wsum[8];
  __syncthreads();
  // 3a. whole 32 KB chunks through the TMA bulk pipeline (as stream_body), each
  //     scanned in shared memory and bulk-stored back
  static_assert(kStreamChunk == kTile * 4, "a scan tile is one pipeline chunk");
  const uint64_t nch = vec ? (b1 - b0) / kTile : 0;
  if (nch) {
    const uint8_t* xb = reinterpret_cast<const uint8_t*>(x + b0);
    uint8_t* yb = reinterpret_cast<uint8_t*>(y + b0);
    const uint32_t ph0 = *reinterpret_cast<volatile uint32_t*>(sphase);   // (stream_body's stage barriers)
    if (threadIdx.x == 0)
      for (int q = 0; q < kStreamLead && (uint64_t)q < nch; ++q) {
        mbar_expect_tx(&sbar[q], kStreamChunk);
        bulk_g2s(stage + q * kStreamChunk, xb + (uint64_t)q * kStreamChunk, kStreamChunk, &sbar[q]);
      }
    for (uint64_t i = 0; i < nch; ++i) {
      const int q = (int)(i % kStreamStages);
      const uint32_t ph = ((ph0 >> q) & 1u) ^ (uint32_t)((i / kStreamStages) & 1);
      if (threadIdx.x == 0 && i + kStreamLead < nch) {
        const int q2 = (int)((i + kStreamLead) % kStreamStages);
        if (i + kStreamLead >= (uint64_t)kStreamStages)
          asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(kStreamStoreSlack) : "memory");
        mbar_expect_tx(&sbar[q2], kStreamChunk);
        bulk_g2s(stage + q2 * kStreamChunk, xb + (i + kStreamLead) * kStreamChunk, kStreamChunk, &sbar[q2]);
      }
      mbar_wait(&sbar[q], ph);
      carry += scan_chunk_smem(reinterpret_cast<uint32_t*>(stage + q * kStreamChunk), carry,
                               wsum + 8 * (int)(i & 1));       // alternate totals: no trailing barrier
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncthreads();
      if (threadIdx.x == 0) bulk_s2g(yb + i * kStreamChunk, stage + q * kStreamChunk, kStreamChunk);
    }
    if (threadIdx.x == 0) {
      *sphase = stage_phases_after(ph0, nch);
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
      asm volatile("fence.proxy.async.global;" ::: "memory");
    }
    __syncthreads();
  }
  // 3b. the rest (unaligned buffers, the ragged last chunk): tiles in registers;
  //     the next tile's 32 elements are loaded while this one is scanned
  const uint64_t r0 = b0 + nch * kTile;
  auto load_tile = [&](uint64_t base, uint32_t* w) {
    const uint64_t e0 = base + (uint64_t)threadIdx.x * kScanPT;
    if (vec && e0 + kScanPT <= b1) {
#pragma unroll
      for (int u = 0; u < kScanPT / 4; ++u) {
        const uint4 q = reinterpret_cast<const uint4*>(x + e0)[u];
        w[4 * u] = q.x; w[4 * u + 1] = q.y; w[4 * u + 2] = q.z; w[4 * u + 3] = q.w;
      }
    } else {
#pragma unroll
      for (int i = 0; i < kScanPT; ++i) w[i] = (e0 + i < b1) ? x[e0 + i] : 0u;
    }
  };
  uint32_t nxt[kScanPT];
  if (r0 < b1) load_tile(r0, nxt);
  for (uint64_t base = r0; base < b1; base += kTile) {
    const uint64_t e0 = base + (uint64_t)threadIdx.x * kScanPT;
    const bool full = vec && e0 + kScanPT <= b1;
    uint32_t v[kScanPT];
#pragma unroll
    for (int i = 0; i < kScanPT; ++i) v[i] = nxt[i];
    if (base + kTile < b1) load_tile(base + kTile, nxt);
    uint32_t run = 0;
#pragma unroll
    for (int i = 0; i < kScanPT; ++i) {
      run += v[i];
      v[i] = run;                                                   // thread-local inclusive
    }
    const uint32_t incl = warp_incl_scan(run);
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    uint32_t wpre = 0, tile = 0;
    for (int w = 0; w < 8; ++w) {
      const uint32_t t = wsum[w];
      if (w < warp) wpre += t;
      tile += t;
    }
    const uint32_t excl = carry + wpre + incl - run;               // sum before this thread's elements
    if (full) {
#pragma unroll
      for (int u = 0; u < kScanPT / 4; ++u)
        reinterpret_cast<uint4*>(y + e0)[u] =
            make_uint4(excl + v[4 * u], excl + v[4 * u + 1], excl + v[4 * u + 2], excl + v[4 * u + 3]);
    } else {
#pragma unroll
      for (int i = 0; i < kScanPT; ++i)
        if (e0 + i < b1) y[e0 + i] = excl + v[i];
    }
    carry += tile;
    __syncthreads();
  }
}

// L2 eviction-priority policies for the cache_hint forms of loads and bulk copies.
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void bulk_g2s_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                              uint64_t pol) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_s2g_hint(void* dst, const void* src, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;"
               :: "l"(dst), "r"(smem_u32(src)), "r"(bytes), "l"(pol) : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}

// Target bytes of one SCAN wave: about three waves of input must stay in L2 (a
// wave's input is read from HBM two waves before it is scanned).  Measured on the
// B200 at 2^28 on 148 CTAs (profiles/r02_scan.md): 16 MB (19 MB waves) reads 1.05x
// the input from DRAM, 22 MB 1.31x; smaller waves add per-wave overhead.
#ifndef STRINGS_SCAN_WAVE_MB
#define STRINGS_SCAN_WAVE_MB 16
#endif

// y = inclusive prefix sum of x (u32, mod 2^32) reading the input from HBM once
// (8n bytes, the algorithmic traffic).  The buffer is cut into waves of S
// sub-blocks (sub-block r of wave k = CTA r's, a whole number of 32 KB chunks,
// about STRINGS_SCAN_WAVE_MB per wave).  CTA r first sums its sub-blocks of
// waves 0 and 1; then for k = 0, 1, ...:
//   lookup(k)  the S tagged words of wave k (published a whole wave earlier, so
//              normally there is no wait): offset = sum of the waves < k + the
//              ranks < r of wave k;
//   scan(k)    its sub-block of wave k, an L2 hit now, through the TMA bulk
//              pipeline: each 32 KB chunk scanned in shared memory and
//              bulk-stored, loads and stores with an evict-first hint (the last
//              use of x; y must not push later waves' x out of L2);
//   sum(k+2)   interleaved with scan(k) chunk by chunk in the same bulk
//              pipeline: one 32 KB chunk of its sub-block of wave k+2 per
//              scanned chunk, summed from shared memory, loaded with the default
//              L2 policy so the lines stay for scan(k+2); published at the end.
// So HBM sees a steady mix of x reads and y writes, and the bulk pipeline runs
// across wave boundaries (a position's load does not depend on any offset).
// No group barrier: the words carry a tag (item epoch, wave index); wave k uses
// row k mod 8, which no CTA can overwrite while another still needs it (a CTA
// writing wave k+2's row has seen every CTA's sum(k), so every CTA is at
// lookup(k-1) or later).  The epoch moves when the item's last CTA finishes.
// Ragged last sub-blocks end in the register tile path.
__device__ inline void scan_regs(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t r0, uint64_t b1,
                                 uint32_t carry, bool vec, uint32_t* wsum) {
  constexpr uint64_t kTile = (uint64_t)kThreads * kScanPT;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  auto load_tile = [&](uint64_t base, uint32_t* w) {
    const uint64_t e0 = base + (uint64_t)threadIdx.x * kScanPT;
    if (vec && e0 + kScanPT <= b1) {
#pragma unroll
      for (int u = 0; u < kScanPT / 4; ++u) {
        const uint4 q = reinterpret_cast<const uint4*>(x + e0)[u];
        w[4 * u] = q.x; w[4 * u + 1] = q.y; w[4 * u + 2] = q.z; w[4 * u + 3] = q.w;
      }
    } else {
#pragma unroll
      for (int i = 0; i < kScanPT; ++i) w[i] = (e0 + i < b1) ? x[e0 + i] : 0u;
    }
  };
  uint32_t nxt[kScanPT];
  if (r0 < b1) load_tile(r0, nxt);
  for (uint64_t base = r0; base < b1; base += kTile) {
    const uint64_t e0 = base + (uint64_t)threadIdx.x * kScanPT;
    const bool full = vec && e0 + kScanPT <= b1;
    uint32_t v[kScanPT];
#pragma unroll
    for (int i = 0; i < kScanPT; ++i) v[i] = nxt[i];
    if (base + kTile < b1) load_tile(base + kTile, nxt);
    uint32_t run = 0;
#pragma unroll
    for (int i = 0; i < kScanPT; ++i) {
      run += v[i];
      v[i] = run;
    }
    const uint32_t incl = warp_incl_scan(run);
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    uint32_t wpre = 0, tile = 0;
    for (int w = 0; w < 8; ++w) {
      const uint32_t t = wsum[w];
      if (w < warp) wpre += t;
      tile += t;
    }
    const uint32_t excl = carry + wpre + incl - run;
    if (full) {
#pragma unroll
      for (int u = 0; u < kScanPT / 4; ++u)
        reinterpret_cast<uint4*>(y + e0)[u] =
            make_uint4(excl + v[4 * u], excl + v[4 * u + 1], excl + v[4 * u + 2], excl + v[4 * u + 3]);
    } else {
#pragma unroll
      for (int i = 0; i < kScanPT; ++i)
        if (e0 + i < b1) y[e0 + i] = excl + v[i];
    }
    carry += tile;
    __syncthreads();
  }
}

__device__ inline void scan_body(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t n, int rank,
                                 int S, GroupSync* gs, uint8_t* stage, uint64_t* sbar, uint32_t* wsum,
                                 uint32_t* sphase) {
  const bool vec = ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(y)) & 15) == 0;
#if defined(STRINGS_SCAN_TWOPASS) && STRINGS_SCAN_TWOPASS
  if (true) {
#else
  if (!vec) {
#endif
    scan_body_twopass(x, y, n, rank, S, gs, stage, sbar, wsum, sphase);
    return;
  }
  // wsum: 32 scratch words: [0, 16) chunk scans (two alternating sets of warp
  // totals), [16, 24) sum / lookup partials, [24, 32) lookup totals
  constexpr uint64_t kTile = (uint64_t)kThreads * kScanPT;       // one 32 KB chunk
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t target = (uint64_t)STRINGS_SCAN_WAVE_MB * (1u << 20) / 4 / (uint64_t)S;
  const uint64_t sb = (target + kTile - 1) / kTile * kTile;        // sub-block elements (>= one chunk)
  const uint64_t W = sb * (uint64_t)S;
  const uint64_t K = (n + W - 1) / W;
  const uint32_t etag = (2u * *reinterpret_cast<volatile uint32_t*>(&gs->scan_epoch) + 1u) << 8;
  const uint64_t pol = l2_policy_evict_first();
  auto lo_of = [&](uint64_t k) { return min(n, k * W + (uint64_t)rank * sb); };
  auto hi_of = [&](uint64_t k) { return min(n, k * W + (uint64_t)(rank + 1) * sb); };
  auto word = [&](uint64_t k, int r) { return &gs->wave[(k % kScanRing) * 256 + r]; };
  // block sum of s, published as wave k's word of this rank
  auto publish = [&](uint64_t k, uint32_t s) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) wsum[16 + warp] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t t = 0;
      for (int w = 0; w < 8; ++w) t += wsum[16 + w];
      st_relaxed_u64(word(k, rank), ((uint64_t)(etag | (uint32_t)(k & 0xFF)) << 32) | t);
    }
    __syncthreads();
  };
  // this thread's share of x[a, b) (a 16-B aligned)
  auto sum_range = [&](uint64_t a, uint64_t b) -> uint32_t {
    uint32_t s = 0;
    if (a >= b) return s;
    const uint4* x4 = reinterpret_cast<const uint4*>(x + a);
    const uint64_t n4 = (b - a) / 4;
    uint64_t i = threadIdx.x;
    for (; i + 7 * kThreads < n4; i += 8 * kThreads) {
      uint4 q[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) q[u] = ld_stream(x4 + i + u * kThreads);
#pragma unroll
      for (int u = 0; u < 8; ++u) s += q[u].x + q[u].y + q[u].z + q[u].w;
    }
    for (; i < n4; i += kThreads) {
      const uint4 q = ld_stream(x4 + i);
      s += q.x + q.y + q.z + q.w;
    }
    for (uint64_t e = a + n4 * 4 + threadIdx.x; e < b; e += kThreads) s += x[e];
    return s;
  };
  for (uint64_t k = 0; k < 2 && k < K; ++k) publish(k, sum_range(lo_of(k), hi_of(k)));
  // One bulk pipeline carries two kinds of 32 KB ops, in this order for every
  // wave k: scan(k, i) for i < nch(k), each followed by sum(k+2, i) while sub-block
  // k+2 has a whole chunk i.  Positions run across waves (no op's load depends on
  // an offset).  A sum op's stage is read by every thread and then reused only
  // after the next op, a scan op, whose __syncthreads orders those reads.
  auto nch_of = [&](uint64_t k) { return k < K ? (hi_of(k) - lo_of(k)) / kTile : 0; };
  const uint32_t ph0 = *reinterpret_cast<volatile uint32_t*>(sphase);   // (stream_body's stage barriers)
  uint64_t pk = 0, pi = 0, issued = 0;                              // thread 0: the next op to load
  bool psum = false;
  auto produce = [&]() {                                            // thread 0: load the next op, if any
    if (pk >= K || pi >= nch_of(pk)) return;
    const int st = (int)(issued % kStreamStages);
    if (issued >= (uint64_t)kStreamStages)                          // the store that last read stage st
      asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(kStreamStoreSlack) : "memory");
    mbar_expect_tx(&sbar[st], kStreamChunk);
    if (!psum) {
      bulk_g2s_hint(stage + st * kStreamChunk, x + lo_of(pk) + pi * kTile, kStreamChunk, &sbar[st], pol);
      psum = pi < nch_of(pk + 2);
    } else {
      bulk_g2s(stage + st * kStreamChunk, x + lo_of(pk + 2) + pi * kTile, kStreamChunk, &sbar[st]);
      psum = false;
    }
    ++issued;
    if (!psum && ++pi >= nch_of(pk)) {
      ++pk;
      pi = 0;
    }
  };
  if (threadIdx.x == 0)
    for (int j = 0; j < kStreamLead; ++j) produce();
  uint32_t base = 0;                                                // sum of the waves before k
  uint64_t pos = 0;                                                 // ops consumed
  uint64_t e = threadIdx.x < S && K ? ld_relaxed_u64(word(0, threadIdx.x)) : 0;
  for (uint64_t k = 0; k < K; ++k) {
    // lookup(k)
    const uint32_t want = etag | (uint32_t)(k & 0xFF);
    if (threadIdx.x < S)
      while ((uint32_t)(e >> 32) != want) {
        __nanosleep(32);
        e = ld_relaxed_u64(word(k, threadIdx.x));
      }
    uint32_t v = threadIdx.x < S ? (uint32_t)e : 0u;
    uint32_t a = threadIdx.x < rank ? v : 0u;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      v += __shfl_xor_sync(0xffffffffu, v, o);
      a += __shfl_xor_sync(0xffffffffu, a, o);
    }
    if (lane == 0) {
      wsum[16 + warp] = a;
      wsum[24 + warp] = v;
    }
    __syncthreads();
    uint32_t pre = 0, tot = 0;
    for (int w = 0; w < 8; ++w) {
      pre += wsum[16 + w];
      tot += wsum[24 + w];
    }
    __syncthreads();
    uint32_t carry = base + pre;
    base += tot;
    // next wave's words: loaded now, checked at the next lookup
    if (k + 1 < K) e = threadIdx.x < S ? ld_relaxed_u64(word(k + 1, threadIdx.x)) : 0;
    const uint64_t lo = lo_of(k), hi = hi_of(k);
    const uint64_t nch = nch_of(k), nfull2 = nch_of(k + 2);
    uint8_t* yb = reinterpret_cast<uint8_t*>(y + lo);
    uint32_t s2 = 0;
    for (uint64_t i = 0; i < nch; ++i) {
      {                                                             // scan(k, i)
        const int st = (int)(pos % kStreamStages);
        const uint32_t ph = ((ph0 >> st) & 1u) ^ (uint32_t)((pos / kStreamStages) & 1);
        if (threadIdx.x == 0) produce();
        mbar_wait(&sbar[st], ph);
        carry += scan_chunk_smem(reinterpret_cast<uint32_t*>(stage + st * kStreamChunk), carry,
                                 wsum + 8 * (int)(pos & 1));
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        if (threadIdx.x == 0) bulk_s2g_hint(yb + i * kStreamChunk, stage + st * kStreamChunk, kStreamChunk, pol);
        ++pos;
      }
      if (i < nfull2) {                                             // sum(k+2, i)
        const int st = (int)(pos % kStreamStages);
        const uint32_t ph = ((ph0 >> st) & 1u) ^ (uint32_t)((pos / kStreamStages) & 1);
        if (threadIdx.x == 0) produce();
        mbar_wait(&sbar[st], ph);
        const uint4* c4 = reinterpret_cast<const uint4*>(stage + st * kStreamChunk);
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const uint4 q = c4[threadIdx.x + u * kThreads];
          s2 += q.x + q.y + q.z + q.w;
        }
        ++pos;
      }
    }
    if (k + 2 < K) {
      const uint64_t lo2 = lo_of(k + 2);
      s2 += sum_range(lo2 + (nch < nfull2 ? nch : nfull2) * kTile, hi_of(k + 2));
      publish(k + 2, s2);
    }
    if (lo + nch * kTile < hi) scan_regs(x, y, lo + nch * kTile, hi, carry, true, wsum);
  }
  if (threadIdx.x == 0) {
    *sphase = stage_phases_after(ph0, pos);
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    asm volatile("fence.proxy.async.global;" ::: "memory");
    __threadfence();
    if (atomicAdd(&gs->scan_done, 1u) == (uint32_t)S - 1) {         // the item's last CTA: next tag
      gs->scan_done = 0;
      atomicAdd(&gs->scan_epoch, 1u);
    }
  }
  __syncthreads();
}

// ------------------------------------------- SORT (Table I: SN, batch sort)
// Each consecutive segment of 2048 u32 keys is sorted ascending by a bitonic
// sorting network (the CUDA SDK "sortingNetworks" workload shape).  Thread t
// keeps keys [8t, 8t + 8) of the segment in registers for the whole network:
// compare-exchange distance j < 8 is inside the thread, 8 <= j < 256 between
// lanes of one warp (shuffles), and only j >= 256 (6 of the 66 stages) goes
// through shared memory (padded one word per 32: conflict-free).
// The body is bound by the integer ALU pipe, so each compare-exchange costs one
// min/max per key.  In merge phase k >= 8 the keys of a descending block (index
// bit k set: bit k - 3 of t, the same for the thread's 8 keys) are held
// complemented; ~ reverses unsigned order, so every compare-exchange of the
// phase is ascending in the held form: in-thread the lower register takes the
// min and the higher the max (no direction select), across lanes or warps the
// lower index takes min(v, p) and the higher max(v, p) (one predicated VIMNMX).
// Between phases one XOR per key moves to the next phase's form; phase 2048
// has no descending block, so the keys end uncomplemented.  Phases 2 and 4
// (k < 8) run on the plain keys with compile-time directions.
constexpr int kSortSeg = 2048;
constexpr int kSortPar = 2;                                       // segments sorted at once per CTA (ILP)
__device__ __forceinline__ int sort_pad(int a) { return a + (a >> 5); }

__device__ inline void sort_body8(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t n, int rank,
                                 int S, uint8_t* stage) {
  static_assert(kSortSeg == 8 * kThreads, "8 keys per thread");
  constexpr int kPadSeg = kSortSeg + kSortSeg / 32;
  uint32_t* key = reinterpret_cast<uint32_t*>(stage);            // [kSortPar][2048 + 64] padded
  const uint64_t nseg = n / kSortSeg;
  const uint32_t t = threadIdx.x;
  const bool vec = ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(y)) & 15) == 0;
  auto load8 = [&](uint64_t seg, uint32_t* w) {
    if (seg >= nseg) return;                                      // idle lane of the pair: garbage, never stored
    const uint32_t* src = x + seg * kSortSeg + 8 * t;
    if (vec) {
      const uint4 q0 = ld_stream(reinterpret_cast<const uint4*>(src));
      const uint4 q1 = ld_stream(reinterpret_cast<const uint4*>(src) + 1);
      w[0] = q0.x; w[1] = q0.y; w[2] = q0.z; w[3] = q0.w;
      w[4] = q1.x; w[5] = q1.y; w[6] = q1.z; w[7] = q1.w;
    } else {
#pragma unroll
      for (int r = 0; r < 8; ++r) w[r] = src[r];
    }
  };
  // segment pairs (rank + 2iS, rank + (2i+1)S)
  uint32_t nxt[kSortPar][8];
#pragma unroll
  for (int h = 0; h < kSortPar; ++h) load8((uint64_t)rank + (uint64_t)h * S, nxt[h]);
  for (uint64_t seg = rank; seg < nseg; seg += (uint64_t)kSortPar * S) {
    uint32_t v[kSortPar][8];
#pragma unroll
    for (int h = 0; h < kSortPar; ++h)
#pragma unroll
      for (int r = 0; r < 8; ++r) v[h][r] = nxt[h][r];
#pragma unroll
    for (int h = 0; h < kSortPar; ++h) load8(seg + (uint64_t)(kSortPar + h) * S, nxt[h]);   // next pair in flight
#pragma unroll
    for (int lk = 1; lk <= 11; ++lk) {
      const int k = 1 << lk;
      if (lk >= 3) {                                               // complement for phase k (held form)
        const uint32_t now = lk < 11 ? (t >> (lk - 3)) & 1u : 0u;  // index bit k
        const uint32_t before = lk > 3 ? (t >> (lk - 4)) & 1u : 0u;
        const uint32_t m = 0u - (now ^ before);
#pragma unroll
        for (int h = 0; h < kSortPar; ++h)
#pragma unroll
          for (int r = 0; r < 8; ++r) v[h][r] ^= m;
      }
#pragma unroll
      for (int lj = lk - 1; lj >= 0; --lj) {
        const int j = 1 << lj;
        if (j >= 256) {                                              // across warps (k >= 512: held form)
          const bool lower = (t & (uint32_t)(j >> 3)) == 0;
#pragma unroll
          for (int h = 0; h < kSortPar; ++h)
#pragma unroll
            for (int r = 0; r < 8; ++r) key[h * kPadSeg + sort_pad(8 * t + r)] = v[h][r];
          __syncthreads();
#pragma unroll
          for (int h = 0; h < kSortPar; ++h)
#pragma unroll
            for (int r = 0; r < 8; ++r) {
              const uint32_t p = key[h * kPadSeg + sort_pad((8 * t + r) ^ j)];
              v[h][r] = lower ? min(v[h][r], p) : max(v[h][r], p);
            }
          __syncthreads();
        } else if (j >= 8) {                                         // lanes t and t ^ (j / 8) (k >= 16: held form)
          const bool lower = (t & (uint32_t)(j >> 3)) == 0;
#pragma unroll
          for (int h = 0; h < kSortPar; ++h)
#pragma unroll
            for (int r = 0; r < 8; ++r) {
              const uint32_t p = __shfl_xor_sync(0xffffffffu, v[h][r], j >> 3);
              v[h][r] = lower ? min(v[h][r], p) : max(v[h][r], p);
            }
        } else {                                                     // registers r and r + j
#pragma unroll
          for (int h = 0; h < kSortPar; ++h)
#pragma unroll
            for (int r = 0; r < 8; ++r) {
              if (r & j) continue;
              // k >= 8: held form, ascending; k < 8: plain keys, direction from r
              const bool asc = k >= 8 || (r & k) == 0;
              const uint32_t lo = v[h][r], hi = v[h][r + j];
              v[h][r] = asc ? min(lo, hi) : max(lo, hi);
              v[h][r + j] = asc ? max(lo, hi) : min(lo, hi);
            }
        }
      }
    }
#pragma unroll
    for (int h = 0; h < kSortPar; ++h) {
      if (seg + (uint64_t)h * S >= nseg) continue;
      uint32_t* dst = y + (seg + (uint64_t)h * S) * kSortSeg + 8 * t;
      if (vec) {
        reinterpret_cast<uint4*>(dst)[0] = make_uint4(v[h][0], v[h][1], v[h][2], v[h][3]);
        reinterpret_cast<uint4*>(dst)[1] = make_uint4(v[h][4], v[h][5], v[h][6], v[h][7]);
      } else {
#pragma unroll
        for (int r = 0; r < 8; ++r) dst[r] = v[h][r];
      }
    }
  }
}

// 32 keys per thread (64 threads = one segment, four segments per CTA at once):
// index a = 32t + r, so 45 of the 66 stages are inside the thread (one VIMNMX
// per key), 20 go across lanes and only j = 1024 through shared memory between
// the group's two warps.  Held-complement form from phase 32 (bit 5 = t bit 0).
constexpr int kSortKPT = 32;
constexpr int kSortTPS = kSortSeg / kSortKPT;                     // 64 threads per segment
constexpr int kSortGroups = kThreads / kSortTPS;                  // 4 segments per CTA

// The network as compile-time stages (template recursion: nvcc does not fully
// unroll the nested loops at 32 keys per thread, and a partly unrolled network
// indexes v[] at run time, i.e. through local memory).
template <int LK, int LJ>
__device__ __forceinline__ void sort32_stage(uint32_t (&v)[kSortKPT], uint32_t t, uint32_t* key) {
  constexpr int k = 1 << LK, j = 1 << LJ;
  if constexpr (j >= 1024) {                                       // the group's two warps
    const bool lower = (t & 32u) == 0;
#pragma unroll
    for (int r = 0; r < kSortKPT; ++r) key[sort_pad(kSortKPT * t + r)] = v[r];
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kSortKPT; ++r) {
      const uint32_t p = key[sort_pad((kSortKPT * t + r) ^ j)];
      v[r] = lower ? min(v[r], p) : max(v[r], p);
    }
    __syncthreads();
  } else if constexpr (j >= kSortKPT) {                            // lanes t and t ^ (j / 32)
    const bool lower = (t & (uint32_t)(j / kSortKPT)) == 0;
#pragma unroll
    for (int r = 0; r < kSortKPT; ++r) {
      const uint32_t p = __shfl_xor_sync(0xffffffffu, v[r], j / kSortKPT);
      v[r] = lower ? min(v[r], p) : max(v[r], p);
    }
  } else {                                                         // registers r and r + j
#pragma unroll
    for (int r = 0; r < kSortKPT; ++r) {
      if (r & j) continue;
      const bool asc = k >= kSortKPT || (r & k) == 0;              // k >= 32: held form
      const uint32_t lo = v[r], hi = v[r + j];
      v[r] = asc ? min(lo, hi) : max(lo, hi);
      v[r + j] = asc ? max(lo, hi) : min(lo, hi);
    }
  }
}
template <int LK, int LJ>
struct Sort32Phase {
  __device__ __forceinline__ static void run(uint32_t (&v)[kSortKPT], uint32_t t, uint32_t* key) {
    sort32_stage<LK, LJ>(v, t, key);
    Sort32Phase<LK, LJ - 1>::run(v, t, key);
  }
};
template <int LK>
struct Sort32Phase<LK, -1> {
  __device__ __forceinline__ static void run(uint32_t (&)[kSortKPT], uint32_t, uint32_t*) {}
};
template <int LK>
struct Sort32Net {
  __device__ __forceinline__ static void run(uint32_t (&v)[kSortKPT], uint32_t t, uint32_t* key) {
    if constexpr (LK >= 5) {                                       // complement for phase 2^LK (held form)
      const uint32_t now = LK < 11 ? (t >> (LK - 5)) & 1u : 0u;    // index bit 2^LK
      const uint32_t before = LK > 5 ? (t >> (LK - 6)) & 1u : 0u;
      const uint32_t m = 0u - (now ^ before);
#pragma unroll
      for (int r = 0; r < kSortKPT; ++r) v[r] ^= m;
    }
    Sort32Phase<LK, LK - 1>::run(v, t, key);
    Sort32Net<LK + 1>::run(v, t, key);
  }
};
template <>
struct Sort32Net<12> {
  __device__ __forceinline__ static void run(uint32_t (&)[kSortKPT], uint32_t, uint32_t*) {}
};

__device__ inline void sort_body32(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t n, int rank,
                                   int S, uint8_t* stage) {
  constexpr int kPadSeg = kSortSeg + kSortSeg / 32;
  const uint32_t t = threadIdx.x % kSortTPS, grp = threadIdx.x / kSortTPS;
  uint32_t* key = reinterpret_cast<uint32_t*>(stage) + grp * kPadSeg;   // this group's padded segment
  const uint64_t nseg = n / kSortSeg;
  const bool vec = ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(y)) & 15) == 0;
  auto load32 = [&](uint64_t seg, uint32_t* w) {
    if (seg >= nseg) return;                                      // idle group: garbage, never stored
    const uint32_t* src = x + seg * kSortSeg + kSortKPT * t;
    if (vec) {
#pragma unroll
      for (int q = 0; q < kSortKPT / 4; ++q) {
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(src) + q);
        w[4 * q] = v.x; w[4 * q + 1] = v.y; w[4 * q + 2] = v.z; w[4 * q + 3] = v.w;
      }
    } else {
#pragma unroll
      for (int r = 0; r < kSortKPT; ++r) w[r] = src[r];
    }
  };
  const uint64_t step = (uint64_t)kSortGroups * S;
  uint32_t nxt[kSortKPT];
  load32((uint64_t)rank + (uint64_t)grp * S, nxt);
  // every group runs the same number of rounds (the smem stage has block barriers)
  for (uint64_t base = rank; base < nseg; base += step) {
    const uint64_t seg = base + (uint64_t)grp * S;
    uint32_t v[kSortKPT];
#pragma unroll
    for (int r = 0; r < kSortKPT; ++r) v[r] = nxt[r];
    load32(seg + step, nxt);                                      // next round in flight
    Sort32Net<1>::run(v, t, key);                                 // the 66 stages, fully expanded
    if (seg < nseg) {
      uint32_t* dst = y + seg * kSortSeg + kSortKPT * t;
      if (vec) {
#pragma unroll
        for (int q = 0; q < kSortKPT / 4; ++q)
          reinterpret_cast<uint4*>(dst)[q] = make_uint4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
      } else {
#pragma unroll
        for (int r = 0; r < kSortKPT; ++r) dst[r] = v[r];
      }
    }
  }
}

#ifndef STRINGS_SORT_KPT
#define STRINGS_SORT_KPT 32
#endif
__device__ __forceinline__ void sort_body(const uint32_t* __restrict__ x, uint32_t* __restrict__ y, uint64_t n,
                                          int rank, int S, uint8_t* stage) {
  if constexpr (STRINGS_SORT_KPT == 32) sort_body32(x, y, n, rank, S, stage);
  else sort_body8(x, y, n, rank, S, stage);
}

// Run one work item on this CTA (rank of S).
// `tmaps` is the item as it sits in global memory (dispatcher mailbox,
// tmap_global = true) or in kernel-parameter space (stand-alone launches).
// rank / S: this CTA's rank and the group's own CTA count (a lent CTA of a
// streaming item has rank >= S); total_word: the dispatcher's word holding the
// item's CTA count with lent ones (nullptr = S).
__device__ __forceinline__ void run_item(const KlItem& it, const KlItem* tmaps, bool tmap_global, int rank, int S,
                                         const GemmSmem& sm, uint32_t tmem_base, uint32_t& mma_phase, GroupSync* gs,
                                         const uint32_t* total_word) {
  switch (it.kclass) {
    case 3:
      hist_body(reinterpret_cast<const uint8_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n, rank, S, gs,
                sm.stage, sm.sbar, sm.sphase);
      break;
    case 4:
      scan_body(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n, rank, S,
                gs, sm.stage, sm.sbar, sm.scratch, sm.sphase);
      break;
    case 5:
      sort_body(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0), it.n, rank, S,
                sm.stage);
      break;
    case 0:
      stream_body<0>(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0),
                     it.n, it.alpha, it.seed, rank, S, sm.stage, sm.sbar, sm.scratch, sm.sphase, gs, total_word);
      break;
    case 2:
      stream_body<2>(reinterpret_cast<const uint32_t*>(it.in0), reinterpret_cast<uint32_t*>(it.out0),
                     it.n, it.alpha, it.seed, rank, S, sm.stage, sm.sbar, sm.scratch, sm.sphase, gs, total_word);
      break;
    case 1:
      gemm_body(tmaps->tmap_a, tmaps->tmap_b, tmaps->tmap_c, tmap_global, reinterpret_cast<float*>(it.out0), it.m,
                it.n, it.k, it.reps, rank, S, sm, tmem_base, mma_phase);
      break;
  }
}

// smem: [A 64 KB][B 128 KB] (or the streaming stages if larger) [tail 256 B: GEMM mbarrier @0, TMEM slot @8,
//        <= 14 stream/fill mbarriers @16.., scratch words @128]
__device__ __forceinline__ GemmSmem carve_smem(uint8_t* base) {
  GemmSmem s;
  s.a = base;
  s.b = base + kSmemA;
  uint8_t* tail = base + kSmemMain;
  s.bar = reinterpret_cast<uint64_t*>(tail);
  s.tmem_slot = reinterpret_cast<uint32_t*>(tail + 8);
  s.stage = base;
  s.sbar = reinterpret_cast<uint64_t*>(tail + 16);
  s.scratch = reinterpret_cast<uint32_t*>(tail + 128);
  s.sphase = reinterpret_cast<uint32_t*>(tail + 12);
  return s;
}

// CTA prologue / epilogue shared by every kernel that may run a GEMM item.
// Every barrier of the smem tail, once per kernel (items track their phases).
__device__ __forceinline__ void mbar_setup(const GemmSmem& sm) {
  if (threadIdx.x == 32) {
    mbar_init(sm.bar, 1);
    for (int b = 0; b < kTailBarriers; ++b) mbar_init(&sm.sbar[b], 1);
    *sm.sphase = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
}
__device__ __forceinline__ uint32_t cta_setup(const GemmSmem& sm) {
  if (threadIdx.x / 32 == 0) tmem_alloc(sm.tmem_slot, kTmemCols);
  mbar_setup(sm);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  return *sm.tmem_slot;
}
__device__ __forceinline__ void cta_teardown(uint32_t tmem_base) {
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (threadIdx.x / 32 == 0) tmem_dealloc(tmem_base, kTmemCols);
}

}  // namespace strings_dev
