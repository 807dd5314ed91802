// hist_probe.cu -- stand-alone A/B of byte-histogram counting schemes on one
// B200 (the HIST tenant body, Table I "HI").  Not part of
// the library: each variant is a plain grid of 148 x 256 threads over n bytes,
// timed with CUDA events (median of 20), checked against a host count.
//   V0  per-warp sub-histograms, u32 smem atomics (the round-1/2 body)
//   V1  lane-private u32 counters [bin][lane] shared by the 8 warps, atomics
//   V2  thread-private u16 counters (128 KB), plain ld/add/st per byte
//   V3  thread-private u16 counters, 4 bytes of a word at once: loads first,
//       duplicates inside the word counted so equal bins store the same value
//   V4  as V3 on 8 bytes (two words, 28 compares)
// Inputs: uniform bytes, and the workload's image-like mix (25% from 8 hot bins).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/hist_probe tools/hist_probe.cu
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <random>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

constexpr int kT = 256;

__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// ---- V0
__global__ void __launch_bounds__(kT, 1) hist_v0(const uint8_t* x, uint32_t* bins, uint64_t n) {
  __shared__ uint32_t sh[8 * 256];
  const int warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 8 * 256; i += kT) sh[i] = 0;
  __syncthreads();
  uint32_t* mine = sh + warp * 256;
  const uint64_t tid = (uint64_t)blockIdx.x * kT + threadIdx.x, nt = (uint64_t)gridDim.x * kT;
  const uint64_t nv = n / 16;
  const uint4* x4 = reinterpret_cast<const uint4*>(x);
  for (uint64_t v = tid; v < nv; v += nt) {
    const uint4 q = ld_stream(x4 + v);
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) atomicAdd(&mine[(w[a] >> (8 * b)) & 0xFF], 1u);
  }
  __syncthreads();
  uint32_t total = 0;
  for (int w = 0; w < 8; ++w) total += sh[w * 256 + threadIdx.x];
  if (total) atomicAdd(&bins[threadIdx.x], total);
}

// ---- V1
__global__ void __launch_bounds__(kT, 1) hist_v1(const uint8_t* x, uint32_t* bins, uint64_t n) {
  __shared__ uint32_t sh[256 * 32];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 256 * 32; i += kT) sh[i] = 0;
  __syncthreads();
  uint32_t* mine = sh + lane;
  const uint64_t tid = (uint64_t)blockIdx.x * kT + threadIdx.x, nt = (uint64_t)gridDim.x * kT;
  const uint64_t nv = n / 16;
  const uint4* x4 = reinterpret_cast<const uint4*>(x);
  for (uint64_t v = tid; v < nv; v += nt) {
    const uint4 q = ld_stream(x4 + v);
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) atomicAdd(&mine[((w[a] >> (8 * b)) & 0xFF) * 32], 1u);
  }
  __syncthreads();
  uint32_t total = 0;
  for (int l = 0; l < 32; ++l) total += sh[threadIdx.x * 32 + ((l + threadIdx.x) & 31)];
  if (total) atomicAdd(&bins[threadIdx.x], total);
}

// ---- thread-private u16 counters: bin b of thread t at byte offset b*512 + swz(t)
// swz(t) = ((warp >> 1) * 32 + lane) * 4 + (warp & 1) * 2: a warp's 32 lanes hit 32 banks
extern __shared__ __align__(16) uint8_t dyn[];
__device__ __forceinline__ uint32_t swz() {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  return (uint32_t)(((warp >> 1) * 32 + lane) * 4 + (warp & 1) * 2);
}
__device__ __forceinline__ uint32_t lds16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts16(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u16 [%0], %1;" :: "r"(a), "h"((uint16_t)v) : "memory");
}
// flush: thread t sums bin t over the 256 threads (row t: 512 B, read as 128 words)
__device__ void flush_u16(uint32_t* acc) {
  __syncthreads();
  const uint32_t* row = reinterpret_cast<const uint32_t*>(dyn) + threadIdx.x * 128;
  uint32_t s = 0;
  for (int i = 0; i < 128; ++i) {
    const uint32_t w = row[(i + threadIdx.x) & 127];
    s += (w & 0xFFFF) + (w >> 16);
  }
  *acc += s;
  __syncthreads();
  uint4* z = reinterpret_cast<uint4*>(dyn);
  for (int i = threadIdx.x; i < 256 * 512 / 16; i += kT) z[i] = make_uint4(0, 0, 0, 0);
  __syncthreads();
}

template <int MODE>
__device__ __forceinline__ void count_word(uint32_t base, uint32_t w) {
  if constexpr (MODE == 2) {
#pragma unroll
    for (int b = 0; b < 4; ++b) {
      const uint32_t a = base + ((w >> (8 * b)) & 0xFF) * 512;
      sts16(a, lds16(a) + 1);
    }
  } else {
    const uint32_t b0 = w & 0xFF, b1 = (w >> 8) & 0xFF, b2 = (w >> 16) & 0xFF, b3 = w >> 24;
    const uint32_t a0 = base + b0 * 512, a1 = base + b1 * 512, a2 = base + b2 * 512, a3 = base + b3 * 512;
    const uint32_t l0 = lds16(a0), l1 = lds16(a1), l2 = lds16(a2), l3 = lds16(a3);
    const uint32_t e01 = b0 == b1, e02 = b0 == b2, e03 = b0 == b3, e12 = b1 == b2, e13 = b1 == b3, e23 = b2 == b3;
    sts16(a0, l0 + 1 + e01 + e02 + e03);
    sts16(a1, l1 + 1 + e01 + e12 + e13);
    sts16(a2, l2 + 1 + e02 + e12 + e23);
    sts16(a3, l3 + 1 + e03 + e13 + e23);
  }
}
__device__ __forceinline__ void count_pair(uint32_t base, uint32_t w0, uint32_t w1) {
  uint32_t b[8], a[8], l[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    b[i] = ((i < 4 ? w0 : w1) >> (8 * (i & 3))) & 0xFF;
    a[i] = base + b[i] * 512;
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) l[i] = lds16(a[i]);
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    uint32_t c = 1;
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (j != i) c += b[i] == b[j];
    sts16(a[i], l[i] + c);
  }
}

template <int MODE>
__global__ void __launch_bounds__(kT, 1) hist_priv(const uint8_t* x, uint32_t* bins, uint64_t n) {
  uint4* z = reinterpret_cast<uint4*>(dyn);
  for (int i = threadIdx.x; i < 256 * 512 / 16; i += kT) z[i] = make_uint4(0, 0, 0, 0);
  __syncthreads();
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(dyn) + swz();
  const uint64_t tid = (uint64_t)blockIdx.x * kT + threadIdx.x, nt = (uint64_t)gridDim.x * kT;
  const uint64_t nv = n / 16;
  const uint4* x4 = reinterpret_cast<const uint4*>(x);
  constexpr uint64_t R = 65535 / 16;          // vectors per thread between flushes (u16 counters)
  uint32_t acc = 0;
  for (uint64_t r0 = 0; r0 < nv; r0 += R * nt) {
    const uint64_t r1 = (nv < r0 + R * nt) ? nv : r0 + R * nt;
    uint64_t v = r0 + tid;
    for (; v + nt < r1; v += 2 * nt) {
      const uint4 q = ld_stream(x4 + v), p = ld_stream(x4 + v + nt);
      if constexpr (MODE == 4) {
        count_pair(base, q.x, q.y); count_pair(base, q.z, q.w);
        count_pair(base, p.x, p.y); count_pair(base, p.z, p.w);
      } else {
        count_word<MODE>(base, q.x); count_word<MODE>(base, q.y); count_word<MODE>(base, q.z); count_word<MODE>(base, q.w);
        count_word<MODE>(base, p.x); count_word<MODE>(base, p.y); count_word<MODE>(base, p.z); count_word<MODE>(base, p.w);
      }
    }
    for (; v < r1; v += nt) {
      const uint4 q = ld_stream(x4 + v);
      count_word<3>(base, q.x); count_word<3>(base, q.y); count_word<3>(base, q.z); count_word<3>(base, q.w);
    }
    flush_u16(&acc);
  }
  if (acc) atomicAdd(&bins[threadIdx.x], acc);
}

// ---- V5/V6: V0 / V1 with U independent 16-B loads in flight per thread
template <int U, bool LANE, int COPIES = 1>
__global__ void __launch_bounds__(kT, 1) hist_u(const uint8_t* x, uint32_t* bins, uint64_t n) {
  __shared__ uint32_t s_static[COPIES > 1 ? 1 : 256 * 32];
  uint32_t* sh = COPIES > 1 ? reinterpret_cast<uint32_t*>(dyn) : s_static;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 256 * 32 * COPIES; i += kT) sh[i] = 0;
  __syncthreads();
  uint32_t* mine = LANE ? sh + lane + (warp % COPIES) * 8192 : sh + warp * 256;
  const int stride = LANE ? 32 : 1;
  const uint64_t tid = (uint64_t)blockIdx.x * kT + threadIdx.x, nt = (uint64_t)gridDim.x * kT;
  const uint64_t nv = n / 16;
  const uint4* x4 = reinterpret_cast<const uint4*>(x);
  uint64_t v = tid;
  for (; v + (U - 1) * nt < nv; v += U * nt) {
    uint4 q[U];
#pragma unroll
    for (int u = 0; u < U; ++u) q[u] = ld_stream(x4 + v + u * nt);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t w[4] = {q[u].x, q[u].y, q[u].z, q[u].w};
#pragma unroll
      for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int b = 0; b < 4; ++b) atomicAdd(&mine[((w[a] >> (8 * b)) & 0xFF) * stride], 1u);
    }
  }
  for (; v < nv; v += nt) {
    const uint4 q = ld_stream(x4 + v);
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) atomicAdd(&mine[((w[a] >> (8 * b)) & 0xFF) * stride], 1u);
  }
  __syncthreads();
  uint32_t total = 0;
  if (LANE) for (int c = 0; c < COPIES; ++c) for (int l = 0; l < 32; ++l) total += sh[c * 8192 + threadIdx.x * 32 + ((l + threadIdx.x) & 31)];
  else for (int w = 0; w < 8; ++w) total += sh[w * 256 + threadIdx.x];
  if (total) atomicAdd(&bins[threadIdx.x], total);
}

// ---- V14: TMA bulk pipeline (NS stages of CH bytes) into smem, lane-private atomics from smem
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"((uint32_t)__cvta_generic_to_shared(b)), "r"(c));
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"((uint32_t)__cvta_generic_to_shared(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t ph) {
  const uint32_t a = (uint32_t)__cvta_generic_to_shared(b);
  asm volatile("{\n\t.reg .pred p;\n\tW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W;\n\t}" :: "r"(a), "r"(ph) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"((uint32_t)__cvta_generic_to_shared(dst)), "l"(src), "r"(bytes), "r"((uint32_t)__cvta_generic_to_shared(bar)) : "memory");
}
template <int NS, int CH, int COPIES = 1>
__global__ void __launch_bounds__(kT, 1) hist_bulk(const uint8_t* x, uint32_t* bins, uint64_t n, uint32_t inc = 1u) {
  uint32_t* sh = reinterpret_cast<uint32_t*>(dyn);             // [256][32] counters
  uint8_t* st = dyn + 32768 * COPIES;                          // NS x CH stages
  __shared__ __align__(8) uint64_t bar[NS];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 256 * 32 * COPIES; i += kT) sh[i] = 0;
  if (threadIdx.x == 0) { for (int s = 0; s < NS; ++s) mbar_init(&bar[s], 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  __syncthreads();
  const uint64_t nch = n / CH;                                 // whole chunks (probe: n multiple of CH)
  const uint64_t mine_n = nch > blockIdx.x ? (nch - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  if (threadIdx.x == 0)
    for (int s = 0; s < NS && s < (int)mine_n; ++s) {
      mbar_expect(&bar[s], CH);
      bulk_g2s(st + s * CH, x + (blockIdx.x + (uint64_t)s * gridDim.x) * CH, CH, &bar[s]);
    }
  uint32_t* mine = sh + lane + ((threadIdx.x >> 5) % COPIES) * 8192;
  for (uint64_t i = 0; i < mine_n; ++i) {
    const int s = (int)(i % NS);
    mbar_wait(&bar[s], (uint32_t)((i / NS) & 1));
    const uint4* b4 = reinterpret_cast<const uint4*>(st + s * CH);
#pragma unroll 4
    for (int j = threadIdx.x; j < CH / 16; j += kT) {
      const uint4 q = b4[j];
      const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
      for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int b = 0; b < 4; ++b) atomicAdd(&mine[((w[a] >> (8 * b)) & 0xFF) * 32], inc);
    }
    __syncthreads();
    if (threadIdx.x == 0 && i + NS < mine_n) {
      mbar_expect(&bar[s], CH);
      bulk_g2s(st + s * CH, x + (blockIdx.x + (i + NS) * gridDim.x) * CH, CH, &bar[s]);
    }
  }
  __syncthreads();
  uint32_t total = 0;
  for (int c = 0; c < COPIES; ++c)
    for (int l = 0; l < 32; ++l) total += sh[c * 8192 + threadIdx.x * 32 + ((l + threadIdx.x) & 31)];
  if (total) atomicAdd(&bins[threadIdx.x], total);
}

int main(int argc, char** argv) {
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  const double peak = argc > 1 ? atof(argv[1]) : 6543.7;
  if (argc > 2) nsm = atoi(argv[2]);
  const uint32_t one = argc > 3 ? (uint32_t)atoi(argv[3]) : 1u;
  for (int dist = 0; dist < 2; ++dist)
    for (uint64_t n : {1ull << 26, 1ull << 28}) {
      std::vector<uint8_t> h(n);
      std::mt19937_64 g(7 + dist);
      uint8_t hot[8];
      for (auto& v : hot) v = g() & 0xFF;
      for (uint64_t i = 0; i < n; ++i) {
        const uint64_t r = g();
        h[i] = (dist == 1 && (r & 3) == 0) ? hot[(r >> 2) & 7] : (uint8_t)(r >> 8);
      }
      std::vector<uint32_t> want(256, 0);
      for (auto v : h) want[v]++;
      uint8_t* dx; uint32_t* db;
      CK(cudaMalloc(&dx, n)); CK(cudaMalloc(&db, 1024));
      CK(cudaMemcpy(dx, h.data(), n, cudaMemcpyHostToDevice));
      CK(cudaFuncSetAttribute(hist_priv<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024));
      CK(cudaFuncSetAttribute(hist_priv<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024));
      CK(cudaFuncSetAttribute(hist_priv<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024));
      CK(cudaFuncSetAttribute(hist_bulk<6, 16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
      CK(cudaFuncSetAttribute(hist_bulk<4, 32768>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
      CK(cudaFuncSetAttribute(hist_bulk<8, 16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
      CK(cudaFuncSetAttribute(hist_bulk<4, 32768, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
      CK(cudaFuncSetAttribute(hist_bulk<3, 32768, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
      CK(cudaFuncSetAttribute(hist_bulk<6, 16384, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
      CK(cudaFuncSetAttribute(hist_u<8, true, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072));
      CK(cudaFuncSetAttribute(hist_u<8, true, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536));
      for (int var = 0; var < 21; ++var) {
        auto launch = [&]() {
          switch (var) {
            case 0: hist_v0<<<nsm, kT>>>(dx, db, n); break;
            case 1: hist_v1<<<nsm, kT>>>(dx, db, n); break;
            case 2: hist_priv<2><<<nsm, kT, 128 * 1024>>>(dx, db, n); break;
            case 3: hist_priv<3><<<nsm, kT, 128 * 1024>>>(dx, db, n); break;
            case 4: hist_priv<4><<<nsm, kT, 128 * 1024>>>(dx, db, n); break;
            case 5: hist_u<2, false><<<nsm, kT>>>(dx, db, n); break;
            case 6: hist_u<4, false><<<nsm, kT>>>(dx, db, n); break;
            case 7: hist_u<8, false><<<nsm, kT>>>(dx, db, n); break;
            case 8: hist_u<2, true><<<nsm, kT>>>(dx, db, n); break;
            case 9: hist_u<4, true><<<nsm, kT>>>(dx, db, n); break;
            case 10: hist_u<8, true><<<nsm, kT>>>(dx, db, n); break;
            case 11: hist_u<16, true><<<nsm, kT>>>(dx, db, n); break;
            case 12: hist_u<8, true, 2><<<nsm, kT, 65536>>>(dx, db, n); break;
            case 13: hist_u<8, true, 4><<<nsm, kT, 131072>>>(dx, db, n); break;
            case 14: hist_bulk<6, 16384><<<nsm, kT, 32768 + 6 * 16384>>>(dx, db, n); break;
            case 15: hist_bulk<4, 32768><<<nsm, kT, 32768 + 4 * 32768>>>(dx, db, n); break;
            case 16: hist_bulk<8, 16384><<<nsm, kT, 32768 + 8 * 16384>>>(dx, db, n); break;
            case 17: hist_bulk<4, 32768, 2><<<nsm, kT, 65536 + 4 * 32768>>>(dx, db, n); break;
            case 18: hist_bulk<3, 32768, 2><<<nsm, kT, 65536 + 3 * 32768>>>(dx, db, n); break;
            case 19: hist_bulk<6, 16384, 2><<<nsm, kT, 65536 + 6 * 16384>>>(dx, db, n); break;
            case 20: hist_bulk<4, 32768, 2><<<nsm, kT, 65536 + 4 * 32768>>>(dx, db, n, one); break;
          }
        };
        for (int w = 0; w < 3; ++w) launch();
        CK(cudaMemset(db, 0, 1024));
        launch();
        CK(cudaDeviceSynchronize());
        std::vector<uint32_t> got(256);
        CK(cudaMemcpy(got.data(), db, 1024, cudaMemcpyDeviceToHost));
        const bool ok = got == want;
        cudaEvent_t e0, e1;
        CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
        std::vector<float> ms;
        for (int it = 0; it < 20; ++it) {
          CK(cudaMemsetAsync(db, 0, 1024));
          CK(cudaEventRecord(e0));
          launch();
          CK(cudaEventRecord(e1));
          CK(cudaEventSynchronize(e1));
          float t; CK(cudaEventElapsedTime(&t, e0, e1)); ms.push_back(t);
        }
        std::sort(ms.begin(), ms.end());
        const double t = ms[ms.size() / 2] * 1e-3;
        printf("{\"ctas\": %d, \"variant\": \"V%d\", \"dist\": \"%s\", \"n\": %llu, \"exact\": %s, \"us\": %.2f, \"gbs\": %.1f, \"frac\": %.3f}\n",
               nsm, var, dist ? "image-like" : "uniform", (unsigned long long)n, ok ? "true" : "false", t * 1e6,
               n / t / 1e9, n / t / 1e9 / peak);
      }
      CK(cudaFree(dx)); CK(cudaFree(db));
    }
  return 0;
}
