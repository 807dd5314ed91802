// stream_bench.cu -- R&D microbenchmark for the streaming tenant body (VSCALE).
// Variants: LDG/STG with U loads in flight per thread, and a TMA bulk-copy
// (cp.async.bulk) shared-memory pipeline.  Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o stream_bench tools/stream_bench.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../paper_conf_sc_senguptagsp14_b200/csrc/tenant_kernels.cuh"

using namespace strings_dev;

template <int U>
__global__ void __launch_bounds__(256, 1) ldg_kernel(const uint32_t* x, uint32_t* y, uint64_t n, float a) {
  const uint64_t tid = (uint64_t)blockIdx.x * 256 + threadIdx.x, nt = (uint64_t)gridDim.x * 256;
  const uint4* xv = reinterpret_cast<const uint4*>(x);
  uint4* yv = reinterpret_cast<uint4*>(y);
  uint64_t nvec = n / 4, i = tid;
  for (; i + (U - 1) * nt < nvec; i += U * nt) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ld_stream(xv + i + u * nt);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      v[u].x = elem_op<0>(v[u].x, a, 0); v[u].y = elem_op<0>(v[u].y, a, 0);
      v[u].z = elem_op<0>(v[u].z, a, 0); v[u].w = elem_op<0>(v[u].w, a, 0);
      st_stream(yv + i + u * nt, v[u]);
    }
  }
  for (; i < nvec; i += nt) {
    uint4 v = ld_stream(xv + i);
    v.x = elem_op<0>(v.x, a, 0); v.y = elem_op<0>(v.y, a, 0); v.z = elem_op<0>(v.z, a, 0); v.w = elem_op<0>(v.w, a, 0);
    st_stream(yv + i, v);
  }
}

__device__ __forceinline__ void mbar_expect(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_store(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
               :: "l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(N) : "memory");
}

// TMA bulk pipeline: NS stages of CH bytes; CTA b processes chunks b, b+G, ...
template <int NS, int CH>
__global__ void __launch_bounds__(256, 1) tma_kernel(const uint32_t* x, uint32_t* y, uint64_t n, float a) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + NS * CH);
  const uint64_t nchunks = (n * 4) / CH;            // assume n*4 % CH == 0 for the bench
  if (threadIdx.x == 0) {
    for (int s = 0; s < NS; ++s) mbar_init(&bars[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const uint64_t first = blockIdx.x, step = gridDim.x;
  uint64_t my = first < nchunks ? (nchunks - 1 - first) / step + 1 : 0;   // chunks for this CTA
  // prologue: issue NS-1 loads
  if (threadIdx.x == 0)
    for (int s = 0; s < NS - 1 && (uint64_t)s < my; ++s) {
      mbar_expect(&bars[s], CH);
      bulk_load(smem + s * CH, reinterpret_cast<const uint8_t*>(x) + (first + s * step) * CH, CH, &bars[s]);
    }
  for (uint64_t i = 0; i < my; ++i) {
    const int s = i % NS;
    const uint32_t ph = (i / NS) & 1;
    // issue the load NS-1 ahead into the stage freed by iteration i-1
    if (threadIdx.x == 0 && i + NS - 1 < my) {
      const int s2 = (i + NS - 1) % NS;
      bulk_wait_read<NS - 2>();       // the store that last used stage s2 has read smem
      mbar_expect(&bars[s2], CH);
      bulk_load(smem + s2 * CH, reinterpret_cast<const uint8_t*>(x) + (first + (i + NS - 1) * step) * CH, CH, &bars[s2]);
    }
    mbar_wait(&bars[s], ph);
    uint4* buf = reinterpret_cast<uint4*>(smem + s * CH);
    for (int j = threadIdx.x; j < CH / 16; j += 256) {
      uint4 v = buf[j];
      v.x = elem_op<0>(v.x, a, 0); v.y = elem_op<0>(v.y, a, 0); v.z = elem_op<0>(v.z, a, 0); v.w = elem_op<0>(v.w, a, 0);
      buf[j] = v;
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) bulk_store(reinterpret_cast<uint8_t*>(y) + (first + i * step) * CH, smem + s * CH, CH);
  }
  if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <typename F>
float time_it(F f, int iters = 10) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  f();
  cudaDeviceSynchronize();
  cudaEventRecord(e0);
  for (int i = 0; i < iters; ++i) f();
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  return ms / iters;
}

int main() {
  const uint64_t n = 1ull << 28;
  uint32_t *x, *y;
  cudaMalloc(&x, n * 4);
  cudaMalloc(&y, n * 4);
  cudaMemset(x, 0x3f, n * 4);
  const double bytes = 8.0 * n;
  for (int ctas : {148, 74, 37}) {
    float t;
    t = time_it([&] { ldg_kernel<8><<<ctas, 256>>>(x, y, n, 1.001f); });
    printf("ctas %3d LDG U=8    %7.1f GB/s\n", ctas, bytes / t / 1e6);
    t = time_it([&] { ldg_kernel<16><<<ctas, 256>>>(x, y, n, 1.001f); });
    printf("ctas %3d LDG U=16   %7.1f GB/s\n", ctas, bytes / t / 1e6);
    {
      auto k = tma_kernel<6, 32768>;
      int sm = 6 * 32768 + 64;
      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
      t = time_it([&] { k<<<ctas, 256, sm>>>(x, y, n, 1.001f); });
      printf("ctas %3d TMA 6x32K  %7.1f GB/s  (%s)\n", ctas, bytes / t / 1e6, cudaGetErrorString(cudaGetLastError()));
    }
    {
      auto k = tma_kernel<12, 16384>;
      int sm = 12 * 16384 + 128;
      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
      t = time_it([&] { k<<<ctas, 256, sm>>>(x, y, n, 1.001f); });
      printf("ctas %3d TMA 12x16K %7.1f GB/s  (%s)\n", ctas, bytes / t / 1e6, cudaGetErrorString(cudaGetLastError()));
    }
    {
      auto k = tma_kernel<4, 49152>;
      int sm = 4 * 49152 + 64;
      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
      t = time_it([&] { k<<<ctas, 256, sm>>>(x, y, n, 1.001f); });
      printf("ctas %3d TMA 4x48K  %7.1f GB/s  (%s)\n", ctas, bytes / t / 1e6, cudaGetErrorString(cudaGetLastError()));
    }
  }
  // correctness of the TMA variant
  std::vector<uint32_t> hx(1 << 20), hy(1 << 20);
  for (size_t i = 0; i < hx.size(); ++i) { float f = (float)i * 0.001f; memcpy(&hx[i], &f, 4); }
  cudaMemcpy(x, hx.data(), hx.size() * 4, cudaMemcpyHostToDevice);
  auto k = tma_kernel<6, 32768>;
  k<<<148, 256, 6 * 32768 + 64>>>(x, y, hx.size(), 3.0f);
  cudaMemcpy(hy.data(), y, hy.size() * 4, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (size_t i = 0; i < hx.size(); ++i) { float f; memcpy(&f, &hx[i], 4); float g; memcpy(&g, &hy[i], 4); bad += (g != f * 3.0f); }
  printf("tma correctness: %d mismatches\n", bad);
  return 0;
}
