// gemm_phases.cu -- per-phase timing of the tenant GEMM body (R&D microbenchmark).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/gemm_phases tools/gemm_phases.cu
#include <cstdio>
#include <vector>
#include <algorithm>
#include "../paper_conf_sc_senguptagsp14_b200/csrc/tenant_kernels.cuh"

using namespace strings_dev;

__device__ __forceinline__ uint64_t gt() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Same phases as gemm_body for one tile per CTA, stamped.
__global__ void __launch_bounds__(kThreads, 1) phases(const uint16_t* A, const uint16_t* B, float* C, uint64_t M,
                                                      uint64_t N, uint64_t K, uint32_t R, uint64_t* stamps) {
  extern __shared__ __align__(1024) uint8_t smem[];
  GemmSmem sm = carve_smem(smem);
  uint64_t t0 = gt();
  uint32_t tmem = cta_setup(sm);
  uint64_t t1 = gt();
  const uint64_t tiles_n = N / kTileN;
  const uint64_t tile = blockIdx.x;
  const uint64_t mt = tile / tiles_n, nt = tile % tiles_n;
  gemm_load_tile(sm, A, B, N, K, mt * kTileM, nt * kTileN);
  uint64_t t2 = gt();
  const uint32_t idesc = umma_idesc_bf16(kTileM, kTileN);
  const uint32_t a_base = smem_u32(sm.a), b_base = smem_u32(sm.b);
  if (threadIdx.x == 0) {
    tc_fence_after();
    for (uint32_t v = 0; v < R; ++v)
      for (uint32_t ks = 0; ks < K / 16; ++ks)
        umma_bf16(tmem, umma_desc(a_base + ks * 2 * 2048, 2048, 128), umma_desc(b_base + ks * 2 * 4096, 4096, 128),
                  idesc, ks > 0 ? 1u : 0u);
    umma_commit(sm.bar);
  }
  __syncwarp();
  mbar_wait(sm.bar, 0);
  tc_fence_after();
  uint64_t t3 = gt();
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int lane_base = (warp & 3) * 32, col0 = (warp >> 2) * 128;
  float* crow = C + (mt * kTileM + lane_base + lane) * N + nt * kTileN;
  for (int cc = 0; cc < 128; cc += 32) {
    uint32_t r[32];
    tmem_ld32(tmem + ((uint32_t)lane_base << 16) + (uint32_t)(col0 + cc), r);
    float4* dst = reinterpret_cast<float4*>(crow + col0 + cc);
#pragma unroll
    for (int q = 0; q < 8; ++q)
      dst[q] = make_float4(__uint_as_float(r[4 * q]), __uint_as_float(r[4 * q + 1]), __uint_as_float(r[4 * q + 2]),
                           __uint_as_float(r[4 * q + 3]));
  }
  __syncthreads();
  uint64_t t4 = gt();
  cta_teardown(tmem);
  uint64_t t5 = gt();
  if (threadIdx.x == 0) {
    uint64_t* s = stamps + blockIdx.x * 6;
    s[0] = t0; s[1] = t1; s[2] = t2; s[3] = t3; s[4] = t4; s[5] = t5;
  }
}

int main() {
  const uint64_t M = 128 * 148, N = 256, K = 256;
  uint16_t *A, *B;
  float* C;
  uint64_t* st;
  cudaMalloc(&A, M * K * 2);
  cudaMalloc(&B, K * N * 2);
  cudaMalloc(&C, M * N * 4);
  cudaMalloc(&st, 148 * 6 * 8);
  cudaMemset(A, 0, M * K * 2);
  cudaMemset(B, 0, K * N * 2);
  cudaFuncSetAttribute(phases, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemGemm);
  for (uint32_t R : {1u, 64u}) {
    for (int it = 0; it < 3; ++it) phases<<<148, kThreads, kSmemGemm>>>(A, B, C, M, N, K, R, st);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    phases<<<148, kThreads, kSmemGemm>>>(A, B, C, M, N, K, R, st);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    std::vector<uint64_t> h(148 * 6);
    cudaMemcpy(h.data(), st, h.size() * 8, cudaMemcpyDeviceToHost);
    uint64_t tmin = ~0ull, tmax = 0;
    double ph[5] = {0, 0, 0, 0, 0};
    for (int b = 0; b < 148; ++b) {
      tmin = std::min(tmin, h[b * 6]);
      tmax = std::max(tmax, h[b * 6 + 5]);
      for (int p = 0; p < 5; ++p) ph[p] += (h[b * 6 + p + 1] - h[b * 6 + p]) / 148.0;
    }
    printf("R=%u event %.2f us | CTA span %.2f us | setup %.2f fill %.2f mma %.2f epilogue %.2f teardown %.2f (us, mean)\n",
           R, ms * 1e3, (tmax - tmin) / 1e3, ph[0] / 1e3, ph[1] / 1e3, ph[2] / 1e3, ph[3] / 1e3, ph[4] / 1e3);
    std::vector<uint64_t> starts;
    for (int b = 0; b < 148; ++b) starts.push_back(h[b * 6] - tmin);
    std::sort(starts.begin(), starts.end());
    printf("   CTA start skew: median %.2f us, max %.2f us; %s\n", starts[74] / 1e3, starts[147] / 1e3,
           cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
