// fill_bench.cu -- smem fill variants for the GEMM tile (R&D).
#include <cstdio>
#include <vector>
#include <algorithm>
#include "../paper_conf_sc_senguptagsp14_b200/csrc/tenant_kernels.cuh"
using namespace strings_dev;
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }

template <int MODE>  // 0 cp.async A+B, 1 A only, 2 B only, 3 LDG/STS batched A+B, 4 cp.async A+B no-division indexing
__global__ void __launch_bounds__(256, 1) fill(const uint16_t* A, const uint16_t* B, uint64_t N, uint64_t K, uint64_t* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  GemmSmem sm = carve_smem(smem);
  __syncthreads();
  uint64_t t0 = gt();
  const uint64_t m0 = blockIdx.x * 128;
  auto cp16 = [](uint8_t* dst, const void* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(smem_u32(dst)), "l"(src) : "memory");
  };
  const int kchunks = (int)(K / 8);
  if (MODE == 0 || MODE == 1 || MODE == 2) {
    if (MODE != 2)
      for (int idx = threadIdx.x; idx < 128 * kchunks; idx += 256) {
        const int rr = idx & 7, c = (idx >> 3) % kchunks, g = (idx >> 3) / kchunks;
        cp16(sm.a + ((c * 16 + g) * 128 + rr * 16), A + (m0 + g * 8 + rr) * K + (uint64_t)c * 8);
      }
    if (MODE != 1)
      for (int idx = threadIdx.x; idx < (int)K * 32; idx += 256) {
        const int kk = idx & 7, q = (idx >> 3) & 31, c = idx >> 8;
        cp16(sm.b + ((c * 32 + q) * 128 + kk * 16), B + (uint64_t)(c * 8 + kk) * N + (uint64_t)q * 8);
      }
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
  } else if (MODE == 4) {
    // K = 256 fixed: kchunks = 32 -> shifts instead of divisions
    for (int idx = threadIdx.x; idx < 128 * 32; idx += 256) {
      const int rr = idx & 7, c = (idx >> 3) & 31, g = idx >> 8;
      cp16(sm.a + ((c * 16 + g) * 128 + rr * 16), A + (m0 + g * 8 + rr) * K + (uint64_t)c * 8);
    }
    for (int idx = threadIdx.x; idx < 256 * 32; idx += 256) {
      const int kk = idx & 7, q = (idx >> 3) & 31, c = idx >> 8;
      cp16(sm.b + ((c * 32 + q) * 128 + kk * 16), B + (uint64_t)(c * 8 + kk) * N + (uint64_t)q * 8);
    }
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
  } else {
    for (int base = 0; base < 128 * kchunks; base += 256 * 8) {
      uint4 v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int idx = base + u * 256 + threadIdx.x;
        const int rr = idx & 7, c = (idx >> 3) % kchunks, g = (idx >> 3) / kchunks;
        v[u] = *reinterpret_cast<const uint4*>(A + (m0 + g * 8 + rr) * K + (uint64_t)c * 8);
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int idx = base + u * 256 + threadIdx.x;
        const int rr = idx & 7, c = (idx >> 3) % kchunks, g = (idx >> 3) / kchunks;
        *reinterpret_cast<uint4*>(sm.a + ((c * 16 + g) * 128 + rr * 16)) = v[u];
      }
    }
    for (int base = 0; base < (int)K * 32; base += 256 * 8) {
      uint4 v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int idx = base + u * 256 + threadIdx.x;
        const int kk = idx & 7, q = (idx >> 3) & 31, c = idx >> 8;
        v[u] = *reinterpret_cast<const uint4*>(B + (uint64_t)(c * 8 + kk) * N + (uint64_t)q * 8);
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int idx = base + u * 256 + threadIdx.x;
        const int kk = idx & 7, q = (idx >> 3) & 31, c = idx >> 8;
        *reinterpret_cast<uint4*>(sm.b + ((c * 32 + q) * 128 + kk * 16)) = v[u];
      }
    }
  }
  __syncthreads();
  uint64_t t1 = gt();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}

template <int MODE>
void run(const char* name, const uint16_t* A, const uint16_t* B, uint64_t* out) {
  auto k = fill<MODE>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemGemm);
  for (int i = 0; i < 3; ++i) k<<<148, 256, kSmemGemm>>>(A, B, 256, 256, out);
  cudaDeviceSynchronize();
  std::vector<uint64_t> h(148);
  cudaMemcpy(h.data(), out, 148 * 8, cudaMemcpyDeviceToHost);
  std::sort(h.begin(), h.end());
  printf("%-28s median %.2f us  max %.2f us  (%s)\n", name, h[74] / 1e3, h[147] / 1e3, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  uint16_t *A, *B;
  uint64_t* out;
  cudaMalloc(&A, 128 * 148 * 256 * 2);
  cudaMalloc(&B, 256 * 256 * 2);
  cudaMalloc(&out, 148 * 8);
  run<0>("cp.async A+B", A, B, out);
  run<1>("cp.async A only", A, B, out);
  run<2>("cp.async B only", A, B, out);
  run<3>("LDG/STS x8 A+B", A, B, out);
  run<4>("cp.async A+B, shifts", A, B, out);
  return 0;
}
