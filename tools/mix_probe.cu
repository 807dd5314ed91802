// Mixed-size host-link traffic (C3's shape): does interleaving small copies with
// 4 MiB copies cost the copy engines throughput, and does moving the small
// copies off the copy engines (SM-driven zero-copy, or separate streams) help?
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/mix_probe tools/mix_probe.cu
//   tools/mix_probe [jobs=128]
//
// Per "VSCALE" job: 4 MiB H2D + 4 MiB D2H.  Per "GEMM" job: 2 x 128 KiB H2D
// (A, B) + 256 KiB D2H (C).  jobs of each kind, all copies pre-queued behind a
// spin kernel (device time only), pinned host memory.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

__global__ void sm_copy(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (; i + 3 * stride < n16; i += 4 * stride) {
    uint4 a = src[i], b = src[i + stride], c = src[i + 2 * stride], d = src[i + 3 * stride];
    dst[i] = a; dst[i + stride] = b; dst[i + 2 * stride] = c; dst[i + 3 * stride] = d;
  }
  for (; i < n16; i += stride) dst[i] = src[i];
}

__global__ void spin(long long ns) {
  long long t0; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  long long t = t0;
  while (t - t0 < ns) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
}

// Stand-in for the persistent dispatcher: one CTA per SM, 256 threads, ~196 KB
// of dynamic smem, spinning until the host sets *stop (mapped memory).
__global__ void __launch_bounds__(256, 1) hog(const volatile int* stop) {
  extern __shared__ uint8_t smem[];
  if (threadIdx.x == 0) {
    smem[0] = 1;
    while (*stop == 0) __nanosleep(1000);
  }
  __syncthreads();
}

constexpr size_t kBig = 4u << 20, kSmallIn = 128u << 10, kSmallOut = 256u << 10;

struct Ctx {
  char *hb_in, *hb_out, *hs_in, *hs_out;        // pinned host (mapped)
  char *hs_in_dev, *hs_out_dev;                 // device views of the small host buffers
  char *db_in, *db_out, *ds_in, *ds_out;        // device
  int jobs, variant, ctas;
  cudaStream_t st[4];
  cudaEvent_t part_end[4];
};

// variant: 0 big only (CE) | 1 small only (CE) | 2 mixed, one stream per direction (CE)
//          3 mixed, small on their own streams (CE) | 4 big CE + small SM | 5 small SM only
//          6 mixed one stream per direction, the two 128 KiB inputs as one 256 KiB copy
static void body(Ctx& c) {
  const bool big = c.variant == 0 || c.variant == 2 || c.variant == 3 || c.variant == 4 || c.variant == 6;
  const bool small = c.variant != 0;
  const bool sm = c.variant == 4 || c.variant == 5;
  const int sh = (c.variant == 3 || sm || c.variant == 1 || c.variant == 5) ? 2 : 0;   // small streams
  for (int j = 0; j < c.jobs; ++j) {
    if (big) {
      CK(cudaMemcpyAsync(c.db_in + (size_t)(j % 8) * kBig, c.hb_in + (size_t)(j % 8) * kBig, kBig,
                         cudaMemcpyHostToDevice, c.st[0]));
      CK(cudaMemcpyAsync(c.hb_out + (size_t)(j % 8) * kBig, c.db_out + (size_t)(j % 8) * kBig, kBig,
                         cudaMemcpyDeviceToHost, c.st[1]));
    }
    if (small) {
      const size_t oi = (size_t)(j % 8) * 2 * kSmallIn, oo = (size_t)(j % 8) * kSmallOut;
      if (sm) {
        sm_copy<<<c.ctas, 512, 0, c.st[sh]>>>((const uint4*)(c.hs_in_dev + oi), (uint4*)(c.ds_in + oi),
                                               2 * kSmallIn / 16);
        sm_copy<<<c.ctas, 512, 0, c.st[sh + 1]>>>((const uint4*)(c.ds_out + oo), (uint4*)(c.hs_out_dev + oo),
                                                   kSmallOut / 16);
      } else if (c.variant == 6) {
        CK(cudaMemcpyAsync(c.ds_in + oi, c.hs_in + oi, 2 * kSmallIn, cudaMemcpyHostToDevice, c.st[sh]));
        CK(cudaMemcpyAsync(c.hs_out + oo, c.ds_out + oo, kSmallOut, cudaMemcpyDeviceToHost, c.st[sh + 1]));
      } else {
        CK(cudaMemcpyAsync(c.ds_in + oi, c.hs_in + oi, kSmallIn, cudaMemcpyHostToDevice, c.st[sh]));
        CK(cudaMemcpyAsync(c.ds_in + oi + kSmallIn, c.hs_in + oi + kSmallIn, kSmallIn, cudaMemcpyHostToDevice,
                           c.st[sh]));
        CK(cudaMemcpyAsync(c.hs_out + oo, c.ds_out + oo, kSmallOut, cudaMemcpyDeviceToHost, c.st[sh + 1]));
      }
    }
  }
}

int main(int argc, char** argv) {
  Ctx c{};
  c.jobs = argc > 1 ? atoi(argv[1]) : 128;
  CK(cudaHostAlloc(&c.hb_in, 8 * kBig, cudaHostAllocMapped));
  CK(cudaHostAlloc(&c.hb_out, 8 * kBig, cudaHostAllocMapped));
  CK(cudaHostAlloc(&c.hs_in, 16 * kSmallIn, cudaHostAllocMapped));
  CK(cudaHostAlloc(&c.hs_out, 8 * kSmallOut, cudaHostAllocMapped));
  CK(cudaHostGetDevicePointer((void**)&c.hs_in_dev, c.hs_in, 0));
  CK(cudaHostGetDevicePointer((void**)&c.hs_out_dev, c.hs_out, 0));
  CK(cudaMalloc(&c.db_in, 8 * kBig));
  CK(cudaMalloc(&c.db_out, 8 * kBig));
  CK(cudaMalloc(&c.ds_in, 16 * kSmallIn));
  CK(cudaMalloc(&c.ds_out, 8 * kSmallOut));
  memset(c.hb_in, 1, 8 * kBig);
  memset(c.hs_in, 2, 16 * kSmallIn);
  for (auto& s : c.st) CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  for (auto& ev : c.part_end) CK(cudaEventCreate(&ev));
  cudaEvent_t a;
  CK(cudaEventCreate(&a));
  // Do small SM-copy kernels co-run with a resident dispatcher-shaped kernel
  // that holds every SM (1 CTA/SM, 196 KB smem)?  Launch the hog on its own
  // stream, then run variant 4 beside it.
  int* stop_h = nullptr;
  int* stop_d = nullptr;
  CK(cudaHostAlloc(&stop_h, 64, cudaHostAllocMapped));
  CK(cudaHostGetDevicePointer((void**)&stop_d, stop_h, 0));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const char* names[] = {"big_only_ce", "small_only_ce", "mixed_ce_1stream", "mixed_ce_sep_streams",
                         "big_ce+small_sm", "small_only_sm", "mixed_ce_1stream_merged_inputs",
                         "big_ce+small_sm_beside_resident_hog"};
  const int hog_smem = 196 * 1024;
  CK(cudaFuncSetAttribute(hog, cudaFuncAttributeMaxDynamicSharedMemorySize, hog_smem));
  cudaStream_t hs;
  CK(cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking));
  for (int v = 0; v < 8; ++v) {
    if (v == 7) {
      *(volatile int*)stop_h = 0;
      hog<<<sms, 256, hog_smem, hs>>>(stop_d);
      CK(cudaGetLastError());
      c.variant = 4;
    }
    for (int ctas : {4, 16}) {
      if (ctas != 4 && v != 4 && v != 5 && v != 7) continue;
      c.variant = v == 7 ? 4 : v;
      c.ctas = ctas;
      float best = 1e30f, best_part[4] = {0, 0, 0, 0};
      for (int r = 0; r < 4; ++r) {
        for (auto& st : c.st) CK(cudaStreamSynchronize(st));
        if (v == 7 && cudaStreamQuery(hs) != cudaErrorNotReady) { printf("{\"error\": \"hog not resident\"}\n"); }
        spin<<<1, 1, 0, c.st[0]>>>(60000000LL);
        CK(cudaEventRecord(a, c.st[0]));
        for (int i = 1; i < 4; ++i) CK(cudaStreamWaitEvent(c.st[i], a));
        body(c);
        for (int i = 0; i < 4; ++i) CK(cudaEventRecord(c.part_end[i], c.st[i]));
        for (auto& st : c.st) CK(cudaStreamSynchronize(st));
        float ms = 0, part[4];
        for (int i = 0; i < 4; ++i) {
          CK(cudaEventElapsedTime(&part[i], a, c.part_end[i]));
          ms = part[i] > ms ? part[i] : ms;
        }
        if (r > 0 && ms < best) {
          best = ms;
          for (int i = 0; i < 4; ++i) best_part[i] = part[i];
        }
      }
      const int vv = c.variant;
      const double big_b = (vv == 1 || vv == 5) ? 0 : (double)c.jobs * kBig;
      const double small_b = vv == 0 ? 0 : (double)c.jobs * 2 * kSmallIn;
      printf("{\"variant\": \"%s\", \"jobs\": %d, \"sm_ctas\": %d, \"ms\": %.4f, \"per_dir_GBps\": %.2f, "
             "\"stream_end_ms\": [%.3f, %.3f, %.3f, %.3f]}\n",
             names[v], c.jobs, (vv == 4 || vv == 5) ? ctas : 0, best, (big_b + small_b) / best / 1e6,
             best_part[0], best_part[1], best_part[2], best_part[3]);
      fflush(stdout);
    }
  }
  *(volatile int*)stop_h = 1;
  CK(cudaStreamSynchronize(hs));
  return 0;
}
