// Host-link microbenchmark: copy-engine (cudaMemcpyAsync) vs SM-driven copies
// over PCIe, for the copy sizes of the BASELINE configs (128 KiB .. 64 MiB).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/link_bench tools/link_bench.cu -lcuda
//   tools/link_bench [total_mib=256]
//
// For each size s, `total/s` copies are pre-queued (device-timed with events):
//   ce_h2d / ce_d2h : one stream, back to back
//   ce_bidir        : one H2D + one D2H stream concurrently (GB/s both ways summed)
//   ce_h2d_x4       : the copies spread round-robin over 4 streams
//   sm_h2d / sm_d2h : a kernel of `ctas` CTAs streaming 16-B words from / to
//                     mapped pinned host memory (one launch per copy, same stream)
//   sm_bidir        : both SM copies concurrently on two streams
// Prints one JSON line per (size, variant).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

__global__ void sm_copy(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  // 4 independent 16-B loads in flight per thread: PCIe latency is ~1-2 us
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

// The streams are held behind a 50 ms spin kernel while the host enqueues the
// copies, so the timed region is device time only (no host enqueue cost).
static float timed(cudaStream_t* st, cudaEvent_t a, cudaEvent_t b, void (*body)(void*), void* ctx) {
  CK(cudaDeviceSynchronize());
  spin<<<1, 1, 0, st[0]>>>(50000000LL);
  CK(cudaEventRecord(a, st[0]));
  for (int i = 1; i < 4; ++i) CK(cudaStreamWaitEvent(st[i], a));
  body(ctx);
  cudaEvent_t j[4];
  for (int i = 1; i < 4; ++i) {
    CK(cudaEventCreateWithFlags(&j[i], cudaEventDisableTiming));
    CK(cudaEventRecord(j[i], st[i]));
    CK(cudaStreamWaitEvent(st[0], j[i]));
  }
  CK(cudaEventRecord(b, st[0]));
  CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  for (int i = 1; i < 4; ++i) CK(cudaEventDestroy(j[i]));
  return ms;
}

struct Ctx {
  char *h_in, *h_out, *h_in_dev, *h_out_dev;  // pinned host + device views
  char *d_in, *d_out;
  size_t s, total;
  int variant, ctas;
  cudaStream_t st[4];
};

static void body(void* p) {
  Ctx& c = *static_cast<Ctx*>(p);
  size_t k = c.total / c.s;
  for (size_t i = 0; i < k; ++i) {
    size_t off = i * c.s;
    switch (c.variant) {
      case 0: CK(cudaMemcpyAsync(c.d_in + off, c.h_in + off, c.s, cudaMemcpyHostToDevice, c.st[0])); break;
      case 1: CK(cudaMemcpyAsync(c.h_out + off, c.d_out + off, c.s, cudaMemcpyDeviceToHost, c.st[0])); break;
      case 2:
        CK(cudaMemcpyAsync(c.d_in + off, c.h_in + off, c.s, cudaMemcpyHostToDevice, c.st[0]));
        CK(cudaMemcpyAsync(c.h_out + off, c.d_out + off, c.s, cudaMemcpyDeviceToHost, c.st[1]));
        break;
      case 3: CK(cudaMemcpyAsync(c.d_in + off, c.h_in + off, c.s, cudaMemcpyHostToDevice, c.st[i % 4])); break;
      case 4: sm_copy<<<c.ctas, 512, 0, c.st[0]>>>((const uint4*)(c.h_in_dev + off), (uint4*)(c.d_in + off), c.s / 16); break;
      case 5: sm_copy<<<c.ctas, 512, 0, c.st[0]>>>((const uint4*)(c.d_out + off), (uint4*)(c.h_out_dev + off), c.s / 16); break;
      case 6:
        sm_copy<<<c.ctas, 512, 0, c.st[0]>>>((const uint4*)(c.h_in_dev + off), (uint4*)(c.d_in + off), c.s / 16);
        sm_copy<<<c.ctas, 512, 0, c.st[1]>>>((const uint4*)(c.d_out + off), (uint4*)(c.h_out_dev + off), c.s / 16);
        break;
      case 7:  // CE H2D + SM D2H
        CK(cudaMemcpyAsync(c.d_in + off, c.h_in + off, c.s, cudaMemcpyHostToDevice, c.st[0]));
        sm_copy<<<c.ctas, 512, 0, c.st[1]>>>((const uint4*)(c.d_out + off), (uint4*)(c.h_out_dev + off), c.s / 16);
        break;
    }
  }
}

int main(int argc, char** argv) {
  size_t total = (argc > 1 ? atoll(argv[1]) : 256) << 20;
  Ctx c{};
  c.total = total;
  CK(cudaHostAlloc(&c.h_in, total, cudaHostAllocMapped));
  CK(cudaHostAlloc(&c.h_out, total, cudaHostAllocMapped));
  CK(cudaHostGetDevicePointer((void**)&c.h_in_dev, c.h_in, 0));
  CK(cudaHostGetDevicePointer((void**)&c.h_out_dev, c.h_out, 0));
  CK(cudaMalloc(&c.d_in, total));
  CK(cudaMalloc(&c.d_out, total));
  memset(c.h_in, 1, total);
  memset(c.h_out, 2, total);
  CK(cudaMemset(c.d_in, 3, total));
  CK(cudaMemset(c.d_out, 4, total));
  for (auto& s : c.st) CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  int ce = 0;
  CK(cudaDeviceGetAttribute(&ce, cudaDevAttrAsyncEngineCount, 0));
  printf("{\"async_engine_count\": %d, \"total_mib\": %zu}\n", ce, total >> 20);
  const char* names[] = {"ce_h2d", "ce_d2h", "ce_bidir", "ce_h2d_x4", "sm_h2d", "sm_d2h", "sm_bidir", "ce_h2d+sm_d2h"};
  size_t sizes[] = {128 << 10, 256 << 10, 1 << 20, 4 << 20, 16 << 20, 64 << 20};
  int ctas_list[] = {8, 16, 32, 74};
  for (size_t s : sizes) {
    c.s = s;
    for (int v = 0; v < 8; ++v) {
      int nct = v >= 4 ? 4 : 1;
      for (int ci = 0; ci < nct; ++ci) {
        c.variant = v;
        c.ctas = ctas_list[ci];
        float best = 1e30f;
        for (int r = 0; r < 4; ++r) {
          float ms = timed(c.st, a, b, body, &c);
          if (r > 0 && ms < best) best = ms;
        }
        double bytes = (double)total * ((v == 2 || v == 6 || v == 7) ? 2 : 1);
        printf("{\"variant\": \"%s\", \"kib\": %zu, \"ctas\": %d, \"copies\": %zu, \"ms\": %.4f, \"GBps\": %.2f, \"us_per_copy\": %.2f}\n",
               names[v], s >> 10, v >= 4 ? c.ctas : 0, total / s, best, bytes / best / 1e6,
               best * 1e3 / (total / s));
        fflush(stdout);
      }
    }
  }
  return 0;
}
