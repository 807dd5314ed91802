// Cost of making a pageable host buffer DMA-able: cudaHostRegister/Unregister
// (pin in place) vs a staging memcpy into pinned memory, per buffer size.
//   nvcc -O2 -o tools/register_probe tools/register_probe.cu
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
static double now() { return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count(); }
int main() {
  size_t sizes[] = {256 << 10, 4 << 20, 64 << 20};
  void* pin; cudaHostAlloc(&pin, 64 << 20, 0);
  void* dev; cudaMalloc(&dev, 64 << 20);
  for (size_t s : sizes) {
    const int n = 8;
    std::vector<char*> bufs;
    for (int i = 0; i < n; ++i) { char* p = (char*)malloc(s); memset(p, i, s); bufs.push_back(p); }
    double t0 = now();
    for (auto p : bufs) cudaHostRegister(p, s, cudaHostRegisterDefault);
    double t1 = now();
    for (auto p : bufs) cudaMemcpy(dev, p, s, cudaMemcpyHostToDevice);
    double t2 = now();
    for (auto p : bufs) cudaHostUnregister(p);
    double t3 = now();
    for (auto p : bufs) memcpy(pin, p, s);
    double t4 = now();
    // fresh (never touched) pageable memory: registration also faults pages in
    std::vector<char*> fresh;
    for (int i = 0; i < n; ++i) fresh.push_back((char*)malloc(s));
    double t5 = now();
    for (auto p : fresh) cudaHostRegister(p, s, cudaHostRegisterDefault);
    double t6 = now();
    for (auto p : fresh) cudaHostUnregister(p);
    printf("{\"kib\": %zu, \"register_us\": %.1f, \"unregister_us\": %.1f, \"dma_from_registered_GBps\": %.2f, "
           "\"memcpy_1thread_us\": %.1f, \"memcpy_GBps\": %.2f, \"register_fresh_us\": %.1f, \"err\": \"%s\"}\n",
           s >> 10, (t1 - t0) / n * 1e6, (t3 - t2) / n * 1e6, s * n / (t2 - t1) / 1e9, (t4 - t3) / n * 1e6,
           s * n / (t4 - t3) / 1e9, (t6 - t5) / n * 1e6, cudaGetErrorString(cudaGetLastError()));
    for (auto p : bufs) free(p);
    for (auto p : fresh) free(p);
  }
  return 0;
}
