// Host memcpy bandwidth vs thread count (pageable -> pageable, 64 MiB per thread,
// buffers pre-touched): the ceiling of the PMT staging path (e2e with pageable buffers).
//   g++ -O2 -pthread -o tools/host_memcpy_probe tools/host_memcpy_probe.cpp
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <vector>
int main() {
  const size_t sz = 64ull << 20;
  const int maxt = (int)std::thread::hardware_concurrency();
  std::vector<char*> src(maxt), dst(maxt);
  for (int i = 0; i < maxt; ++i) {
    src[i] = (char*)malloc(sz); dst[i] = (char*)malloc(sz);
    memset(src[i], i, sz); memset(dst[i], 0, sz);
  }
  for (int t : {1, 2, 4, 6, 8, 12, 16}) {
    if (t > maxt) break;
    double best = 0;
    for (int r = 0; r < 3; ++r) {
      auto t0 = std::chrono::steady_clock::now();
      std::vector<std::thread> th;
      for (int i = 0; i < t; ++i) th.emplace_back([&, i] { for (int k = 0; k < 4; ++k) memcpy(dst[i], src[i], sz); });
      for (auto& x : th) x.join();
      double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
      best = std::max(best, 4.0 * t * sz / s / 1e9);
    }
    printf("{\"threads\": %d, \"memcpy_GBps\": %.1f}\n", t, best);
  }
  return 0;
}
