// PMT staging copy: glibc memcpy vs non-temporal-store copies (SSE2 / AVX2 / AVX-512),
// at the staging pool's chunk size (64 MiB buffer split over T threads), buffers
// pre-touched, a fresh src/dst pair per thread per repetition so nothing is
// cache-resident.  Regular stores read each destination line before writing it
// (read-for-ownership), so a copy moves 3 bytes of DRAM traffic per byte; NT
// stores move 2.  The e2e (pageable) path is host-DRAM bound, so this is its lever.
//   g++ -O2 -pthread -o tools/host_ntcopy_probe tools/host_ntcopy_probe.cpp
#include <immintrin.h>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <vector>

static void nt_copy(void* dst, const void* src, size_t n) {
  char* d = static_cast<char*>(dst);
  const char* s = static_cast<const char*>(src);
  size_t head = (size_t)(-(uintptr_t)d) & 63;
  if (head > n) head = n;
  memcpy(d, s, head);
  d += head; s += head; n -= head;
  for (size_t i = 0, nv = n / 64; i < nv; ++i, d += 64, s += 64) {
    __m128i a = _mm_loadu_si128(reinterpret_cast<const __m128i*>(s));
    __m128i b = _mm_loadu_si128(reinterpret_cast<const __m128i*>(s + 16));
    __m128i c = _mm_loadu_si128(reinterpret_cast<const __m128i*>(s + 32));
    __m128i e = _mm_loadu_si128(reinterpret_cast<const __m128i*>(s + 48));
    _mm_stream_si128(reinterpret_cast<__m128i*>(d), a);
    _mm_stream_si128(reinterpret_cast<__m128i*>(d + 16), b);
    _mm_stream_si128(reinterpret_cast<__m128i*>(d + 32), c);
    _mm_stream_si128(reinterpret_cast<__m128i*>(d + 48), e);
  }
  memcpy(d, s, n & 63);
  _mm_sfence();
}

__attribute__((target("avx2"))) static void nt_copy_avx2(void* dst, const void* src, size_t n) {
  char* d = static_cast<char*>(dst);
  const char* s = static_cast<const char*>(src);
  size_t head = (size_t)(-(uintptr_t)d) & 63;
  if (head > n) head = n;
  memcpy(d, s, head);
  d += head; s += head; n -= head;
  for (size_t i = 0, nv = n / 128; i < nv; ++i, d += 128, s += 128) {
    __m256i a = _mm256_loadu_si256(reinterpret_cast<const __m256i*>(s));
    __m256i b = _mm256_loadu_si256(reinterpret_cast<const __m256i*>(s + 32));
    __m256i c = _mm256_loadu_si256(reinterpret_cast<const __m256i*>(s + 64));
    __m256i e = _mm256_loadu_si256(reinterpret_cast<const __m256i*>(s + 96));
    _mm256_stream_si256(reinterpret_cast<__m256i*>(d), a);
    _mm256_stream_si256(reinterpret_cast<__m256i*>(d + 32), b);
    _mm256_stream_si256(reinterpret_cast<__m256i*>(d + 64), c);
    _mm256_stream_si256(reinterpret_cast<__m256i*>(d + 96), e);
  }
  memcpy(d, s, n & 127);
  _mm_sfence();
}

__attribute__((target("avx512f"))) static void nt_copy_avx512(void* dst, const void* src, size_t n) {
  char* d = static_cast<char*>(dst);
  const char* s = static_cast<const char*>(src);
  size_t head = (size_t)(-(uintptr_t)d) & 63;
  if (head > n) head = n;
  memcpy(d, s, head);
  d += head; s += head; n -= head;
  for (size_t i = 0, nv = n / 256; i < nv; ++i, d += 256, s += 256) {
    __m512i a = _mm512_loadu_si512(s);
    __m512i b = _mm512_loadu_si512(s + 64);
    __m512i c = _mm512_loadu_si512(s + 128);
    __m512i e = _mm512_loadu_si512(s + 192);
    _mm512_stream_si512(reinterpret_cast<__m512i*>(d), a);
    _mm512_stream_si512(reinterpret_cast<__m512i*>(d + 64), b);
    _mm512_stream_si512(reinterpret_cast<__m512i*>(d + 128), c);
    _mm512_stream_si512(reinterpret_cast<__m512i*>(d + 192), e);
  }
  memcpy(d, s, n & 255);
  _mm_sfence();
}

int main() {
  const size_t buf = 64ull << 20;
  const int maxt = (int)std::thread::hardware_concurrency();
  const int nbuf = 8;                                  // rotate 8 x 64 MiB pairs (1 GiB) to defeat the LLC
  std::vector<char*> src(nbuf), dst(nbuf);
  for (int i = 0; i < nbuf; ++i) {
    src[i] = (char*)aligned_alloc(4096, buf); dst[i] = (char*)aligned_alloc(4096, buf);
    memset(src[i], i + 1, buf); memset(dst[i], 0, buf);
  }
  const char* names[4] = {"memcpy", "nt_sse2", "nt_avx2", "nt_avx512"};
  const int nv = __builtin_cpu_supports("avx512f") ? 4 : __builtin_cpu_supports("avx2") ? 3 : 2;
  for (int t : {1, 4, 8, 12, 14, 16}) {
    if (t > maxt) break;
    for (int nt = 0; nt < nv; ++nt) {
      double best = 0;
      for (int r = 0; r < 3; ++r) {
        auto t0 = std::chrono::steady_clock::now();
        for (int b = 0; b < nbuf; ++b) {             // one 64 MiB buffer at a time, split over t threads
          std::vector<std::thread> th;
          const size_t per = ((buf / t) + 63) & ~size_t(63);
          for (int i = 0; i < t; ++i)
            th.emplace_back([&, i, b] {
              size_t off = i * per;
              if (off >= buf) return;
              size_t n = std::min(per, buf - off);
              if (nt == 1) nt_copy(dst[b] + off, src[b] + off, n);
              else if (nt == 2) nt_copy_avx2(dst[b] + off, src[b] + off, n);
              else if (nt == 3) nt_copy_avx512(dst[b] + off, src[b] + off, n);
              else memcpy(dst[b] + off, src[b] + off, n);
            });
          for (auto& x : th) x.join();
        }
        double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        best = std::max(best, (double)nbuf * buf / s / 1e9);
      }
      printf("{\"threads\": %d, \"copy\": \"%s\", \"chunk_MiB\": %.2f, \"GBps\": %.1f}\n", t,
             names[nt], (double)buf / t / (1 << 20), best);
      fflush(stdout);
    }
  }
  for (int b = 0; b < nbuf; ++b) if (memcmp(src[b], dst[b], buf)) { printf("MISMATCH\n"); return 1; }
  return 0;
}
