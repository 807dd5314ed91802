/* Plain C versions of the oracle's tenant kernels (oracle/kernels.py), and a
 * thread-pool runner for bench.py's cpu_baseline leg.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle/__init__.py): only tests/, smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code with the CUDA path.  Each kernel is the closed-form result of
 * SURVEY.md §8(c) "Plain CPU kernels", written out directly, no blocking:
 *
 *   VSCALE  y[i] = a * x[i], one IEEE fp32 multiply (compiled with
 *           -ffp-contract=off, no -ffast-math: reading R-23)
 *   GEMM    C = A.B, bf16 operands widened to double, products summed in
 *           double for k = 0..K-1, rounded once to float (R-22); the KL phase
 *           repeats the product R times (R-17): every repetition is computed
 *   XFER    y[i] = fmix32(x[i] ^ seed) (MurmurHash3 finaliser)
 *   HIST    bins[b] = #{i : x[i] == b}, 256 u32 bins
 *   SCAN    y[i] = x[0] + ... + x[i] mod 2^32
 *   SORT    every 2048-key segment sorted ascending
 *
 * Pinned against oracle/kernels.py (and through it against the published
 * vectors / closed forms) by tests/test_oracle_c.py.
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static double bf16_to_double(uint16_t b) {
  uint32_t u = (uint32_t)b << 16;
  float f;
  memcpy(&f, &u, sizeof f);
  return (double)f;
}

void oc_vscale(const float* x, float* y, uint64_t n, float a) {
  for (uint64_t i = 0; i < n; ++i) y[i] = a * x[i];
}

/* A: m x k bf16 row-major, B: k x n bf16 row-major, C: m x n float. */
void oc_gemm(const uint16_t* A, const uint16_t* B, float* C, uint64_t m, uint64_t n, uint64_t k, uint32_t reps) {
  for (uint32_t r = 0; r < (reps ? reps : 1); ++r)
    for (uint64_t i = 0; i < m; ++i)
      for (uint64_t j = 0; j < n; ++j) {
        double s = 0.0;
        for (uint64_t q = 0; q < k; ++q) s += bf16_to_double(A[i * k + q]) * bf16_to_double(B[q * n + j]);
        C[i * n + j] = (float)s;
      }
}

static uint32_t fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6Bu;
  h ^= h >> 13;
  h *= 0xC2B2AE35u;
  h ^= h >> 16;
  return h;
}

void oc_xfer(const uint32_t* x, uint32_t* y, uint64_t n, uint32_t seed) {
  for (uint64_t i = 0; i < n; ++i) y[i] = fmix32(x[i] ^ seed);
}

void oc_hist(const uint8_t* x, uint32_t* bins, uint64_t n) {
  memset(bins, 0, 256 * sizeof(uint32_t));
  for (uint64_t i = 0; i < n; ++i) bins[x[i]] += 1;
}

void oc_scan(const uint32_t* x, uint32_t* y, uint64_t n) {
  uint32_t s = 0;
  for (uint64_t i = 0; i < n; ++i) {
    s += x[i];
    y[i] = s;
  }
}

static int cmp_u32(const void* a, const void* b) {
  const uint32_t x = *(const uint32_t*)a, z = *(const uint32_t*)b;
  return (x > z) - (x < z);
}

void oc_sort_segments(const uint32_t* x, uint32_t* y, uint64_t n, uint64_t seg) {
  memcpy(y, x, n * sizeof(uint32_t));
  for (uint64_t s = 0; s + seg <= n; s += seg) qsort(y + s, seg, sizeof(uint32_t), cmp_u32);
}

/* ---------------------------------------------------------------- runner --
 * One job = copy the H2D buffers into "device" memory (a host allocation),
 * run the kernel, copy the output back to the caller's D2H buffer: the same
 * bytes the GPU path moves.  Jobs are given in submission order; job j may
 * start only after every earlier job of its tenant finished (c_t = 1).
 * Workers claim whole tenants from a shared counter (a tenant's jobs run in
 * order on its worker), so long and short tenants balance over the pool. */
typedef struct {
  uint32_t kclass, reps, tenant, seed;
  uint64_t n, m, k;
  float alpha;
  const void* in0;
  const void* in1;
  void* out0;
} oc_job_t;

static uint64_t in_bytes(const oc_job_t* j, int which) {
  switch (j->kclass) {
    case 0: case 2: case 4: case 5: return which == 0 ? 4 * j->n : 0;
    case 1: return which == 0 ? 2 * j->m * j->k : 2 * j->k * j->n;
    case 3: return which == 0 ? j->n : 0;
  }
  return 0;
}
static uint64_t out_bytes(const oc_job_t* j) {
  switch (j->kclass) {
    case 0: case 2: case 4: case 5: return 4 * j->n;
    case 1: return 4 * j->m * j->n;
    case 3: return 1024;
  }
  return 0;
}

static void run_one(const oc_job_t* j) {
  void* d0 = malloc(in_bytes(j, 0) ? in_bytes(j, 0) : 1);
  void* d1 = malloc(in_bytes(j, 1) ? in_bytes(j, 1) : 1);
  void* dout = malloc(out_bytes(j) ? out_bytes(j) : 1);
  if (in_bytes(j, 0)) memcpy(d0, j->in0, in_bytes(j, 0));
  if (in_bytes(j, 1)) memcpy(d1, j->in1, in_bytes(j, 1));
  switch (j->kclass) {
    case 0: oc_vscale((const float*)d0, (float*)dout, j->n, j->alpha); break;
    case 1: oc_gemm((const uint16_t*)d0, (const uint16_t*)d1, (float*)dout, j->m, j->n, j->k, j->reps); break;
    case 2: oc_xfer((const uint32_t*)d0, (uint32_t*)dout, j->n, j->seed); break;
    case 3: oc_hist((const uint8_t*)d0, (uint32_t*)dout, j->n); break;
    case 4: oc_scan((const uint32_t*)d0, (uint32_t*)dout, j->n); break;
    case 5: oc_sort_segments((const uint32_t*)d0, (uint32_t*)dout, j->n, 2048); break;
  }
  if (out_bytes(j)) memcpy(j->out0, dout, out_bytes(j));
  free(d0);
  free(d1);
  free(dout);
}

typedef struct {
  const oc_job_t* jobs;
  uint64_t njobs;
  const uint32_t* tenants;   /* distinct tenant ids, in claim order */
  uint32_t ntenants;
  uint32_t* next;            /* shared claim counter */
} oc_pool_t;

static void* worker_main(void* arg) {
  oc_pool_t* p = (oc_pool_t*)arg;
  for (;;) {
    const uint32_t c = __atomic_fetch_add(p->next, 1u, __ATOMIC_RELAXED);
    if (c >= p->ntenants) return NULL;
    for (uint64_t i = 0; i < p->njobs; ++i)
      if (p->jobs[i].tenant == p->tenants[c]) run_one(&p->jobs[i]);
  }
}

/* Runs every job on `threads` workers; returns 0 (the caller times it). */
int oc_run_jobs(const oc_job_t* jobs, uint64_t njobs, uint32_t threads) {
  if (threads == 0) threads = 1;
  /* tenants in order of their total kernel work, largest first (longest-first
     claiming keeps the pool balanced) */
  uint32_t* ten = (uint32_t*)malloc(sizeof(uint32_t) * (njobs ? njobs : 1));
  double* work = (double*)calloc(njobs ? njobs : 1, sizeof(double));
  uint32_t nt = 0;
  for (uint64_t i = 0; i < njobs; ++i) {
    uint32_t t = 0;
    while (t < nt && ten[t] != jobs[i].tenant) ++t;
    if (t == nt) ten[nt++] = jobs[i].tenant;
    const oc_job_t* j = &jobs[i];
    work[t] += j->kclass == 1 ? (double)j->m * j->n * j->k * (j->reps ? j->reps : 1) : (double)(in_bytes(j, 0) + out_bytes(j));
  }
  for (uint32_t a = 1; a < nt; ++a)            /* insertion sort by work, descending */
    for (uint32_t b = a; b > 0 && work[b] > work[b - 1]; --b) {
      double w = work[b]; work[b] = work[b - 1]; work[b - 1] = w;
      uint32_t x = ten[b]; ten[b] = ten[b - 1]; ten[b - 1] = x;
    }
  uint32_t next = 0;
  oc_pool_t pool = {jobs, njobs, ten, nt, &next};
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * threads);
  for (uint32_t t = 0; t < threads; ++t) pthread_create(&th[t], NULL, worker_main, &pool);
  for (uint32_t t = 0; t < threads; ++t) pthread_join(th[t], NULL);
  free(th);
  free(ten);
  free(work);
  return 0;
}

uint64_t oc_job_struct_size(void) { return sizeof(oc_job_t); }
