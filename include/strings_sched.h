/*
 * strings_sched.h -- C ABI of the B200-native Strings scheduler hot path.
 *
 * Method: Sengupta, Goswami, Schwan, Pallavi, "Scheduling Multi-tenant Cloud
 * Workloads on Accelerator-based Systems", SC14.  Citations "P:L<n>" refer to
 * lines of the paper text; "R-n" to the readings in DESIGN.md §6;
 * "§4.x" to the scheduler semantics in DESIGN.md §4.
 *
 * The library owns device selection (the runtime overrides the
 * application's cudaSetDevice), merges all tenants of a GPU into one context
 * (P:L179-185), and co-schedules tenants' H2D / kernel / D2H phases on
 * the copy engines and on SM partitions of a persistent kernel.
 *
 * Conventions
 *  - Every call returns a strings_status_t (0 = STRINGS_OK, negative = error);
 *    no call aborts the process.  The last CUDA error seen by the library is
 *    kept per process (strings_last_cuda_error).
 *  - All calls are thread-safe.  Tenants are typically distinct host threads.
 *  - Host buffers are owned by the caller.  Device memory is owned by the
 *    library (per-GPU arena of resident job slots).
 *  - Times are ns on the library clock: CLOCK_MONOTONIC since strings_init in
 *    MEASURED mode, the virtual clock in INJECTED / DECISIONS_ONLY mode.
 *
 * Environment knobs (read at strings_init; none changes a decision, only how
 * the decided ops execute; DESIGN.md §2 and §11 give the measurements):
 *   STRINGS_COPY_CTAS=n      SMs of the persistent kernel serving small H2D/D2H
 *                            ops as zero-copy SM copies (default 4; 0 = every
 *                            copy on the copy engines)
 *   STRINGS_SM_COPY_MAX=b    largest op (bytes, all buffers) sent to those SMs
 *                            (default 1 MiB); host buffers must be mapped pinned
 *                            memory, 16-B aligned, sizes multiples of 16
 *   STRINGS_SM_COPY_WHEN=always  send every eligible op there (default: only
 *                            while that direction's copy engine has queued work)
 *   STRINGS_ITEM_VIA_COPY=1  also send KL work items of copy-engine jobs there
 *   STRINGS_COPY_STREAMS=physical  one H2D and one D2H stream per GPU instead of
 *                            per logical device
 *   STRINGS_COPY_THREADS=n   host threads of the pageable-buffer staging pool
 *   STRINGS_NT_COPY=0|1|2|3  staging copy loop: memcpy | SSE2 (default) | AVX2 |
 *                            AVX-512 non-temporal stores
 *   STRINGS_KL_HELP=0        an idle KL slot does not lend its SMs to its sibling
 *                            slot's VSCALE/XFER item (default: it does)
 *   STRINGS_SM_LIMIT=n       run the persistent kernel on n SMs (tests)
 *   STRINGS_POLL_MAX_NS=ns   idle-poll back-off cap of partition leaders (1024)
 *   STRINGS_STALL_DUMP_S=s   print in-flight ops to stderr if none completes
 *                            for s seconds (default 20)
 *   STRINGS_FAULT_JOB=id     inject a device fault in that job's KL (tests)
 */
#ifndef STRINGS_SCHED_H
#define STRINGS_SCHED_H

#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t strings_status_t;
typedef uint32_t strings_tenant_t;
typedef uint64_t strings_job_t;

#define STRINGS_OK       0
#define STRINGS_EINVAL  (-1)  /* bad argument (sizes, class, unknown tenant/job)          */
#define STRINGS_ENOMEM  (-2)  /* host or device allocation failed                          */
#define STRINGS_EAGAIN  (-3)  /* not ready / try again                                      */
#define STRINGS_ECUDA   (-4)  /* CUDA error; see strings_last_cuda_error()                  */
#define STRINGS_ESTATE  (-5)  /* not initialised, already initialised, or shutting down     */
#define STRINGS_EFAULT  (-6)  /* a job of this tenant failed (fault localisation)   */

/* Workload-balancing policies (balancer = level 1). */
#define STRINGS_BAL_GRR      0  /* Global Round Robin                                  */
#define STRINGS_BAL_GMIN     1  /* fewest bound jobs, ties -> lowest GID            */
#define STRINGS_BAL_GWTMIN   2  /* load / device weight                                 */
#define STRINGS_BAL_RTF      3  /* runtime feedback                                 */
#define STRINGS_BAL_GUF      4  /* GPU-utilisation feedback                             */
#define STRINGS_BAL_DTF      5  /* data-transfer feedback                               */
#define STRINGS_BAL_MBF      6  /* memory-bandwidth feedback                            */
#define STRINGS_BAL_DYNAMIC  7  /* policy arbiter: GMin until feedback, then MBF, P:L311 (R-15) */

/* Device-level dispatch policies (level 2). */
#define STRINGS_DEV_FIFO 0      /* wake in placement order (baseline)                          */
#define STRINGS_DEV_LAS  1      /* least attained service, weighted, phase-blind (R-7) */
#define STRINGS_DEV_PS   2      /* Phase Selection: one per phase, else KL > H2D = D2H */
#define STRINGS_DEV_TFS  3      /* True Fair-Share: one tenant awake, weight-proportional slices,
                                   service-history penalty, work conserving    */

/* Tenant kernel classes (the paper's workload classes, Table I). */
#define STRINGS_VSCALE 0        /* y = alpha * x, fp32, n elements          (memory-bound)      */
#define STRINGS_GEMM   1        /* C = A.B, bf16 in / fp32 out, R repetitions (compute-bound)   */
#define STRINGS_XFER   2        /* y = fmix32(x ^ seed), u32, n elements    (transfer-heavy)    */
#define STRINGS_HIST   3        /* bins[256] u32 = byte histogram of x[n] u8 (Table I: HI)      */
#define STRINGS_SCAN   4        /* y = inclusive prefix sum of x[n] u32, mod 2^32 (Table I: SC) */
#define STRINGS_SORT   5        /* each 2048-key segment of x[n] u32 sorted ascending (SN)      */

/* Timing modes. */
#define STRINGS_TIMING_MEASURED        0  /* real clock, real completions                       */
#define STRINGS_TIMING_INJECTED        1  /* virtual clock from descriptor durations; every
                                             op still runs on the GPU; decisions bit-exact     */
#define STRINGS_TIMING_DECISIONS_ONLY  2  /* test-only: decision core without device work;
                                             D2H buffers are NOT written                        */

typedef struct {
    int32_t  num_gpus;       /* G logical devices; 0 = number of physical GPUs used             */
    int32_t  physical_gpus;  /* physical GPUs to use (first N visible); 0 = all visible         */
    int32_t  balancer;       /* STRINGS_BAL_*                                                   */
    int32_t  las_admission;  /* 1 = admit pending jobs in weighted-LAS order (R-9)              */
    int32_t  device_policy;  /* STRINGS_DEV_* (FIFO, LAS, PS, TFS)                              */
    int32_t  partitions;     /* P KL slots (SM partitions) per device; 0 -> 2                   */
    int32_t  awake_budget;   /* A woken-unfinished ops per device; 0 -> 2 + P (R-11)            */
    int32_t  admit_cap;      /* M resident jobs per device; 0 -> 2 * A (R-12)                   */
    int32_t  joint_select;   /* -1 auto (on for DTF/MBF/DYNAMIC), 0 off, 1 on (R-16)            */
    int32_t  timing_mode;    /* STRINGS_TIMING_*                                                */
    uint64_t quantum_ns;     /* LAS epoch Q; 0 -> 1,000,000 (R-5)                               */
    uint64_t slot_bytes;     /* device bytes per resident job slot; 0 -> 160 MiB                */
    const char* trace_path;  /* if non-NULL the decision trace is written there at drain/shutdown (string copied at init) */
    int32_t  trace_in_memory;/* 1 = keep the trace for strings_trace_copy; with trace_path NULL
                                and trace_in_memory 0 no record is formatted (counters only)    */
    int32_t  kl_mode;        /* 0 = persistent dispatcher kernel (product); 1 = per-job launches of
                                the same bodies on per-slot streams (profilers that replay kernels).
                                0 becomes 1 when a kernel profiler is injected (Nsight Compute's
                                NV_COMPUTE_PROFILER_* / NSIGHT_COMPUTE_* variables or LD_PRELOAD
                                interceptor, or CUDA_INJECTION64_PATH) unless STRINGS_KL_MODE_FORCE=1; the effective
                                mode is reported in strings_stats_t::kl_mode                       */
    int32_t  reserved[6];
    uint64_t tfs_slice_ns;   /* TFS base slice S: a tenant of weight w is awake for w*S; 0 -> 500 us */
    const uint32_t* device_weights; /* num_gpus DST weights >= 1 (GWtMin); NULL = all 1.
                                       Logical devices sharing a physical GPU get SM partitions
                                       in proportion to their weights (heterogeneous pool).     */
    void* const* ext_arenas;        /* optional, per physical GPU used: caller-owned device memory
                                       (e.g. a torch allocation) for the resident-job slots; must
                                       hold (logical devices on that GPU) x admit_cap x slot_bytes
                                       and stay valid until strings_shutdown.  NULL = cudaMalloc.  */
    const uint64_t* ext_arena_bytes;/* sizes of ext_arenas[i]                                      */
    void* const* ext_streams;       /* optional: 2 * num_gpus caller-owned cudaStream_t handles (e.g.
                                       torch.cuda.Stream().cuda_stream), [2g] = H2D and [2g+1] = D2H
                                       copy stream of logical device g (the paper's per-app stream,
                                       P:L315; the copy engines' FIFOs of DESIGN §2).  Each must be a
                                       non-blocking stream of the physical GPU that hosts g, distinct
                                       from every other entry, stay valid until strings_shutdown and
                                       carry no other work meanwhile; the library never destroys it.
                                       An entry may be NULL (the library creates that stream).  Bad
                                       handles -> STRINGS_EINVAL.  NULL = all library streams.     */
} strings_config_t;

/* Kernel descriptor: which tenant kernel the KL phase runs, and its sizes.
 * Fixed kernel table, no user function pointers.  H2D / D2H buffer layout:
 *   VSCALE: h2d = { x[n] fp32 },                 d2h = { y[n] fp32 }
 *   GEMM:   h2d = { A[m*k] bf16, B[k*n] bf16 },  d2h = { C[m*n] fp32 }  (row-major)
 *           m % 128 == 0, n % 256 == 0, k % 64 == 0, k <= 256, reps >= 1
 *   XFER:   h2d = { x[n] u32 },                  d2h = { y[n] u32 }
 *   HIST:   h2d = { x[n] u8 },                   d2h = { bins[256] u32 }
 *   SCAN:   h2d = { x[n] u32 },                  d2h = { y[n] u32 }
 *   SORT:   h2d = { x[n] u32 }, n % 2048 == 0,   d2h = { y[n] u32 }                           */
typedef struct {
    uint32_t kclass;         /* STRINGS_VSCALE / GEMM / XFER / HIST / SCAN / SORT              */
    uint32_t reps;           /* GEMM repetitions R (R-17); ignored otherwise                  */
    uint64_t n, m, k;        /* sizes (see above)                                             */
    float    alpha;          /* VSCALE scalar                                                 */
    uint32_t seed;           /* XFER seed                                                     */
    uint64_t arrival_ns;     /* INJECTED / DECISIONS_ONLY: virtual arrival time (Eq. 4 inputs);
                                MEASURED: ignored (arrival = submit time)                     */
    uint64_t inj_h2d_ns, inj_kl_ns, inj_d2h_ns;  /* injected phase durations (INJECTED modes)   */
} strings_kernel_desc_t;

typedef struct { void* host; uint64_t bytes; } strings_buf_t;

typedef struct {
    uint64_t job;
    uint32_t tenant, seq;
    int32_t  gid;            /* logical device chosen by the balancer (-1 before PLACE)       */
    int32_t  status;         /* STRINGS_OK, STRINGS_EAGAIN (not done) or an error             */
    uint64_t t_arrival, t_place;
    uint64_t t_start[3], t_done[3];          /* per phase H2D, KL, D2H (library clock)       */
    int32_t  kl_slot;                        /* logical KL slot                               */
    int32_t  kl_partition;                   /* physical SM partition that ran the KL        */
    uint64_t kl_gpu_start_ns, kl_gpu_end_ns; /* %globaltimer: partition leader saw the doorbell, last
                                                CTA finished                                  */
    uint64_t kl_gpu_exec_ns;                 /* %globaltimer: the body started (after broadcast) */
    uint64_t kl_host_issue_ns;               /* CLOCK_REALTIME: item published in the ring     */
    uint64_t kl_host_observe_ns;             /* CLOCK_REALTIME: completion seen by the engine  */
} strings_job_info_t;

typedef struct {
    uint64_t jobs_submitted, jobs_done, jobs_failed;
    uint64_t t_first_submit_ns, t_last_done_ns;   /* library clock                              */
    uint64_t h2d_bytes, d2h_bytes, kernel_bytes, kernel_flop;
    uint64_t trace_records;
    uint64_t decisions;                           /* PLACE + WAKE records                       */
    uint64_t decision_ns;                         /* engine time inside the decision core,
                                                     including issuing the woken ops            */
    uint64_t engine_busy_ns[8][3];                /* per logical device (first 8), per engine   */
    int32_t  num_gpus, physical_gpus, partitions, sms_per_partition;
    uint64_t issue_ns;                            /* part of decision_ns spent issuing woken ops
                                                     (cudaMemcpyAsync, stream writes, KL ring
                                                     publish); decision_ns - issue_ns = decisions.
                                                     With one issuer thread per GPU
                                                     (STRINGS_ISSUE_THREADS, default when the
                                                     process drives >= 4 GPUs) the issuing runs
                                                     on those threads, off the engine thread */
    int64_t  gpu_clock_offset_ns[8];              /* per physical GPU (first 8): %globaltimer minus
                                                     CLOCK_REALTIME, calibrated at init (kl_gpu_*
                                                     stamps - offset = host clock); 0 if unknown */
    uint64_t sm_copy_ops;                         /* H2D/D2H ops served as zero-copy SM copies by the
                                                     dispatcher's copy partition (small ops with mapped
                                                     pinned host buffers; STRINGS_COPY_CTAS,
                                                     STRINGS_SM_COPY_MAX) instead of the copy engines */
    int32_t  kl_mode;                             /* effective KL mode (0 persistent, 1 per-op launches) */
    int32_t  reserved_i32;
    uint64_t eager_jobs;                          /* MEASURED: jobs whose KL and D2H were queued on the
                                                     device behind their H2D (eager chaining, DESIGN §2;
                                                     STRINGS_EAGER=0 disables)                        */
} strings_stats_t;

/* Initialise the runtime (gPool creation): enumerate the GPUs,
 * create one context + H2D/D2H streams per GPU, allocate the resident-slot
 * arena, launch the persistent dispatcher kernel, start the engine thread.
 * cfg may be NULL (defaults).  STRINGS_ECUDA if no CUDA device is usable
 * (except in DECISIONS_ONLY mode).  STRINGS_ESTATE if already initialised.    */
strings_status_t strings_init(const strings_config_t* cfg);

/* Register a tenant (Request Manager; RCB entry P:L489-515).
 * weight >= 1 is the tenant priority/weight; max_inflight >= 1 is the number of
 * its jobs that may be admitted at once (server threads).              */
strings_status_t strings_register_tenant(uint32_t weight, uint32_t max_inflight,
                                         strings_tenant_t* out);

/* Submit one job (asynchronous): H2D of the h2d buffers, the KL
 * phase described by desc, D2H into the d2h buffers.  Jobs of one tenant are
 * admitted in submission order.  Buffer counts and sizes must match
 * desc (see strings_kernel_desc_t).  Pinned buffers (strings_host_alloc or
 * cudaHostRegister'ed) are DMA'd directly; pageable ones are staged (MOT/PMT,
 * P:L327-329): H2D data is copied at submit, D2H data is copied back before the
 * job counts as done.  The caller must not read d2h buffers (nor modify pinned
 * h2d buffers) until strings_sync(tenant) returns.  priority 0 = tenant
 * weight.  *out receives the job id.                                          */
strings_status_t strings_submit(strings_tenant_t tenant, const strings_kernel_desc_t* desc,
                                const strings_buf_t* h2d, int32_t n_h2d,
                                const strings_buf_t* d2h, int32_t n_d2h,
                                uint32_t priority, strings_job_t* out);

/* Block until every job this tenant submitted is done (Sync Stream Translator,
 * never a device-wide sync).  Returns STRINGS_EFAULT if one of
 * them failed.  In INJECTED mode this also starts virtual-time processing.   */
strings_status_t strings_sync(strings_tenant_t tenant);

/* Block until every submitted job of every tenant is done; flush the trace.    */
strings_status_t strings_drain(void);

/* Implicit sync, then remove the tenant (cudaThreadExit path, P:L329, P:L667,
 * frees its PMT staging; its feedback already reached the SFT).       */
strings_status_t strings_unregister_tenant(strings_tenant_t tenant);

/* Drain, stop the dispatcher kernel and the engine thread, free everything.   */
strings_status_t strings_shutdown(void);

/* Pinned host memory for the zero-copy fast path (R-19).                       */
strings_status_t strings_host_alloc(uint64_t bytes, void** p);
strings_status_t strings_host_free(void* p);

/* Per-job record (Request Monitor view): GID, phase times, status.     */
strings_status_t strings_job_info(strings_job_t job, strings_job_info_t* info);

/* Aggregate counters (RMO / FE view).                              */
strings_status_t strings_get_stats(strings_stats_t* stats);

/* Decision trace, kept when trace_in_memory = 1.              */
strings_status_t strings_trace_size(uint64_t* bytes);
strings_status_t strings_trace_copy(char* buf, uint64_t capacity, uint64_t* written);

const char* strings_strerror(strings_status_t s);
int32_t strings_last_cuda_error(void);
const char* strings_version(void);

/* Stand-alone tenant kernel launch (outside the scheduler) for kernel-level
 * parity tests and roofline measurements (SURVEY §8(d) "kernel-level checks").
 * dev_in / dev_out are device pointers laid out as the H2D / D2H buffers of
 * desc; ctas = number of CTAs (0 = one per SM); stream = cudaStream_t (NULL =
 * legacy default).  Asynchronous.                                              */
strings_status_t strings_kernel_launch(int32_t physical_gpu, const strings_kernel_desc_t* desc,
                                       void* const* dev_in, int32_t n_in,
                                       void* const* dev_out, int32_t n_out,
                                       int32_t ctas, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* STRINGS_SCHED_H */
