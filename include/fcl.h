/*
 * fcl.h -- C-ABI of the B200-native FluidiCL hot path.
 *
 * FluidiCL (Pandit & Govindarajan, CGO 2014; /root/reference/PAPER.md, cited
 * as L<line>.s<sentence>) takes a kernel written for one
 * device and executes its flattened work-group range cooperatively: the GPU
 * claims work-groups from the bottom (ascending flattened id), host threads
 * execute chunks from the top (descending) and publish a completed-from
 * watermark; a GPU work-group exits early once the host covers it; a
 * diff-merge then restores one coherent buffer (L14.s32-44, L16.s5-22,
 * L16.s28-35, Fig 9).
 *
 * Conventions shared by every entry point:
 *  - Plain C types only; no torch/CUDA types.  "device pointer" arguments are
 *    CUDA device addresses; "stream" arguments are cudaStream_t passed as
 *    void* (NULL = the context's own stream).
 *  - Every function returns an fcl_status (FCL_SUCCESS = 0; errors < 0 use
 *    OpenCL-style codes).  No C++ exception crosses this boundary.
 *  - Asynchronous CUDA / host-thread failures are reported by the next call
 *    that synchronises (fcl_finish) and make the context sticky-failed
 *    (FCL_CONTEXT_LOST), mirroring CUDA's sticky errors.
 *  - A context is NOT thread-safe: one in-order queue, as an OpenCL command
 *    queue (L22.s14: kernel calls block).  One context per GPU per process.
 *  - Kernels must not use atomics (L14.s50 footnote): work-groups are
 *    independent (L14.s22-23), which is what makes the split legal.
 */
#ifndef FCL_H
#define FCL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t fcl_status;

/* Status codes (values follow OpenCL where an equivalent exists). */
#define FCL_SUCCESS                   0
#define FCL_DEVICE_NOT_AVAILABLE     -2
#define FCL_OUT_OF_RESOURCES         -5
#define FCL_INVALID_VALUE           -30
#define FCL_INVALID_CONTEXT         -34
#define FCL_INVALID_MEM_OBJECT      -38
#define FCL_INVALID_KERNEL_NAME     -46
#define FCL_INVALID_KERNEL          -48
#define FCL_INVALID_KERNEL_ARGS     -52
#define FCL_INVALID_WORK_DIMENSION  -53
#define FCL_INVALID_WORK_GROUP_SIZE -54
#define FCL_INVALID_GLOBAL_WORK_SIZE -63
#define FCL_CONTEXT_LOST          -1000  /* sticky: a prior asynchronous failure */
#define FCL_CUDA_ERROR            -1001  /* a CUDA runtime call failed (see fcl_last_error) */
#define FCL_NOT_SUPPORTED         -1002

typedef struct fcl_context_st *fcl_context;
typedef struct fcl_buffer_st  *fcl_buffer;
typedef struct fcl_kernel_st  *fcl_kernel;

/* Where the GPU reads the host's watermark from.
 * DEVICE (default): a 64-bit word in device memory;
 * HOST_MAPPED: a 64-bit word in pinned, mapped host memory, read over PCIe.
 * In both cases the word is written by a stream memory operation on the `hd`
 * stream right after the chunk's data copy, so status always follows data on
 * an in-order queue (L16.s15).  Measured on B200: GPU reads of the mapped word
 * serialise over PCIe (~0.6 ms per 1k-task launch), the device word costs
 * ~0.5 us per read from L2. */
#define FCL_STATUS_DEVICE      0
#define FCL_STATUS_HOST_MAPPED 1

typedef struct {
    int32_t device;          /* CUDA device ordinal */
    int32_t n_host_threads;  /* host executor threads; 0 = (cores of the affinity mask on the GPU's
                                NUMA node, or all of the mask if fewer than 3) - 2: one core is
                                the coordinator's, one is left to the calling thread */
    int32_t pin_threads;     /* 1 = pin executor threads to cores of the affinity mask */
    int32_t status_location; /* FCL_STATUS_DEVICE (default) | FCL_STATUS_HOST_MAPPED */
    void   *main_stream;     /* optional cudaStream_t for kernels/merge; NULL = own stream */
    void   *hd_stream;       /* optional cudaStream_t for CPU->GPU staging (L20.s10-12) */
    void   *dh_stream;       /* optional cudaStream_t for GPU->CPU results   (L20.s10-12) */
    /* optional device allocator for buffers and the twin/stage pool (C6, L20.s23-29), e.g. the
       torch caching allocator; both NULL = cudaMalloc / cudaFree.  dev_alloc returns a device
       pointer (16-byte aligned) or NULL on failure; alloc_user is passed through. */
    void *(*dev_alloc)(size_t bytes, void *alloc_user);
    void  (*dev_free)(void *ptr, void *alloc_user);
    void   *alloc_user;
} fcl_context_desc;

/* Create a context on desc->device (desc may be NULL: device 0, defaults) -- FluidiCL's runtime
 * initialization (L20.s10-12: the hd / dh command queues; L18.s18-21: the CPU scheduler thread;
 * L20.s23-29: the buffer pool).
 * Owns: streams it creates, the pinned status words, device counters, the
 * twin/stage pool and the host executor threads.  Loads every kernel of the
 * library (no lazy loading at a first launch, which can wait for the device
 * while a grid waits for host-driven copies).  Errors: FCL_INVALID_VALUE,
 * FCL_DEVICE_NOT_AVAILABLE, FCL_OUT_OF_RESOURCES, FCL_CUDA_ERROR. */
fcl_status fcl_create_context(const fcl_context_desc *desc, fcl_context *out);
fcl_status fcl_release_context(fcl_context ctx);

/* ---- Buffers (C3, L14.s49-50; L16.s1): every buffer exists on both the
 * host (a pinned mirror) and the device; writes go to both. ---- */
#define FCL_MEM_READ_WRITE     (1u << 0)
#define FCL_MEM_WRITE_ONLY     (1u << 1)
#define FCL_MEM_READ_ONLY      (1u << 2)
#define FCL_MEM_USE_HOST_PTR   (1u << 3)  /* host mirror = caller's memory (must be pinned) */
#define FCL_MEM_USE_DEVICE_PTR (1u << 4)  /* device copy = caller's device allocation */

/* Create a dual-resident buffer of `bytes` bytes whose merge granularity is
 * `elem_size` bytes (the buffer's base type, L16.s32-35; must be 1, 2, 4 or
 * 8 and divide `bytes`).  host_init (nullable) is copied to both copies.
 * Errors: FCL_INVALID_VALUE (size/elem_size), FCL_OUT_OF_RESOURCES. */
fcl_status fcl_create_buffer(fcl_context ctx, uint32_t flags, size_t bytes, uint32_t elem_size,
                             const void *host_init, fcl_buffer *out);

/* As fcl_create_buffer, but adopt caller-owned memory: with
 * FCL_MEM_USE_HOST_PTR, host_ptr (pinned, >= bytes) becomes the host mirror;
 * with FCL_MEM_USE_DEVICE_PTR, device_ptr (>= bytes, 16-byte aligned)
 * becomes the device copy.  The caller keeps ownership and must keep the
 * memory alive until fcl_release_buffer.  Both copies are assumed coherent
 * on entry unless only one pointer is given, in which case the other copy is
 * initialised from it. */
fcl_status fcl_create_buffer_ext(fcl_context ctx, uint32_t flags, size_t bytes, uint32_t elem_size,
                                 void *host_ptr, void *device_ptr, fcl_buffer *out);
fcl_status fcl_release_buffer(fcl_buffer buf);

/* Write [offset, offset+n) of buf from host memory src to both copies
 * (clEnqueueWriteBuffer -> writes to both devices, L16.s1).  src may be the
 * buffer's own host mirror (then only the device copy is updated).  With
 * blocking == 1 the host->device copy is made before the call returns.  With
 * blocking == 0 a partial write copies asynchronously on the main stream, and
 * a write of the whole buffer refreshes the device copy lazily: when a launch
 * first needs it on the GPU (never, if the data is consumed on the host alone
 * under device selection).  src may be reused as soon as the
 * call returns (it is copied to the pinned mirror first).
 * Errors: FCL_INVALID_VALUE (range), FCL_CONTEXT_LOST. */
fcl_status fcl_write_buffer(fcl_context ctx, fcl_buffer buf, size_t offset, size_t n,
                            const void *src, int32_t blocking);

/* Read [offset, offset+n) of buf into dst.  Uses the host mirror when it is
 * current (data location tracking, L20.s31-33), else copies device->host.
 * Always blocking for the returned bytes. */
fcl_status fcl_read_buffer(fcl_context ctx, fcl_buffer buf, size_t offset, size_t n,
                           void *dst, int32_t blocking);

/* Buffer versions (C18, L20.s1-9): the kernel ID (a per-context launch counter, from 1) of the
 * last launch that writes the buffer, and of the data its host and device copies hold once the
 * work queued for them has landed -- after fcl_finish both equal `expected` unless a copy is
 * stale by design (the device copy after a CPU-only launch until a GPU launch needs it, the host
 * copy after fcl_buffer_device_written until it is read).  Any out pointer may be NULL. */
fcl_status fcl_buffer_versions(fcl_buffer buf, uint64_t *expected, uint64_t *host, uint64_t *device);

/* Query a buffer's pointers and sizes (any out pointer may be NULL). */
fcl_status fcl_buffer_info(fcl_buffer buf, void **host_ptr, void **device_ptr, size_t *bytes,
                           uint32_t *elem_size);

/* ---- Kernels.  Built in: each is a GPU body (instantiated in the
 * persistent dispatcher) plus a host work-group body with the same
 * arithmetic.  Names: atax_tmp, atax_y, bicg_s, bicg_q,
 * gesummv, syrk, syr2k, conv2d (suffix _f32 or _i32) and corr_mean,
 * corr_std, corr_reduce, corr_corr (suffix _f32).  Argument signatures are
 * listed in DESIGN.md §5 and returned by fcl_kernel_signature. ---- */
fcl_status fcl_get_kernel(fcl_context ctx, const char *name, fcl_kernel *out);
/* Writes a '\0'-terminated signature such as "A:in x:in tmp:out n0:i n1:i"
 * into buf (at most len bytes). */
fcl_status fcl_kernel_signature(fcl_kernel k, char *buf, size_t len);
/* Alternate host bodies of a kernel (C26, L22.s4-11): *n (>= 1) variants; names[v] for v < *n
 * is "cpu" (the CPU-oriented body, variant 0) or "wi" (the kernel as written for the GPU, run
 * work-item by work-item).  All variants of a kernel produce bit-identical outputs.
 * names may be NULL. */
fcl_status fcl_kernel_host_variants(fcl_kernel k, int32_t *n, const char **names, int32_t max_names);

#define FCL_ARG_BUFFER 0
#define FCL_ARG_INT    1
#define FCL_ARG_FLOAT  2

#define FCL_ACCESS_IN    1
#define FCL_ACCESS_OUT   2
#define FCL_ACCESS_INOUT 3   /* IN | OUT (C4: out/inout identification, L16.s2) */

typedef struct {
    int32_t    kind;    /* FCL_ARG_BUFFER | FCL_ARG_INT | FCL_ARG_FLOAT */
    int32_t    access;  /* for buffers: FCL_ACCESS_*; must cover what the kernel writes */
    fcl_buffer buffer;
    int64_t    i;       /* FCL_ARG_INT value */
    double     f;       /* FCL_ARG_FLOAT value (rounded to the kernel's float type) */
} fcl_arg;

#define FCL_MODE_COOP     0  /* FluidiCL cooperative execution (the method) */
#define FCL_MODE_GPU_ONLY 1  /* the same GPU bodies as a plain grid, + D2H of outputs */
#define FCL_MODE_CPU_ONLY 2  /* the host executor runs every work-group */

typedef struct {
    int32_t mode;            /* FCL_MODE_* (default COOP) */
    int64_t forced_split;    /* >= 0: test hook -- the host executes exactly [s, hi) and the GPU
                                is told so before it starts (deterministic split); -1 = race */
    int32_t init_chunk_pct;  /* C11 initial chunk, % of work-groups (default 2; L26.s28) */
    int32_t step_pct;        /* C11 growth step, % of work-groups (default 2) */
    int32_t cpu_wg_split;    /* C23 work-group splitting across host threads (default 1) */
    int32_t abort_period;    /* in-loop abort check every K inner iterations (C24/C25); 0 = default,
                                < 0 = checks at work-group start only (NoAbortUnroll analog) */
    int32_t defer_merge;     /* 1 = leave staged results unmerged until fcl_merge (test hook) */
    int32_t n_host_threads;  /* 0 = context default; else use at most this many */
    int32_t host_delay_us;   /* fault injection: sleep before each host chunk */
    int32_t drop_publish;    /* fault injection: stage chunks but never publish the watermark */
    int64_t wg_lo, wg_hi;    /* execute only flattened ids [wg_lo, wg_hi) (multi-GPU slice, SURVEY
                                §8e); wg_hi < 0 (default) = the whole NDRange; wg_lo == wg_hi = an
                                empty slice: the call returns FCL_SUCCESS and runs nothing */
    int32_t blocking;        /* 1 = return only when the launch's host side is done (the paper's
                                blocking calls, L22.s14); 0 (default) = OpenCL-style enqueue */
    int32_t flags;           /* FCL_LAUNCH_* bits */
    int32_t host_variant;    /* host body variant (C26 online profiling, L22.s4-11): -1 (default) =
                                profile -- when the kernel has alternate host bodies, the first
                                host chunks try each on a small allocation and the fastest per
                                work-group runs the rest (and later launches of the same kernel
                                and shape); >= 0 = always this one (fcl_kernel_host_variants) */
    int32_t select;          /* COOP device selection from online profiles:
                                FCL_SELECT_DEFAULT (0) = the context's setting (on unless the
                                environment sets FCL_SELECT=0), FCL_SELECT_ON (1), FCL_SELECT_OFF (-1:
                                always the cooperative path).  When on, a free-running COOP launch of a
                                kernel and shape whose last cooperative probe showed that one device
                                cannot contribute runs on the other alone: GPU-only if the host
                                finished less than FCL_SELECT_MIN_SHARE (10 %) of the work-groups
                                before the GPU exited, CPU-only if the host covered the whole range
                                first on an idle GPU, or at least FCL_SELECT_STREAM_SHARE (75 %) of a
                                launch whose stale inputs were streamed over PCIe;
                                the FCL_SELECT_PERIOD-th (16) launch after a
                                probe probes cooperatively again, a period that doubles (up to 16x)
                                while probes keep confirming the choice.  Forced splits, deferred
                                merges and fault injection are never redirected.  Sequence
                                selection on top (FCL_SEQ_SELECT=0 turns it off): the eligible
                                launches between two fcl_finish calls are timed as a whole, first
                                enqueue to the end of fcl_finish, per signature; when the probes'
                                host rates predict the host alone faster (or, with no rate, the
                                sequence is small), three sequences now and then run on the host
                                alone, and the better of each kind's last four wins
                                (info.seq_host). */
    int32_t gpu_delay_us;        /* fault injection: in a COOP launch every GPU task starts this many us
                                    late (a slow GPU, so that the host covers part of the range in a
                                    free-running race); such a launch runs the persistent dispatcher */
    int32_t record_exec_counts;  /* test hook (1 = on): count, per work-group, how often each device
                                    executed it to completion -- read with fcl_get_exec_counts after
                                    fcl_finish.  The launch first waits for pending launches. */
} fcl_launch_opts;

#define FCL_SELECT_OFF     (-1)
#define FCL_SELECT_DEFAULT 0
#define FCL_SELECT_ON      1

/* opts.flags: record CUDA events around the GPU kernel (info.t_gpu_kernel_ms); off by default
 * because each event costs host time on the launch path. */
#define FCL_LAUNCH_TIMING 1u

/* Fill *opts with the defaults above. */
fcl_status fcl_default_launch_opts(fcl_launch_opts *opts);

/* info.gpu_path */
#define FCL_GPU_PATH_NONE       0  /* no GPU kernel (CPU-only mode, empty range) */
#define FCL_GPU_PATH_DISPATCHER 1  /* persistent dispatcher: ascending claims, watermark checks, fused merge */
#define FCL_GPU_PATH_LITE       2  /* cooperative single wave without in-task polls: every CTA's one task is
                                      unchecked, so the dispatcher reduces to a plain grid + exit signal */
#define FCL_GPU_PATH_PLAIN      3  /* GPU-only mode: plain grid */

typedef struct {
    int64_t n_wg;                /* work-groups in the executed range */
    int64_t wg_lo, wg_hi;
    int64_t gpu_watermark;       /* lowest watermark the GPU acted on (hi if it never skipped) */
    int64_t published_watermark; /* last watermark the host published (hi if none) */
    int64_t gpu_tasks, gpu_tasks_total;  /* GPU tasks executed / in the range */
    int64_t cpu_wgs;             /* work-groups the host executed (incl. abandoned partial chunks) */
    int32_t n_chunks;            /* host chunks started */
    int32_t cpu_did_all;         /* the host covered the whole range first (L16.s21) */
    int32_t merged;              /* a diff-merge was enqueued */
    int32_t gpu_launches;        /* kernels of ours launched for this call */
    int64_t merge_bytes;         /* bytes of each stream covered by the merge(s) */
    int64_t h2d_bytes, d2h_bytes;
    double  t_call_ms;           /* host wall time of fcl_enqueue_ndrange */
    double  t_gpu_kernel_ms;     /* CUDA-event time of the dispatcher / plain grid on the main stream */
    double  t_merge_ms;          /* CUDA-event time of the merge kernel(s) */
    double  t_host_ms;           /* host executor busy time */
    int32_t chunk_sizes[64];     /* first chunk sizes (C11 trace) */
    int32_t gpu_path;            /* FCL_GPU_PATH_*: how the GPU side of the launch ran */
    int32_t race;                /* 1 = large output returned by the return race */
    int32_t host_variant;        /* host body variant used after profiling (-1: the host ran nothing) */
    int32_t n_host_variants;     /* alternate host bodies the kernel has */
    double  profile_ms_per_wg[4];/* online-profiling time per work-group of each variant (0 = not
                                    measured in this launch) */
    int32_t selected;            /* FCL_SELECTED_*: what a COOP launch ran as (opts.select) */
    int32_t probe;               /* 1 = this cooperative launch refreshes the selection profile */
    int64_t streamed_wgs;        /* work-groups whose stale input rows were streamed to the GPU in
                                    pieces while the host computed */
    double  chunk_ms[64];        /* host time of each started chunk (chunk_sizes order) that completed;
                                    0 = abandoned.  The first n_c11_chunks are the C11 chunks, timed
                                    exactly as the heuristic saw them (L18.s23-32) */
    int32_t n_c11_chunks;        /* chunks sized by C11; the rest of n_chunks are return-race chunks */
    int32_t seq_host;            /* 1 = run on the host alone by sequence selection: the launches
                                    between two fcl_finish calls, timed as a whole, ran faster on
                                    the host alone than with per-launch selection */
} fcl_launch_info;

/* info.selected */
#define FCL_SELECTED_COOP 0  /* both devices (the method) */
#define FCL_SELECTED_GPU  1  /* GPU alone: the host could not finish a work-group before the GPU */
#define FCL_SELECTED_CPU  2  /* host alone: it covered the whole range before the GPU exited */

/* Launch `kernel` over the NDRange (work_dim in 1..3, gws[k] % lws[k] == 0,
 * prod(lws) <= 1024) with args in the kernel's signature order.
 * COOP: the GPU dispatcher and the host executor race over the range.  The
 * call queues the GPU work and hands the host side to the context's
 * coordinator thread, then returns (like clEnqueueNDRangeKernel); a launch
 * that writes a buffer a pending launch touches (or vice versa) first waits
 * for the pending launches.  After fcl_finish every output buffer is coherent
 * on host and device.  GPU_ONLY / CPU_ONLY wait for pending launches first.
 * opts / info may be NULL; info receives what is known at return (complete
 * with opts.blocking = 1, otherwise use fcl_get_launch_info after fcl_finish).
 * Errors: FCL_INVALID_WORK_DIMENSION, FCL_INVALID_WORK_GROUP_SIZE,
 * FCL_INVALID_GLOBAL_WORK_SIZE, FCL_INVALID_KERNEL_ARGS, FCL_INVALID_VALUE,
 * FCL_OUT_OF_RESOURCES, FCL_CONTEXT_LOST. */
fcl_status fcl_enqueue_ndrange(fcl_context ctx, fcl_kernel kernel, uint32_t work_dim,
                               const size_t gws[3], const size_t lws[3],
                               const fcl_arg *args, uint32_t n_args,
                               const fcl_launch_opts *opts, fcl_launch_info *info);

/* Merge the staged host results of the last kernel into buf's device copy
 * (only needed with opts.defer_merge = 1; otherwise a no-op).  Fig 9. */
fcl_status fcl_merge(fcl_context ctx, fcl_buffer buf);

/* The diff-merge kernel on raw device memory (microbench / test entry):
 * for every elem_size-byte element e of [0, bytes):
 *     if (cpu[e] != twin[e]) gpu[e] = cpu[e]        (bitwise compare)
 * gpu, cpu, twin: device pointers, equal alignment mod 16 for the vector
 * path; bytes % elem_size == 0; elem_size in {1,2,4,8}.  Asynchronous on
 * `stream` (cudaStream_t; NULL = legacy default stream). */
fcl_status fcl_merge_raw(void *gpu, const void *cpu, const void *twin, size_t bytes,
                         uint32_t elem_size, void *stream);

/* The caller changed [offset, offset+n) of buf's device copy outside the runtime -- the NCCL
 * all-gather that brings other ranks' output slices into it ("the slices are
 * concatenated ... when the kernel's output is needed whole").  The writes were queued on
 * `stream` (cudaStream_t; NULL = the context's main stream): later work of the context is ordered
 * after them.  The device copy becomes authoritative; the host mirror is refreshed on demand (a
 * read, a host-side launch).  Waits for pending launches first.
 * Errors: FCL_INVALID_MEM_OBJECT, FCL_INVALID_VALUE (range), FCL_CONTEXT_LOST. */
fcl_status fcl_buffer_device_written(fcl_context ctx, fcl_buffer buf, size_t offset, size_t n, void *stream);

/* Mirror the upper triangle of an n x n row-major matrix on the device into its lower
 * triangle: a[j][i] = a[i][j] for every i < j (elem_size 4 or 8; the diagonal is untouched).
 * The combine step of CORR's symmat across ranks: work-group j1 writes row j1 right of the
 * diagonal and column j1 below it (PolyBench CORR, Table 2 / L22.s36), so a rank's slice is
 * L-shaped; after the row slabs are all-gathered, the upper triangle is complete and the lower
 * one follows from it.  `a` is a device pointer; asynchronous on `stream`.
 * Errors: FCL_INVALID_VALUE, FCL_CUDA_ERROR. */
fcl_status fcl_mirror_upper(void *a, size_t n, uint32_t elem_size, void *stream);

/* Wait until every launch, merge and copy of the context has completed (clFinish; the results
 * "returned to the host", L16.s36-38, L20.s13-19);
 * outputs are then coherent on host and device.  Reports deferred errors. */
fcl_status fcl_finish(fcl_context ctx);

/* Info of the most recent fcl_enqueue_ndrange, with event timings resolved
 * (call after fcl_finish). */
fcl_status fcl_get_launch_info(fcl_context ctx, fcl_launch_info *info);

/* Cumulative launch counters of the context since its creation (diagnostics; how COOP launches
 * ran under device selection).  counts[FCL_COUNT_*] for k < n are written; n
 * larger than FCL_COUNT_N writes FCL_COUNT_N entries.  Thread-compatible like every call on the
 * context.  Errors: FCL_INVALID_CONTEXT, FCL_INVALID_VALUE (counts NULL or n < 0). */
#define FCL_COUNT_COOP       0  /* COOP launches that ran cooperatively (probes included) */
#define FCL_COUNT_PROBE      1  /* ... of which device-selection probes */
#define FCL_COUNT_SEL_GPU    2  /* COOP launches run on the GPU alone by device selection */
#define FCL_COUNT_SEL_CPU    3  /* COOP launches run on the host alone by device selection */
#define FCL_COUNT_GPU_ONLY   4  /* GPU_ONLY-mode launches */
#define FCL_COUNT_CPU_ONLY   5  /* CPU_ONLY-mode launches */
#define FCL_COUNT_H2D_BYTES  6  /* bytes copied host -> device (writes, refreshes, staged chunks) */
#define FCL_COUNT_D2H_BYTES  7  /* bytes copied device -> host (returns, reads) */
#define FCL_COUNT_LAUNCH_DRAINS 8  /* launches that had to wait for pending host sides first (the
                                      hazards buffer versions do not order) */
#define FCL_COUNT_SEQ_HOST   9  /* COOP launches run on the host alone by sequence selection (also
                                      counted in FCL_COUNT_SEL_CPU) */
#define FCL_COUNT_SEQ_TRIALS 10 /* sequence-selection trials started */
#define FCL_COUNT_N          11
fcl_status fcl_get_counters(fcl_context ctx, int64_t *counts, int32_t n);

/* Per-work-group execution counts of the most recent launch made with opts.record_exec_counts
 * (test hook; north_star's invariant "every output word is written by exactly one
 * device", L16.s9 "non-overlapping parts").  Arrays of n >= the NDRange's work-group count,
 * indexed by flattened id (Fig 5); entries outside the launch's [wg_lo, wg_hi) are 0.
 *   gpu_done[f]  : completed GPU task fragments that stored work-group f's outputs
 *   gpu_frags[f] : GPU task fragments covering f (a tile task spans several work-groups, a
 *                  row/column-dot task is a part of one: f ran completely on the GPU iff
 *                  gpu_done[f] == gpu_frags[f], and not at all iff gpu_done[f] == 0)
 *   cpu_done[f]  : host executions of f that completed (all its parts stored)
 * Any pointer may be NULL.  Waits for the context (like fcl_finish).
 * Errors: FCL_INVALID_CONTEXT; FCL_INVALID_VALUE (no recorded launch, n too small). */
fcl_status fcl_get_exec_counts(fcl_context ctx, int64_t n, int32_t *gpu_done, int32_t *gpu_frags,
                               int32_t *cpu_done);

/* Multi-GPU slicing helper: a contiguous flattened-id range for
 * rank `rank` of `nranks`, balanced and aligned to the kernel's GPU task
 * granularity so slices never split a task. */
fcl_status fcl_slice_range(fcl_kernel kernel, uint32_t work_dim, const size_t gws[3],
                           const size_t lws[3], int32_t rank, int32_t nranks,
                           int64_t *wg_lo, int64_t *wg_hi);

const char *fcl_status_string(fcl_status s);
const char *fcl_last_error(fcl_context ctx);
/* Library version string, e.g. "fcl-b200 0.1 sm_100a". */
const char *fcl_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FCL_H */
