// fcl_internal.h -- internal interfaces of the FluidiCL B200 runtime (not part of the C-ABI).
//
// Three translation units share these declarations:
//   runtime.cpp      context, buffers, twin/stage pool, host executor, launch orchestration, C-ABI
//   host_bodies.cpp  host work-group bodies (the CPU side of every kernel)
//   kernels.cu       sm_100a persistent dispatcher, GPU task bodies, diff-merge kernel
//
// Bit-identity contract: for every fp32 kernel the host body
// and the GPU body perform the same IEEE-754 operations on the same operands in the same
// order (explicit fma / add / mul / div / sqrt, no contraction: host code is compiled with
// -ffp-contract=off, device code uses __f*_rn intrinsics).  Hence a word computed by the
// host is bit-identical to the word the GPU would have computed, for any split.
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>
#include <atomic>

typedef struct CUstream_st *cudaStream_t_fwd;

namespace fcl {

// The host executor's abort flag: set by the coordinator when the GPU has finished (L18.s19),
// polled by the host bodies inside long loops (relaxed loads; a data race with a plain int).
typedef std::atomic<int> AbortFlag;

enum KernelId : int {
    K_ATAX_TMP = 0, K_ATAX_Y, K_BICG_S, K_BICG_Q, K_GESUMMV, K_SYRK, K_SYR2K,
    K_CORR_MEAN, K_CORR_STD, K_CORR_REDUCE, K_CORR_CORR, K_CONV2D, K_NUM
};

// Canonical reduction shapes shared by host and device bodies (they define the
// fp32 operation order, not a thread mapping).
constexpr int kRowPartitions = 128;  // row-dot: partial q sums columns j with j % 128 == q
constexpr int kColPartitions = 32;   // col-dot: partial q sums rows i with i % 32 == q

// NDRange geometry.  fgid = g0 + ng0 * (g1 + ng1 * g2) (Fig 5, dimension 0 fastest).
struct Geom {
    int work_dim;
    int64_t gws[3], lws[3], ng[3];
    int64_t n_wg;
};

// Resolved kernel arguments (device and host addresses of every buffer argument).
struct KArgs {
    int kernel;
    bool integer;
    int nbuf;
    void *dev[6];
    void *host[6];
    int host_variant;      // host body variant (C26): 0 = CPU-oriented (default), 1 = work-item order
    int64_t n0, n1;        // rows / columns of the row-major input (SYRK/SYR2K: N, M)
    float alpha, beta, eps;
    int32_t ialpha, ibeta;
    // SYRK / SYR2K over the whole range: the GPU runs only the upper-triangle tiles and writes
    // each one's mirror too -- fma(A_i, A_j, acc) == fma(A_j, A_i, acc) bit for bit, and SYR2K's
    // per-k pair order is symmetric, so C's accumulator is symmetric; a slice
    // runs every tile of its rows (its lower-left blocks' mirrors lie outside it, and its own
    // mirrors would land outside it)
    bool sym;
    // Row-dot inputs streamed to the device in pieces while the grid runs: the
    // body loads them through L2 only
    bool streamed;
    // Test hook (opts.record_exec_counts): per work-group host completions, counted by the
    // executor (rec_parts: parts of a split work-group done so far).  nullptr = off.
    int32_t *rec_cpu_done, *rec_cpu_parts;
};

// Device-side merge of a cooperative launch's output buffers (domain read from wm_word).
struct DevMergeList {
    unsigned char *gpu[6];
    const unsigned char *cpu[6];
    const unsigned char *twin[6];
    long long unit_wgs[6], unit_bytes[6], total[6];   // span descriptor (unit_wgs 0 = whole buffer)
    int es[6];
    int n;
    const unsigned long long *wm_word;
    unsigned int epoch;
    long long hi;
    unsigned long long *tstamp;         // optional %globaltimer stamps [start, end] (stats mode)
    unsigned long long *exit_word;      // mapped host word: set to `epoch` when this kernel starts
};

// Parameters of one cooperative (FluidiCL) dispatcher launch.
struct CoopCtl {
    const unsigned long long *status;   // {epoch:32 | W:32}; device-visible address
    unsigned int epoch;                 // this launch's kernel id (C14)
    unsigned int w_default;             // watermark when the status is stale: the range end
    unsigned long long *claim;          // this launch's claim counter (0 on entry)
    unsigned long long *claim_next;     // the next launch's claim counter (reset here)
    unsigned long long *tasks;          // optional: tasks executed (0 on entry), nullptr = off
    unsigned long long *tasks_next;     // optional: next launch's task counter (reset here)
    unsigned long long *wm_out;         // {epoch | ~lowest watermark acted on}, atomicMax
    long long task_lo, task_hi;         // task index range of this launch
    int abort_period;                   // in-task poll period (body-specific units); 0 = none
    int check_first;                    // 1: check the watermark before a CTA's first task too
    int status_mapped;                  // 1: status in mapped host memory (synchronous loads only)
    unsigned long long *tstamp;         // optional %globaltimer stamps [start, end] (stats mode)
    unsigned long long *tstamp_next;    // the next launch's stamps (its end stamp is reset here)
    int fused;                          // 1: grid barrier + exit signal + merge in this kernel
    unsigned int *barrier;              // this launch's grid-barrier counter (0 on entry)
    unsigned int *barrier_next;         // the next launch's counter (reset here)
    unsigned long long *merge_ctr;      // fused merge: chunk counter (0 on entry)
    unsigned long long *merge_ctr_next; // the next launch's chunk counter (reset here)
    unsigned long long *exit_word;      // mapped host word set to `epoch` after the barrier
    DevMergeList mg;                    // merge list (mg.n == 0: nothing to merge in-kernel)
    // Streamed inputs: {epoch:32 | front:32}, device word written by stream
    // memops behind the H2D pieces -- work-groups [0, front) have their input rows on the
    // device.  nullptr: every input is resident.  A task waits for its rows or for the host to
    // cover it.
    const unsigned long long *arrival;
    unsigned long long task_delay_ns;   // fault injection (opts.gpu_delay_us): every task starts late
    unsigned int *exec_cnt;             // test hook: per task (index - task_lo) completions, or nullptr
    unsigned int *exec_w;               // ... and the work-group mask the task ran with
};

// Decode the dispatcher's wm word: the lowest watermark launch `epoch` acted on, or
// 0xFFFFFFFF if it never skipped a task.
#ifdef __CUDACC__
#define FCL_HD __host__ __device__
#else
#define FCL_HD
#endif
FCL_HD inline unsigned int decode_wm_word(unsigned long long r, unsigned int epoch) {
    return ((unsigned int)(r >> 32) == epoch) ? 0xFFFFFFFFu - (unsigned int)r : 0xFFFFFFFFu;
}


// ---- GPU side (kernels.cu) ----
struct TaskSpace {
    int64_t ntasks;      // tasks covering the whole NDRange, keys ascending
    int threads;         // CTA size of the body
};
TaskSpace gpu_task_space(const KArgs &a, const Geom &g);
int64_t gpu_task_key(const KArgs &a, const Geom &g, int64_t t);   // min fgid of task t
// Work-groups task t writes outputs of (a tile spans several; row/column dot tasks are part of
// one; SYRK's upper-triangle tiles also their mirror block), appended to `out`.
void gpu_task_wgs(const KArgs &a, const Geom &g, int64_t t, std::vector<int64_t> &out);
bool gpu_geometry_ok(const KArgs &a, const Geom &g, const char **why);
int gpu_default_abort_period(const KArgs &a);
// Slice boundaries (multi-GPU / wg_lo, wg_hi) must be multiples of this many work-groups
// so that no GPU task straddles a boundary.
int64_t gpu_slice_align(const KArgs &a, const Geom &g);
// Launch the persistent cooperative dispatcher; returns the grid size used (<= 0 on error).
int gpu_launch_coop(const KArgs &a, const Geom &g, const CoopCtl &c, int num_sms, void *stream);
// Plain grid over tasks [task_lo, task_hi) with no status reads (GPU-only baseline, and the
// cooperative single-wave case, see gpu_coop_capacity).  `reset` (nullable): the dispatcher
// counters of the next launch slot, zeroed by block 0 as a dispatcher would.
struct SlotReset {
    unsigned long long *claim, *tasks, *merge_ctr;
    unsigned int *barrier;   // 17 words
    // exit signal of a lite cooperative launch (nullable): the last CTA to arrive on `arrive`
    // (this slot's 17 counters, zero on entry) stores `epoch` to the mapped host word
    unsigned int *arrive;
    unsigned long long *exit_word;
    unsigned int epoch;
    unsigned long long *tstamp;   // optional (stats): [block-0 start, last CTA end] %globaltimer
    unsigned long long delay_ns;  // test hook (FCL_TEST_GPU_DELAY_US): block 0 idles this long first
    unsigned int *exec_cnt;       // test hook: per block completions (opts.record_exec_counts), or nullptr
};
// pdl: PDL_OFF = ordinary launch; PDL_NOWAIT = programmatic stream serialization, the grid may
// start while the previous plain grid drains and does not wait for it (the runtime found no
// buffer shared with any grid possibly still in flight); PDL_WAIT = same, but every CTA first
// waits for the grids before it (griddepcontrol.wait).
enum { PDL_OFF = 0, PDL_NOWAIT = 1, PDL_WAIT = 2 };
int gpu_launch_plain(const KArgs &a, const Geom &g, int64_t task_lo, int64_t task_hi, void *stream,
                     const SlotReset *reset = nullptr, int pdl = PDL_OFF);
// CTAs of the persistent dispatcher resident at once (occupancy x SMs): a launch with no more
// tasks than this runs in a single wave, every CTA's only task unchecked.
int64_t gpu_coop_capacity(const KArgs &a, const Geom &g, int num_sms);
// Load every kernel of the library now (CUDA lazy loading would load a kernel at its first
// launch, which may wait for the device -- see kernels.cu).  0 on success.
int gpu_preload_kernels();
// Fig 9 diff-merge on [0, bytes) of three device buffers.
int gpu_launch_merge(void *gpu, const void *cpu, const void *twin, size_t bytes, int elem_size,
                     int num_sms, void *stream);
int gpu_launch_merge_dev(const DevMergeList &L, size_t max_bytes, int num_sms, void *stream);
// Copy up to 6 (dst, src, bytes) regions in one launch (16-byte aligned pointers; dst may be the
// device-visible address of mapped host memory).  1 = launched, 0 = nothing to copy, -2 = a
// pointer is not 16-byte aligned (nothing launched), -1 = launch failure.
// pdl: launched with programmatic serialization behind plain grids, waiting in-kernel for them.
int gpu_launch_copies(int n, void *const *dst, const void *const *src, const size_t *bytes, int num_sms,
                      void *stream, bool pdl = false);
// a[j][i] = a[i][j] for i < j on an n x n row-major device matrix (multi-rank CORR combine).
int gpu_launch_mirror_upper(void *a, long long n, int elem_size, int num_sms, void *stream);
// One-thread kernel that stores `value` to `addr` (status publication fallback).
// stamp (nullable): %globaltimer right after the store (exit-drain measurement, FCL_TEST_PUBLISH_ZERO_US).
int gpu_launch_store64(unsigned long long *addr, unsigned long long value, void *stream,
                       unsigned long long *stamp = nullptr);
const char *gpu_last_error_string();

// ---- Host side (host_bodies.cpp) ----
// Execute part `part` of `nparts` of work-group `fgid` on host memory (C9 / C23).
// `abort_flag` is polled inside long bodies; a body that sees it set stops before
// storing an incomplete value (write-once).
// Returns true when the part completed (every output stored), false when the abort flag stopped it.
bool host_exec_wg(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts,
                  const AbortFlag *abort_flag);
// Alternate host bodies (C26): how many a kernel has and their names ("cpu", "wi").
int host_num_variants(int kernel);
const char *host_variant_name(int kernel, int v);
// Work-groups per executor claim (host_exec_range) and the range executor itself.
int64_t host_batch(const KArgs &a, const Geom &g);
bool host_exec_range(const KArgs &a, const Geom &g, int64_t f_lo, int64_t f_hi, const AbortFlag *abort_flag);

// Conservative contiguous byte span [*b0, *b1) of output buffer `buf_index` written by
// work-groups [lo, hi) (superset of the exact footprint; the diff-merge tolerates it).
void out_span(const KArgs &a, const Geom &g, int buf_index, int64_t lo, int64_t hi,
              size_t *b0, size_t *b1);
// The same spans in closed form: span_lo(W) = min(floor(W / unit_wgs) * unit_bytes, total),
// span_hi(W) = min(ceil(W / unit_wgs) * unit_bytes, total); unit_wgs == 0: the whole buffer.
void out_span_desc(const KArgs &a, const Geom &g, int buf_index, long long *unit_wgs,
                   long long *unit_bytes, long long *total);

}  // namespace fcl
