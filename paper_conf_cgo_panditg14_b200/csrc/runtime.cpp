// runtime.cpp -- the FluidiCL runtime for one B200 + its host cores, behind the C-ABI fcl.h.
//
// Components:
//   * context: CUDA device, streams main / hd / dh (L20.s10-13), the 64-bit watermark words
//     {epoch, W} (D1, C14; one per launch slot) in device or pinned mapped memory, the mapped
//     GPU-exit word, per-slot device claim counters, the kernel-id epoch;
//   * launch queue: fcl_enqueue_ndrange queues a launch's GPU work (twin capture, dispatcher,
//     merge, return copy) from the calling thread and hands its host side to the coordinator
//     thread -- the paper's CPU scheduler thread (C10, L18.s18-21) -- so, like OpenCL's
//     clEnqueueNDRangeKernel, the call does not block on the GPU (the paper's blocking calls
//     were a stated limitation, L22.s14); fcl_finish waits for everything;
//   * dual-resident buffers (C3, L14.s49-50 / L16.s1) with element-size metadata (C16, D6) and
//     host/device validity flags (minimal data-location tracking, C22 / L20.s31-33);
//   * twin + stage buffer pool (C5/C6, L16.s2-3, L20.s23-29);
//   * host executor: a pinned, spinning thread pool that runs descending chunks of work-groups
//     (C9/C10, L16.s6-10, L18.s18-21) sized by the adaptive heuristic (C11, L18.s23-32), with
//     work-group splitting (C23, L20.s34-39);
//   * stager/publisher: after each chunk, its output span goes host->device on `hd` and a stream
//     memory operation then stores {epoch, lo} -- status follows data (C13, L16.s11/s.15-18);
//   * merge launcher (C15, Fig 9) and the device->host return of the GPU's part (C17, L16.s36-38).
#include <execinfo.h>
#include <csignal>
#include <unistd.h>
#include <cuda.h>
#include <cuda_runtime.h>
#include <immintrin.h>
#include <sched.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <cctype>
#include <map>
#include <array>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../../include/fcl.h"
#include "fcl_internal.h"

using namespace fcl;

namespace {

using Clock = std::chrono::steady_clock;
inline double now_ms() {
    return std::chrono::duration<double, std::milli>(Clock::now().time_since_epoch()).count();
}

// ------------------------------------------------------------------------------------------
// Kernel table (built-in kernels; C27's source transformation is replaced by templates)
// ------------------------------------------------------------------------------------------
struct ArgSpec {
    const char *name;
    char kind;      // 'b' buffer, 'i' int, 'f' float
    uint8_t acc;    // buffers: 1 read, 2 written, 3 read+written
};
struct KernelDef {
    const char *name;
    int id;
    bool integer;
    int nargs;
    ArgSpec args[9];
};

#define B_IN(n) {n, 'b', 1}
#define B_OUT(n) {n, 'b', 2}
#define B_INOUT(n) {n, 'b', 3}
#define I_(n) {n, 'i', 0}
#define F_(n) {n, 'f', 0}

const KernelDef kKernels[] = {
    {"atax_tmp_f32", K_ATAX_TMP, false, 5, {B_IN("A"), B_IN("x"), B_OUT("tmp"), I_("nx"), I_("ny")}},
    {"atax_tmp_i32", K_ATAX_TMP, true, 5, {B_IN("A"), B_IN("x"), B_OUT("tmp"), I_("nx"), I_("ny")}},
    {"atax_y_f32", K_ATAX_Y, false, 5, {B_IN("A"), B_IN("tmp"), B_OUT("y"), I_("nx"), I_("ny")}},
    {"atax_y_i32", K_ATAX_Y, true, 5, {B_IN("A"), B_IN("tmp"), B_OUT("y"), I_("nx"), I_("ny")}},
    {"bicg_s_f32", K_BICG_S, false, 5, {B_IN("A"), B_IN("r"), B_OUT("s"), I_("nx"), I_("ny")}},
    {"bicg_s_i32", K_BICG_S, true, 5, {B_IN("A"), B_IN("r"), B_OUT("s"), I_("nx"), I_("ny")}},
    {"bicg_q_f32", K_BICG_Q, false, 5, {B_IN("A"), B_IN("p"), B_OUT("q"), I_("nx"), I_("ny")}},
    {"bicg_q_i32", K_BICG_Q, true, 5, {B_IN("A"), B_IN("p"), B_OUT("q"), I_("nx"), I_("ny")}},
    {"gesummv_f32", K_GESUMMV, false, 8,
     {B_IN("A"), B_IN("B"), B_IN("x"), B_OUT("tmp"), B_OUT("y"), I_("n"), F_("alpha"), F_("beta")}},
    {"gesummv_i32", K_GESUMMV, true, 8,
     {B_IN("A"), B_IN("B"), B_IN("x"), B_OUT("tmp"), B_OUT("y"), I_("n"), I_("alpha"), I_("beta")}},
    {"syrk_f32", K_SYRK, false, 6, {B_IN("A"), B_INOUT("C"), I_("n"), I_("m"), F_("alpha"), F_("beta")}},
    {"syrk_i32", K_SYRK, true, 6, {B_IN("A"), B_INOUT("C"), I_("n"), I_("m"), I_("alpha"), I_("beta")}},
    {"syr2k_f32", K_SYR2K, false, 7,
     {B_IN("A"), B_IN("B"), B_INOUT("C"), I_("n"), I_("m"), F_("alpha"), F_("beta")}},
    {"syr2k_i32", K_SYR2K, true, 7,
     {B_IN("A"), B_IN("B"), B_INOUT("C"), I_("n"), I_("m"), I_("alpha"), I_("beta")}},
    {"corr_mean_f32", K_CORR_MEAN, false, 4, {B_IN("data"), B_OUT("mean"), I_("n"), I_("m")}},
    {"corr_std_f32", K_CORR_STD, false, 6,
     {B_IN("data"), B_IN("mean"), B_OUT("std"), I_("n"), I_("m"), F_("eps")}},
    {"corr_reduce_f32", K_CORR_REDUCE, false, 5, {B_INOUT("data"), B_IN("mean"), B_IN("std"), I_("n"), I_("m")}},
    {"corr_corr_f32", K_CORR_CORR, false, 4, {B_IN("data"), B_OUT("symmat"), I_("n"), I_("m")}},
    {"conv2d_f32", K_CONV2D, false, 4, {B_IN("A"), B_OUT("B"), I_("ni"), I_("nj")}},
    {"conv2d_i32", K_CONV2D, true, 4, {B_IN("A"), B_OUT("B"), I_("ni"), I_("nj")}},
};
constexpr int kNumKernels = sizeof(kKernels) / sizeof(kKernels[0]);

// Elements each buffer argument must hold, given the problem extents (n0, n1).
int64_t required_elems(int kid, int b, int64_t n0, int64_t n1) {
    switch (kid) {
    case K_ATAX_TMP: { const int64_t r[] = {n0 * n1, n1, n0}; return r[b]; }
    case K_ATAX_Y: { const int64_t r[] = {n0 * n1, n0, n1}; return r[b]; }
    case K_BICG_S: { const int64_t r[] = {n0 * n1, n0, n1}; return r[b]; }
    case K_BICG_Q: { const int64_t r[] = {n0 * n1, n1, n0}; return r[b]; }
    case K_GESUMMV: { const int64_t r[] = {n0 * n0, n0 * n0, n0, n0, n0}; return r[b]; }
    case K_SYRK: { const int64_t r[] = {n0 * n1, n0 * n0}; return r[b]; }
    case K_SYR2K: { const int64_t r[] = {n0 * n1, n0 * n1, n0 * n0}; return r[b]; }
    case K_CORR_MEAN: { const int64_t r[] = {n0 * n1, n1}; return r[b]; }
    case K_CORR_STD: { const int64_t r[] = {n0 * n1, n1, n1}; return r[b]; }
    case K_CORR_REDUCE: { const int64_t r[] = {n0 * n1, n1, n1}; return r[b]; }
    case K_CORR_CORR: { const int64_t r[] = {n0 * n1, n1 * n1}; return r[b]; }
    case K_CONV2D: { const int64_t r[] = {n0 * n1, n0 * n1}; return r[b]; }
    default: return 0;
    }
}

// NDRange extent each dimension must cover (PolyBench pads gws up to a multiple of lws).
void required_extent(int kid, int64_t n0, int64_t n1, int64_t ext[3]) {
    ext[0] = ext[1] = ext[2] = 1;
    switch (kid) {
    case K_ATAX_TMP: case K_BICG_Q: case K_GESUMMV: ext[0] = n0; break;
    case K_ATAX_Y: case K_BICG_S: case K_CORR_MEAN: case K_CORR_STD: case K_CORR_CORR: ext[0] = n1; break;
    case K_SYRK: case K_SYR2K: ext[0] = n0; ext[1] = n0; break;
    case K_CORR_REDUCE: case K_CONV2D: ext[0] = n1; ext[1] = n0; break;
    default: break;
    }
}

// ------------------------------------------------------------------------------------------
// Host executor (C9/C10/C23): T pinned worker threads, spinning while hot.
// ------------------------------------------------------------------------------------------
struct Executor {
    std::vector<std::thread> threads;
    std::vector<int> cores;
    int T = 0;
    std::atomic<uint64_t> gen{0};
    std::atomic<int> stop{0};
    std::mutex mu;
    std::condition_variable cv;
    std::atomic<int> sleepers{0};
    // current job (written before `next` is released)
    KArgs a{};
    Geom g{};
    int64_t lo = 0, hi = 0;
    int nparts = 1;
    // read by workers before their claim is validated (a worker still looping on the previous
    // job): atomics, relaxed -- the compare-and-swap on `next` decides
    std::atomic<int64_t> total{0};
    std::atomic<int> active{0};
    // claim word: (job generation << 40) | next item.  Claims use compare-and-swap so a
    // worker still looping on a finished job can never consume an item of the next one.
    std::atomic<uint64_t> next{0};
    std::atomic<int64_t> done{0};
    int64_t batch = 1;   // work-groups per claim (host_batch), 1 when work-groups are split
    AbortFlag abort_flag{0};
    int64_t spin_ns = 2 * 1000 * 1000;    // spin 2 ms after a job before sleeping

    // local: the cores of the GPU's NUMA node (empty: unknown); the executor uses those of the
    // process affinity mask that are local to the GPU when there are at least three of them
    void start(int nthreads, bool pin, const std::vector<int> &local = {}) {
        cpu_set_t set;
        CPU_ZERO(&set);
        if (sched_getaffinity(0, sizeof set, &set) == 0) {
            for (int c = 0; c < CPU_SETSIZE; ++c)
                if (CPU_ISSET(c, &set)) cores.push_back(c);
        }
        if (!local.empty()) {
            std::vector<int> both;
            for (int c : cores)
                if (std::find(local.begin(), local.end(), c) != local.end()) both.push_back(c);
            if (both.size() >= 3) cores = both;
        }
        if (cores.empty()) cores.push_back(0);
        // default: every core but two -- one for the coordinator (cores[0]), one left free for
        // the calling thread -- so no spinning party ever time-slices with another
        T = nthreads > 0 ? nthreads : std::max<int>(1, (int)cores.size() - 2);
        active = T;
        for (int k = 0; k < T; ++k) threads.emplace_back([this, k, pin] { worker(k, pin); });
    }
    void shutdown() {
        stop.store(1);
        {
            std::lock_guard<std::mutex> lk(mu);
            cv.notify_all();
        }
        for (auto &t : threads) t.join();
        threads.clear();
    }
    void worker(int idx, bool pin) {
        if (pin && cores.size() > 1) {
            cpu_set_t s;
            CPU_ZERO(&s);
            // cores[0]: the coordinator; cores[1]: the caller (unless there are too few cores)
            const size_t skip = cores.size() > 2 ? 2 : 1;
            CPU_SET(cores[(size_t)(idx + skip) % cores.size()], &s);
            sched_setaffinity(0, sizeof s, &s);
        }
        uint64_t seen = 0;
        for (;;) {
            auto t0 = Clock::now();
            while (gen.load(std::memory_order_acquire) == seen && !stop.load(std::memory_order_relaxed)) {
                _mm_pause();
                if (std::chrono::duration_cast<std::chrono::nanoseconds>(Clock::now() - t0).count() > spin_ns) {
                    std::unique_lock<std::mutex> lk(mu);
                    sleepers.fetch_add(1);
                    cv.wait(lk, [&] { return gen.load() != seen || stop.load(); });
                    sleepers.fetch_sub(1);
                    t0 = Clock::now();
                }
            }
            if (stop.load()) return;
            seen = gen.load(std::memory_order_acquire);
            if (idx >= active.load(std::memory_order_relaxed)) continue;
            for (;;) {
                uint64_t v = next.load(std::memory_order_acquire);
                if ((v >> 40) != (seen & 0xFFFFFFu)) break;
                const int64_t it = (int64_t)(v & ((1ull << 40) - 1));
                if (it >= total.load(std::memory_order_relaxed)) break;
                if (!next.compare_exchange_weak(v, v + 1, std::memory_order_acq_rel)) continue;
                if (!abort_flag.load(std::memory_order_relaxed)) {
                    if (batch == 1) {
                        const int64_t fgid = hi - 1 - it / nparts;   // descending (L14.s36)
                        const bool ok = host_exec_wg(a, g, fgid, (int)(it % nparts), nparts, &abort_flag);
                        if (ok && a.rec_cpu_done) {   // test hook: a work-group counts once all its parts completed
                            if (nparts == 1 || __atomic_add_fetch(a.rec_cpu_parts + fgid, 1, __ATOMIC_ACQ_REL) == nparts) {
                                if (nparts > 1) __atomic_store_n(a.rec_cpu_parts + fgid, 0, __ATOMIC_RELAXED);
                                __atomic_add_fetch(a.rec_cpu_done + fgid, 1, __ATOMIC_RELAXED);
                            }
                        }
                    } else {   // a run of work-groups, runs claimed in descending order
                        const int64_t fh = hi - it * batch, fl = std::max<int64_t>(lo, fh - batch);
                        const bool ok = host_exec_range(a, g, fl, fh, &abort_flag);
                        if (ok && a.rec_cpu_done)
                            for (int64_t f = fl; f < fh; ++f) __atomic_add_fetch(a.rec_cpu_done + f, 1, __ATOMIC_RELAXED);
                    }
                }
                done.fetch_add(1, std::memory_order_acq_rel);
            }
        }
    }
    // Submit work-groups [lo_, hi_) split `parts` ways; returns immediately.  The previous job
    // must be finished (every claimed item executed or skipped): callers quiesce first.
    void submit(const KArgs &a_, const Geom &g_, int64_t lo_, int64_t hi_, int parts, int nact) {
        wait();   // (defensive: a straggler's done increment must not count for the new job)
        const uint64_t g1 = gen.load(std::memory_order_relaxed) + 1;
        // Close the claim word first (new generation, no item claimable): a worker still looping
        // on the previous job -- e.g. one that woke for an empty job -- may have loaded the old
        // word and be about to compare-and-swap it; with the word changed its CAS fails, so it
        // can never claim an "item" of the old job while the fields below already describe the
        // new one (that executed a work-group twice: in-place kernels applied twice).
        next.store(((g1 & 0xFFFFFFu) << 40) | ((1ull << 40) - 1), std::memory_order_seq_cst);
        a = a_; g = g_; lo = lo_; hi = hi_; nparts = parts;
        batch = parts > 1 ? 1 : std::max<int64_t>(1, host_batch(a_, g_));
        total.store(parts > 1 ? (hi_ - lo_) * parts : (hi_ - lo_ + batch - 1) / batch, std::memory_order_relaxed);
        active.store(std::max(1, std::min(nact, T)), std::memory_order_relaxed);
        done.store(0, std::memory_order_relaxed);
        next.store((g1 & 0xFFFFFFu) << 40, std::memory_order_release);
        gen.store(g1, std::memory_order_release);
        if (sleepers.load() > 0) {
            std::lock_guard<std::mutex> lk(mu);
            cv.notify_all();
        }
    }
    bool finished() const { return done.load(std::memory_order_acquire) >= total.load(std::memory_order_relaxed); }
    void wait() {
        while (!finished()) _mm_pause();
    }
};

// Optional host-side event trace (FCL_TRACE=1): (time, tag, epoch) triples printed at
// context release; used to attribute host latency, never on by default.
struct TraceRec { double t; const char *tag; uint32_t epoch; };
struct Tracer {
    bool on = false;
    std::mutex mu;
    std::vector<TraceRec> recs;
    void add(const char *tag, uint32_t e) {
        if (!on) return;
        std::lock_guard<std::mutex> lk(mu);
        if (recs.size() < 200000) recs.push_back({now_ms(), tag, e});
    }
};

struct PoolEnt {
    void *p;
    size_t bytes;
    bool used;
    bool hd_pending;      // a staging copy on hd may still write it (wait on ev_hd_release)
    uint32_t last_epoch;
};

}  // namespace

// ------------------------------------------------------------------------------------------
// Opaque handle types
// ------------------------------------------------------------------------------------------
struct fcl_kernel_st {
    const KernelDef *def;
};

struct fcl_buffer_st {
    fcl_context ctx;
    size_t bytes;
    uint32_t elem_size;
    uint32_t flags;
    void *dev;
    void *host;
    bool own_dev, own_host;
    bool host_valid, dev_valid;
    // The return-copy state below is written by the API thread (queueing a return) and read,
    // for the buffers of its job, by the coordinator's phase B while later launches are being
    // enqueued: atomics (relaxed -- the order that matters comes from the job queue and events)
    std::atomic<bool> d2h_pending{false};
    std::atomic<bool> d2h_on_main{false};   // the pending return copy is queued on main (a lazy
                                            // return): later grids on main are ordered behind it
                                            // without a cross-stream wait
    std::atomic<bool> d2h_on_race{false};   // ... queued on the race stream (a later return on dh
                                            // waits for it)
    bool ret_lazy;         // a lazy return of [ret_b0, ret_b1) is registered, not yet queued
    size_t ret_b0, ret_b1;
    std::atomic<uint64_t> d2h_gen{0};   // ctx->finish_gen when the pending return was queued
    void *host_dptr;       // device-visible address of the (mapped) host mirror, nullptr = none
    cudaEvent_t d2h_ev;    // completion of the buffer's pending return copy (recorded on dh)
    // deferred merge state (opts.defer_merge)
    bool merge_pending;
    void *twin, *stage;
    size_t m_b0, m_b1, r_b0, r_b1;   // merge span, return (D2H) span
    // Buffer versions (C18, L20.s1-9): the kernel ID of the last launch that writes the buffer
    // (expected), and of the data its host and device copies hold once everything queued for
    // them has landed (host_ver / dev_ver).  host_seq: the host-only job (a queued CPU-only
    // launch) that last writes its host copy -- while it is pending, a GPU-side reader waits for
    // the copy's transfer on the device (a stream memory wait), not on the host.
    uint64_t ver_expected, ver_host, ver_dev;
    uint64_t host_seq;
};

typedef CUresult (*PFN_writeValue64)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
typedef CUresult (*PFN_waitValue64)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);

namespace {

struct Launch {
    fcl_context ctx;
    const KernelDef *kd;
    KArgs a;
    Geom g;
    fcl_buffer bufs[6];
    uint8_t acc[6];   // 1 read, 2 written, 3 both
    int out_idx[6];
    int nout;
    bool any_inout;   // some output is read-modify-written in place (INOUT)
    int64_t lo, hi;
    fcl_launch_opts o;
};

// One cooperative launch in flight: phase A (GPU side, calling thread) then phase B (host
// side, coordinator thread).
struct Job {
    // JOB_COOP: a cooperative launch's host side (phase B); JOB_CPU: a CPU-only launch, run by the
    // coordinator in queue order; JOB_XFER: host->device copies of buffers a pending JOB_CPU
    // writes, published by a ticket a later GPU launch waits for on the device
    enum { JOB_COOP = 0, JOB_CPU = 1, JOB_XFER = 2 };
    int kind = JOB_COOP;
    uint64_t host_seq = 0;     // JOB_CPU: its host-job sequence number
    uint64_t ticket = 0;       // JOB_XFER: the value stored to the transfer word after the copies
    int nx = 0;
    fcl_buffer xb[6] = {};     // JOB_XFER: the buffers
    Launch L;
    uint32_t epoch = 0;
    int slot = 0;
    int64_t t0 = 0, t1 = 0, s_forced = -1;
    bool forced = false, dev_merge = false, eager = false, gpu_launched = false;
    bool lazy = false;         // outputs return lazily (batched on main at the next flush point)
    bool lite = false;         // single wave, no in-task polls: plain grid + exit memop, never a merge
    bool exact_spans = false;  // every output's footprint of a work-group range is one exact span
    bool twin_alias = false;   // exact spans: the merge compares against the device copy itself
    int64_t unit = 1;          // host chunk boundaries are multiples of this many work-groups
    void *twin[6] = {nullptr}, *stage[6] = {nullptr};
    // ev_k0/ev_t1/ev_m0/ev_m1 carry timestamps and are recorded only when timing is asked for:
    // a timing event between two grids on main stops the second from overlapping the first
    // (PDL) and costs ~3 us per boundary even without it (scripts/ubench_dots.cu)
    cudaEvent_t ev_t1 = nullptr;
    cudaEvent_t ev_start = nullptr, ev_k0 = nullptr, ev_k1 = nullptr, ev_m0 = nullptr, ev_m1 = nullptr,
                ev_staged = nullptr, ev_ret = nullptr, ev_wm = nullptr, ev_d2h = nullptr;
    cudaEvent_t main_before = nullptr;   // an event on main at or after every earlier launch's merge
    bool have_k = false, have_m = false, wm_pending = false;
    fcl_launch_info info{};
    fcl_status status = FCL_SUCCESS;
    std::atomic<int> done{0};
    bool stream = false;                 // inputs streamed to the device in row pieces (§6.7)
    int nstream = 0, sbuf[6] = {0};      // streamed buffers (argument indices)
    bool probe = false;                  // refreshes the device-selection profile of its shape
    bool probe_gpu_idle = false;         // the GPU had nothing queued when the probe was enqueued
    std::array<int64_t, 9> sel_key{};
};

}  // namespace

struct fcl_context_st {
    int device = 0;
    int num_sms = 148;
    void *(*dev_alloc)(size_t, void *) = nullptr;   // fcl_context_desc allocator (nullptr: cudaMalloc)
    void (*dev_free)(void *, void *) = nullptr;
    void *alloc_user = nullptr;
    cudaStream_t main = nullptr, hd = nullptr, dh = nullptr;
    bool own_main = false, own_hd = false, own_dh = false;
    // JOB_XFER copies and their tickets.  Not hd: phase A queues waits for main positions on hd
    // (forced splits, staging) that can lie behind a launch's wait for a ticket -- a transfer on
    // hd would then wait for itself.  xt only ever waits for main positions before that wait.
    cudaStream_t xt = nullptr;
    std::atomic<int> xt_used{0};
    // Return-race pieces (DESIGN.md §6.4 item 8) go on their own stream: on dh they would queue
    // behind a later launch's return that waits for its (long) kernel, and stop returning while
    // that kernel runs.  A later return of the same buffer waits for the race's d2h_ev.
    cudaStream_t dr = nullptr;
    std::atomic<int> dr_used{0};
    int status_location = FCL_STATUS_DEVICE;
    // One 64-bit status word per launch slot (epoch % kSlots): a dispatcher that is still
    // running after its host side returned never sees a later launch's watermark.
    static constexpr int kSlots = 16;
    unsigned long long *status_host = nullptr;   // mapped host words (HOST_MAPPED)
    unsigned long long *status_dptr = nullptr;   // device-visible address of slot 0
    bool slot_used[kSlots] = {};
    unsigned long long *wm_host = nullptr;       // pinned copy of the dispatcher's wm word
    // mapped words, one per launch slot: epoch of the last finished GPU grid of that slot (per
    // slot, because grids of consecutive launches may overlap and finish out of order, PDL)
    unsigned long long *exit_host = nullptr;
    unsigned long long *exit_dptr = nullptr;     // their device-visible address
    // Programmatic dependent launch of plain grids (FCL_NO_PDL=1 disables): buffers touched by
    // plain grids that may still be in flight -- a new grid sharing one with them (and at least
    // one side writing) waits for them in-kernel; an op queued on main that a grid must not
    // overtake (a stream wait, a copy on main) makes the next grid an ordinary launch.
    struct ChainEnt { fcl_buffer b; int acc; };
    bool pdl = true;
    std::vector<ChainEnt> pdl_chain;
    int pdl_chain_grids = 0;
    std::atomic<int> main_fenced{1};
    // fcl_finish generation: a return copy queued before the last fcl_finish has completed
    std::atomic<uint64_t> finish_gen{1};
    // something was queued on dh / hd since the last fcl_finish (else it skips their syncs)
    std::atomic<int> dh_used{1}, hd_used{1};
    unsigned long long *dclaim = nullptr, *dtasks = nullptr, *dwm = nullptr;
    unsigned long long *dstamp = nullptr;        // stats mode: %globaltimer stamps, 4 per slot
    unsigned long long *dpstamp = nullptr;       // stats mode: plain-grid stamps, 2 per grid since fcl_finish
    int pst_n = 0;
    static constexpr int kPlainStamps = 64;
    unsigned int *dbar = nullptr;                // grid-barrier counters, one per slot
    unsigned long long *dmctr = nullptr;         // fused-merge chunk counters, one per slot
    bool unfused = false;                        // FCL_UNFUSED_MERGE=1: merge as a separate kernel
    bool no_lite = false;                        // FCL_NO_LITE=1: always the full dispatcher
    bool no_sym = false;                         // FCL_NO_SYM=1: SYRK runs every tile (no mirrored writes)
    bool ktiming = false;                        // CUDA events around every kernel (FCL_KTIMING=1)
    cudaEvent_t main_tail = nullptr;             // ev_k1 of the last cooperative dispatcher
    uint32_t epoch = 0;
    PFN_writeValue64 write64 = nullptr;
    PFN_waitValue64 wait64 = nullptr;
    // Buffer versions (C18/C21): launch ids (the paper's kernel IDs), host-only jobs and transfers
    uint64_t kid = 0;                            // kernel ID of the latest launch
    uint64_t host_seq = 0;                       // host-only jobs queued
    std::atomic<uint64_t> host_done_seq{0};      // host-only jobs completed (in queue order)
    uint64_t xfer_seq = 0;                       // transfer tickets issued
    unsigned long long *d_xfer = nullptr;        // device word: the last ticket whose copies landed
    // Exit-drain measurement (FCL_TEST_PUBLISH_ZERO_US, with FCL_STATS=1): the host side
    // of a free-running dispatcher launch computes nothing, publishes W = wg_lo this many us after
    // it starts, with a store kernel that stamps %globaltimer, and no merge runs -- the outputs are
    // INCOMPLETE; only for scripts/exit_drain.py.  dpub: the stamps, one per slot.
    int64_t test_publish_zero_us = 0;
    unsigned long long *dpub = nullptr;
    bool no_version_wait = false;                // FCL_NO_VERSION_WAIT=1: skip the device-side wait
                                                 // (test hook: shows the stale read it prevents)
    bool stats = false;                          // count executed GPU tasks, time merges (FCL_STATS=1)
    size_t eager_return_bytes = 8u << 20;        // outputs up to this size return right behind the merge
    // Lazy return: small outputs of free-running and GPU-only launches are not
    // copied back behind each grid (a copy on dh waits on an event of main, which keeps the next
    // grid from starting under this one's tail and costs ~5 us per kernel boundary).  Their spans
    // are registered and copied in ONE batched copy on main at the next point that needs a host
    // copy: fcl_finish, fcl_read_buffer, a launch whose host side reads them (FCL_LAZY_BYTES,
    // 0 = off).  At that point the device copy is authoritative for every registered span.
    size_t lazy_max_bytes = 1u << 20;
    std::vector<fcl_buffer> lazy;
    // Online profiling of alternate host bodies (C26): the winner per kernel and shape, so that
    // only the first launch of a shape pays for trying the slower variants
    std::mutex var_mu;
    std::map<std::array<int64_t, 6>, int> variant_cache;
    // Device selection from online profiles: per kernel and shape, what the
    // last cooperative probe showed (FCL_SELECTED_*) and how many launches the shape has had.
    // next_probe: the launch index of the next probe; period: launches between probes, which
    // doubles (up to 16x select_period) each time a probe confirms the standing choice and
    // falls back to select_period when it changes
    // host_ms_per_wg: the host's best rate in the last probe (min over its completed C11 chunks of
    // chunk time / chunk size; -1 = it completed none)
    struct SelectEnt { int64_t launches = 0; int choice = FCL_SELECTED_COOP; int64_t next_probe = 0; int64_t period = 0;
                       double host_ms_per_wg = -1; };
    std::mutex sel_mu;
    std::map<std::array<int64_t, 9>, SelectEnt> sel;
    // Sequence selection (last item): the selection-eligible COOP launches
    // between two fcl_finish calls form a sequence.  Per signature (the launches' keys in order,
    // the stale bit counting only inputs no earlier launch of the sequence wrote: seq_key) the wall times from the first enqueue to the end of fcl_finish of the
    // default per-launch selection and of the host alone (last four of each), the standing
    // choice, and the trial schedule.
    typedef std::array<int64_t, 8> SeqKey;
    struct SeqEnt {
        std::vector<SeqKey> keys;
        double t_run[2][4] = {}; int n_run[2] = {0, 0};   // [0] default selection, [1] host alone
        double est_host = -1;                             // Σ host-alone estimates (ms); -1 unknown
        double work = 0;                                  // Σ multiply-adds of its launches
        int choice = 0, trial = 0, trial_kind = 0;        // trial: sequences left in the running trial
        int64_t seqs = 0, next_trial = 1, period = 64, loss_period = 32;
        int64_t inert = 0;   // sequences still to run untracked (a signature no trial is worth)
    };
    std::map<uint64_t, SeqEnt> seq_tab;
    std::map<SeqKey, uint64_t> seq_first;   // a signature's first key -> the signature
    struct SeqCur {
        std::vector<SeqKey> keys; uint64_t h = 0; double t0 = 0; double est = 0, work = 0;
        std::vector<const void *> written;   // buffers written by the sequence's launches so far
        bool ok = true;       // every launch eligible, the plan (if any) followed
        int run = -1;         // what this sequence runs: -1 no plan, 0 default, 1 host alone
        bool trial = false; uint64_t plan = 0;
        const std::vector<SeqKey> *plan_keys = nullptr;   // the planned signature's keys
    } seq;
    // Streamed launches (§6.7) queued or in phase B: their grids wait for pieces the coordinator
    // issues, so the API thread must not allocate device or pinned memory meanwhile -- an
    // allocation is an implicit synchronisation point, after which the pieces could not run
    // before the grid that waits for them (a deadlock the 5 s stream guard turned into a trap)
    std::atomic<int> stream_jobs{0};
    bool seq_on = true;                          // FCL_SEQ_SELECT=0: per-launch selection only
    bool seq_debug = false;                      // FCL_SEQ_DEBUG=1: one stderr line per recorded sequence
    bool select_on = true;                       // FCL_SELECT=0: off unless a launch asks for it
    std::atomic<int64_t> counts[FCL_COUNT_N] = {};   // fcl_get_counters (launch counts, bytes moved)
    int select_period = 16;                      // FCL_SELECT_PERIOD: every n-th launch of a shape probes
    double select_min_share = 0.10;              // FCL_SELECT_MIN_SHARE: host share a probe must reach
    double select_stream_share = 0.75;           // FCL_SELECT_STREAM_SHARE: host share of a streamed probe
                                                 // above which the host runs the shape alone
    uint32_t pool_keep = 256;                    // FCL_POOL_KEEP: launches an unused pool buffer survives
    size_t pool_cap = 16ull << 30;               // FCL_POOL_CAP_MB: unused buffers beyond this are freed
    unsigned long long test_gpu_delay_ns = 0;    // FCL_TEST_GPU_DELAY_US: lite grids start late (test hook)
    // Streamed inputs: arrival fronts, one per launch slot, and the piece events
    bool stream_on = true;                       // FCL_NO_STREAM=1: stale inputs are copied whole first
    unsigned long long *darrival = nullptr;
    cudaEvent_t stream_ev[4] = {};
    // hd position after the last piece of the last streamed launch: pieces still in flight read
    // the pinned mirror and write the device copy, so a later write of the mirror
    // (fcl_write_buffer) or a refresh of the device copy (make_valid) waits for it
    cudaEvent_t ev_stream_done = nullptr;
    bool stream_pending = false;                 // set by phase B, read after drain()
    size_t stream_piece_bytes = 8u << 20;        // FCL_STREAM_PIECE_BYTES
    // Return race: when the GPU finishes first and a large output is still to come
    // back, it is returned in ascending pieces while the host keeps computing from the top.
    bool no_race = false;                        // FCL_NO_RACE=1
    bool memop_nobarrier_ok = true;              // cleared when the driver rejects NO_MEMORY_BARRIER
    int exit_poll_pauses = 8;                    // pause instructions between exit-word polls (FCL_EXIT_POLL_PAUSES)
    // Lite grids store no exit word by default (FCL_LITE_EXIT=1 restores it): the last-CTA
    // arrival it needs costs ~2 us of grid tail per launch.  The coordinator learns that a lite
    // grid finished from fcl_finish's main-stream synchronisation (main_done_epoch) or, between
    // finishes, from its completion event polled every exit_query_mask+1 iterations.
    bool lite_exit_word = false;
    unsigned exit_query_mask = 0xFFFF;           // event polls every mask+1 exit-word polls
    unsigned lite_query_mask = 0x3F;             // the same for lite grids without an exit word
    // every grid queued on main up to this epoch has completed (set by fcl_finish)
    std::atomic<uint32_t> main_done_epoch{0};
    // Deferred quiescence: an abandoned chunk of an eagerly returned launch may
    // still be running; its launch's buffers are kept here until quiesce() has waited for it.
    std::mutex qz_mu;
    std::atomic<int> quiescing{0};
    fcl_buffer qz_bufs[6] = {};
    int qz_n = 0;
    int env_abort_period = 0;                    // FCL_ABORT_PERIOD: default for opts.abort_period == 0
    size_t race_min_bytes = 32u << 20;           // only for returns at least this large
    size_t race_piece_bytes = 8u << 20;          // return-copy piece
    double race_chunk_ms = 1.0;                  // host chunk length during the race
    cudaEvent_t race_ev[4] = {};                 // completion of the outstanding pieces (on dh)
    bool force_twin = false;                     // FCL_FORCE_TWIN=1: always capture a twin (Fig 9 as printed)
    // twin/stage pool (C6, L20.s23-29)
    std::mutex pool_mu;
    std::vector<PoolEnt> pool;
    cudaEvent_t ev_hd_release = nullptr;         // hd position after the last released stage copies
    // host executor + coordinator (the CPU scheduler thread, C10)
    Executor ex;
    std::mutex q_mu;
    std::condition_variable q_cv;
    std::vector<Job *> queue;                    // pending jobs, FIFO
    // Lock-free mirrors for the spin waits (coordinator wake-up, drain): a futex wake costs
    // several microseconds on the launch path, so both sides spin for a while before sleeping.
    std::atomic<int> q_len{0};                   // queue.size()
    std::atomic<int> coord_sleeping{0}, drain_sleeping{0};
    std::atomic<int> q_stop_flag{0};
    std::vector<Job *> free_jobs;
    Job *running = nullptr;
    Job *last = nullptr;                         // most recent launch (for fcl_get_launch_info)
    bool q_stop = false;
    int coord_core = -1;                         // core the coordinator is pinned to (-1: none)
    std::thread coord;
    // errors
    std::mutex err_mu;
    std::string err;
    std::atomic<fcl_status> sticky{FCL_SUCCESS};
    // single-device modes
    cudaEvent_t ev_k0 = nullptr, ev_t1 = nullptr, ev_k1 = nullptr, ev_mark = nullptr;   // k0/t1: timing only
    cudaEvent_t ev_gd2h = nullptr;               // completion of single-device / deferred returns (on dh)
    fcl_launch_info sync_info{};
    bool sync_have_k = false;
    // Test hook (opts.record_exec_counts): per-task GPU completions (with the
    // work-group mask each task ran with) and per-work-group host completions of the last
    // launch that asked for them -- fcl_get_exec_counts turns them into per-work-group counts.
    struct ExecRec {
        bool valid = false;
        KArgs a{};
        Geom g{};
        int64_t lo = 0, hi = 0, t0 = 0, t1 = 0;
        std::vector<int32_t> cpu_done, cpu_parts;
        unsigned int *d_cnt = nullptr, *d_w = nullptr;   // [t1 - t0] each
        size_t d_cap = 0;
    } rec;
    std::vector<fcl_buffer> defer_list;
    Tracer tr;
};

namespace {

// Device memory of buffers and pool entries: the context's allocator, or cudaMalloc / cudaFree.
void *dmalloc(fcl_context ctx, size_t bytes) {
    if (ctx->dev_alloc) return ctx->dev_alloc(bytes ? bytes : 16, ctx->alloc_user);
    void *p = nullptr;
    if (cudaMalloc(&p, bytes ? bytes : 16) != cudaSuccess) { cudaGetLastError(); return nullptr; }
    return p;
}
void dfree(fcl_context ctx, void *p) {
    if (!p) return;
    if (ctx->dev_free) ctx->dev_free(p, ctx->alloc_user);
    else cudaFree(p);
}

fcl_status set_err(fcl_context ctx, fcl_status s, const char *fmt, ...) {
    if (ctx) {
        char b[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(b, sizeof b, fmt, ap);
        va_end(ap);
        std::lock_guard<std::mutex> lk(ctx->err_mu);
        ctx->err = b;
    }
    return s;
}

fcl_status cuda_fail(fcl_context ctx, cudaError_t e, const char *what) {
    set_err(ctx, FCL_CUDA_ERROR, "%s: %s", what, cudaGetErrorString(e));
    if (ctx) ctx->sticky = FCL_CONTEXT_LOST;
    return FCL_CUDA_ERROR;
}

#define CK(ctx, call)                                                   \
    do {                                                                \
        cudaError_t _e = (call);                                        \
        if (_e != cudaSuccess) return cuda_fail((ctx), _e, #call);      \
    } while (0)

// A buffer's return copy may still be reading its device copy (not if an fcl_finish has
// synchronised dh since it was queued).
bool d2h_busy(fcl_context ctx, fcl_buffer b) {
    if (b->d2h_pending && b->d2h_gen < ctx->finish_gen.load(std::memory_order_acquire)) b->d2h_pending = false;
    return b->d2h_pending;
}

// ---- pool ----
// Returns the buffer and whether main must wait for ctx->ev_hd_release before writing it.
void drain(fcl_context ctx);
void *pool_get(fcl_context ctx, size_t bytes, bool *hd_wait, bool drained = false);
void *pool_get(fcl_context ctx, size_t bytes, bool *hd_wait, bool drained) {
    std::unique_lock<std::mutex> lk(ctx->pool_mu);
    int best = -1;
    for (size_t k = 0; k < ctx->pool.size(); ++k) {
        const PoolEnt &e = ctx->pool[k];
        // best fit, but never a buffer much larger than asked for (a 16 KB stage must not take
        // the 64 MB one the next launch of the step needs)
        const bool fits = e.bytes >= bytes && e.bytes <= std::max(2 * bytes, bytes + ((size_t)1 << 20));
        if (!e.used && fits && (best < 0 || e.bytes < ctx->pool[(size_t)best].bytes)) best = (int)k;
    }
    if (best >= 0) {
        PoolEnt &e = ctx->pool[(size_t)best];
        e.used = true;
        e.last_epoch = ctx->epoch;
        if (e.hd_pending) { *hd_wait = true; e.hd_pending = false; }
        return e.p;
    }
    if (!drained && ctx->stream_jobs.load(std::memory_order_acquire) > 0) {
        // (pool_mu released: the coordinator returns buffers under it while it drains)
        lk.unlock();
        drain(ctx);
        return pool_get(ctx, bytes, hd_wait, true);
    }
    void *p = dmalloc(ctx, bytes);
    if (!p) {
        // free every unused entry and retry once (L20.s29: reclaim older unused buffers)
        for (auto it = ctx->pool.begin(); it != ctx->pool.end();) {
            if (!it->used) { dfree(ctx, it->p); it = ctx->pool.erase(it); }
            else ++it;
        }
        if (!(p = dmalloc(ctx, bytes))) return nullptr;
    }
    ctx->pool.push_back({p, bytes, true, false, ctx->epoch});
    return p;
}

void pool_put(fcl_context ctx, void *p, bool hd_pending) {
    std::lock_guard<std::mutex> lk(ctx->pool_mu);
    for (auto &e : ctx->pool)
        if (e.p == p) { e.used = false; e.hd_pending = e.hd_pending || hd_pending; e.last_epoch = ctx->epoch; }
}

// "At the end of each kernel execution, older unused buffers are freed" (L20.s29).  "Older" on a
// 180 GB device: unused for pool_keep cooperative launches, or beyond pool_cap bytes in total.
// (A short horizon made a kernel that runs cooperatively only now and then -- a device-selection
// probe, DESIGN.md §6.6 -- pay cudaMalloc/cudaFree, and cudaFree synchronises the device.)
void pool_trim(fcl_context ctx) {
    std::lock_guard<std::mutex> lk(ctx->pool_mu);
    size_t total = 0;
    for (const auto &e : ctx->pool) total += e.bytes;
    for (auto it = ctx->pool.begin(); it != ctx->pool.end();) {
        const bool old = it->last_epoch + ctx->pool_keep < ctx->epoch || total > ctx->pool_cap;
        if (!it->used && !it->hd_pending && old) {
            total -= it->bytes;
            dfree(ctx, it->p);
            it = ctx->pool.erase(it);
        } else {
            ++it;
        }
    }
}

// Store `v` to `dst` after everything already queued on `s` (stream memory operation; a
// one-thread kernel store if the driver lacks 64-bit memops).
fcl_status stream_store(fcl_context ctx, unsigned long long *dst, unsigned long long v, cudaStream_t s,
                        bool barrier = true, fcl_launch_info *info = nullptr) {
    if (ctx->write64) {
        // With a barrier the store is ordered after the data of earlier operations on `s`
        // (needed for publication, C13); a bare completion signal may skip it where the driver
        // allows (it rejects NO_MEMORY_BARRIER for mapped host memory on some systems).
        const bool nb = !barrier && ctx->memop_nobarrier_ok;
        CUresult r = ctx->write64((CUstream)s, (CUdeviceptr)dst, v, nb ? (unsigned)CU_STREAM_WRITE_VALUE_NO_MEMORY_BARRIER : 0u);
        if (r == CUDA_SUCCESS) return FCL_SUCCESS;
        if (nb) {
            ctx->memop_nobarrier_ok = false;
            r = ctx->write64((CUstream)s, (CUdeviceptr)dst, v, 0u);
            if (r == CUDA_SUCCESS) return FCL_SUCCESS;
        }
        fprintf(stderr, "fcl: cuStreamWriteValue64 failed (CUresult %d, dst %p): stream memops disabled, "
                        "falling back to a store kernel\n", (int)r, (void *)dst);
        ctx->write64 = nullptr;   // fall back to the kernel store from now on
    }
    if (gpu_launch_store64(dst, v, s) < 0) return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
    if (info) info->gpu_launches += 1;   // the fallback is a kernel of ours
    return FCL_SUCCESS;
}

// Publish {epoch, W} behind everything queued on hd: status follows data (C13, L16.s15).
fcl_status publish(fcl_context ctx, const Job &j, uint32_t w) {
    const unsigned long long v = ((unsigned long long)j.epoch << 32) | w;
    ctx->hd_used.store(1, std::memory_order_relaxed);
    return stream_store(ctx, ctx->status_dptr + j.slot, v, ctx->hd, true, const_cast<fcl_launch_info *>(&j.info));
}

// Bring a buffer's copies to what a launch needs.  A pending return copy is waited for on the
// host only when the host copy is needed; a device-only use of a buffer the launch writes is
// ordered behind it on the device (write-after-read), and device-only reads need nothing.
fcl_status flush_returns(fcl_context ctx, bool at_finish);

fcl_status make_valid(fcl_context ctx, fcl_buffer b, bool need_host, bool need_dev, fcl_launch_info *info,
                      bool dev_write = true) {
    if (need_host && b->ret_lazy) {
        fcl_status f = flush_returns(ctx, false);
        if (f != FCL_SUCCESS) return f;
    }
    if (d2h_busy(ctx, b)) {
        if (need_host || !b->dev_valid) {
            CK(ctx, cudaEventSynchronize(b->d2h_ev));
            b->d2h_pending = false;
        } else if (dev_write && !b->d2h_on_main) {   // (a write-through "return" reads nothing)
            CK(ctx, cudaStreamWaitEvent(ctx->main, b->d2h_ev, 0));
            ctx->main_fenced.store(1);
        }
    }
    if (need_dev && !b->dev_valid) {
        if (ctx->stream_pending) {   // pieces of a streamed launch may still write this device copy
            CK(ctx, cudaStreamWaitEvent(ctx->main, ctx->ev_stream_done, 0));
        }
        ctx->main_fenced.store(1);
        CK(ctx, cudaMemcpyAsync(b->dev, b->host, b->bytes, cudaMemcpyHostToDevice, ctx->main));
        ctx->counts[FCL_COUNT_H2D_BYTES] += (int64_t)b->bytes;
        b->dev_valid = true;
        b->ver_dev = b->ver_host;
        if (info) info->h2d_bytes += (int64_t)b->bytes;
    }
    if (need_host && !b->host_valid) {
        CK(ctx, cudaMemcpyAsync(b->host, b->dev, b->bytes, cudaMemcpyDeviceToHost, ctx->main));
        ctx->counts[FCL_COUNT_D2H_BYTES] += (int64_t)b->bytes;
        CK(ctx, cudaStreamSynchronize(ctx->main));
        b->host_valid = true;
        b->ver_host = b->ver_dev;
        if (info) info->d2h_bytes += (int64_t)b->bytes;
    }
    return FCL_SUCCESS;
}

int64_t ceil_pct(int64_t pct, int64_t n) { return (pct * n + 99) / 100; }

// First task index whose key is >= f (keys are non-decreasing in the task index).
int64_t first_task_at(const KArgs &a, const Geom &g, int64_t ntasks, int64_t f) {
    int64_t lo = 0, hi = ntasks;
    while (lo < hi) {
        const int64_t mid = lo + (hi - lo) / 2;
        if (gpu_task_key(a, g, mid) < f) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// Device->host return of the outputs' spans of work-groups [wlo, whi), on dh behind
// `main_mark` (an event already recorded on main after the kernel / merge).
fcl_status enqueue_d2h(fcl_context ctx, Launch &L, int64_t wlo, int64_t whi, fcl_launch_info &info,
                       cudaEvent_t main_mark) {
    if (whi <= wlo) return FCL_SUCCESS;
    if (main_mark) CK(ctx, cudaStreamWaitEvent(ctx->dh, main_mark, 0));   // nullptr: dh already waits
    for (int q = 0; q < L.nout; ++q) {
        fcl_buffer b = L.bufs[L.out_idx[q]];
        size_t b0, b1;
        out_span(L.a, L.g, L.out_idx[q], wlo, whi, &b0, &b1);
        if (b1 <= b0) continue;
        ctx->dh_used.store(1, std::memory_order_relaxed);
        if (d2h_busy(ctx, b) && b->d2h_on_race) CK(ctx, cudaStreamWaitEvent(ctx->dh, b->d2h_ev, 0));
        CK(ctx, cudaMemcpyAsync((char *)b->host + b0, (char *)b->dev + b0, b1 - b0, cudaMemcpyDeviceToHost, ctx->dh));
        ctx->counts[FCL_COUNT_D2H_BYTES] += (int64_t)(b1 - b0);
        info.d2h_bytes += (int64_t)(b1 - b0);
        CK(ctx, cudaEventRecord(b->d2h_ev, ctx->dh));
        b->d2h_pending = true; b->d2h_on_main = false; b->d2h_on_race = false; b->d2h_gen = ctx->finish_gen.load();
    }
    return FCL_SUCCESS;
}

// Host-decided merges (forced split, deferred merge) on main.
fcl_status enqueue_merges(fcl_context ctx, Job &j, int64_t mlo, int64_t mhi) {
    Launch &L = j.L;
    if (mhi <= mlo) return FCL_SUCCESS;
    if (ctx->stats && !L.o.defer_merge) CK(ctx, cudaEventRecord(j.ev_m0, ctx->main));
    for (int q = 0; q < L.nout; ++q) {
        fcl_buffer b = L.bufs[L.out_idx[q]];
        size_t b0, b1;
        out_span(L.a, L.g, L.out_idx[q], mlo, mhi, &b0, &b1);
        if (b1 <= b0) continue;
        if (L.o.defer_merge) {
            b->merge_pending = true;
            b->twin = j.twin[q];   // nullptr: twin aliases the device copy
            b->stage = j.stage[q];
            b->m_b0 = b0; b->m_b1 = b1;
            j.twin[q] = j.stage[q] = nullptr;   // ownership moves to the buffer until fcl_merge
            ctx->defer_list.push_back(b);
            continue;
        }
        const char *tw = j.twin_alias ? (const char *)b->dev : (const char *)j.twin[q];
        ctx->main_tail = nullptr;
        if (gpu_launch_merge((char *)b->dev + b0, (char *)j.stage[q] + b0, tw + b0, b1 - b0,
                             (int)b->elem_size, ctx->num_sms, ctx->main) < 0)
            return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
        j.info.gpu_launches += 1;
        j.info.merge_bytes += (int64_t)(b1 - b0);
    }
    if (ctx->stats && !L.o.defer_merge) {
        CK(ctx, cudaEventRecord(j.ev_m1, ctx->main));
        j.have_m = true;
    }
    return FCL_SUCCESS;
}

// Lowest watermark the dispatcher of job j acted on (hi if it never skipped); a synchronous
// 8-byte read used off the fast path.  Only valid until a later dispatcher touches the word.
fcl_status read_gpu_watermark(fcl_context ctx, Job &j, int64_t *wm) {
    ctx->dh_used.store(1, std::memory_order_relaxed);
    CK(ctx, cudaStreamWaitEvent(ctx->dh, j.ev_k1, 0));
    CK(ctx, cudaMemcpyAsync(ctx->wm_host, ctx->dwm, 8, cudaMemcpyDeviceToHost, ctx->dh));
    CK(ctx, cudaEventRecord(j.ev_wm, ctx->dh));
    CK(ctx, cudaEventSynchronize(j.ev_wm));
    const unsigned int w = decode_wm_word(*ctx->wm_host, j.epoch);
    *wm = (w == 0xFFFFFFFFu) ? j.L.hi : std::min<int64_t>(j.L.hi, (int64_t)w);
    return FCL_SUCCESS;
}

// Wait until an abandoned chunk (deferred by an eager launch's phase B) has stopped, and clear
// the abort flag.  Serialised with the deferral itself, so a new abandonment is never lost.
void quiesce(fcl_context ctx) {
    if (!ctx->quiescing.load(std::memory_order_acquire)) return;
    std::lock_guard<std::mutex> lk(ctx->qz_mu);
    if (!ctx->quiescing.load(std::memory_order_relaxed)) return;
    ctx->ex.wait();
    ctx->ex.abort_flag = 0;
    ctx->qz_n = 0;
    ctx->quiescing.store(0, std::memory_order_release);
}

// Non-blocking quiesce: true once no abandoned chunk is running (clearing the state then).
bool quiesce_try(fcl_context ctx) {
    if (!ctx->quiescing.load(std::memory_order_acquire)) return true;
    if (!ctx->ex.finished()) return false;
    quiesce(ctx);   // (finished: returns at once)
    return true;
}

// Does launch L write a buffer the still-quiescing chunk reads or writes?
bool conflicts_with_quiescing(fcl_context ctx, const Launch &L) {
    if (!ctx->quiescing.load(std::memory_order_acquire)) return false;
    std::lock_guard<std::mutex> lk(ctx->qz_mu);
    for (int a = 0; a < L.a.nbuf; ++a)
        if (L.acc[a] & 2)
            for (int b = 0; b < ctx->qz_n; ++b)
                if (L.bufs[a] == ctx->qz_bufs[b]) return true;
    return false;
}

// Lazy return: register the launch's output spans [lo, hi) if they are small (returns false
// otherwise; the caller then queues an ordinary return copy).
bool lazy_return(fcl_context ctx, const Launch &L, fcl_launch_info &info) {
    if (ctx->lazy_max_bytes == 0) return false;
    size_t tot = 0, b0[6], b1[6];
    for (int q = 0; q < L.nout; ++q) {
        out_span(L.a, L.g, L.out_idx[q], L.lo, L.hi, &b0[q], &b1[q]);
        tot += b1[q] - b0[q];
    }
    if (tot > ctx->lazy_max_bytes) return false;
    for (int q = 0; q < L.nout; ++q) {
        fcl_buffer b = L.bufs[L.out_idx[q]];
        if (b1[q] <= b0[q]) continue;
        if (!b->ret_lazy) {
            b->ret_lazy = true;
            b->ret_b0 = b0[q]; b->ret_b1 = b1[q];
            ctx->lazy.push_back(b);
        } else {
            b->ret_b0 = std::min(b->ret_b0, b0[q]);
            b->ret_b1 = std::max(b->ret_b1, b1[q]);
        }
        info.d2h_bytes += (int64_t)(b1[q] - b0[q]);
    }
    return true;
}

// Queue every registered lazy return as one batched copy on main.  `at_finish`: the caller
// synchronises main next and clears the buffers itself (no per-buffer completion events).
fcl_status flush_returns(fcl_context ctx, bool at_finish) {
    if (ctx->lazy.empty()) return FCL_SUCCESS;
    const size_t n = ctx->lazy.size();
    std::vector<void *> dst(n), src(n);
    std::vector<size_t> sz(n);
    for (size_t k = 0; k < n; ++k) {
        fcl_buffer b = ctx->lazy[k];
        dst[k] = (char *)b->host + b->ret_b0;
        src[k] = (char *)b->dev + b->ret_b0;
        sz[k] = b->ret_b1 - b->ret_b0;
    }
    // The gather may start under the tail of the plain grids before it (programmatic dependent
    // launch) and waits in-kernel for all of them; with no PDL chain in flight it is ordinary.
    const bool pdl_gather = ctx->pdl && !ctx->main_fenced.load() && ctx->pdl_chain_grids > 0;
    ctx->main_fenced.store(1);   // a copy between grids on main: the next grid is ordinary
    for (size_t k = 0; k < n; ++k) ctx->counts[FCL_COUNT_D2H_BYTES] += (int64_t)sz[k];
    // One gather kernel stores every span through the mapped host mirrors (16-byte SM stores
    // over PCIe, posted): one launch instead of one copy-engine transfer per buffer.  Spans that
    // are not 16-byte aligned, buffers without a mapping, or more than 6 spans: one
    // cudaMemcpyAsync per span.
    bool gathered = false;
    if (n <= 6) {
        std::vector<void *> hdst(n);
        bool ok = true;
        for (size_t k = 0; k < n && ok; ++k) {
            fcl_buffer b = ctx->lazy[k];
            ok = b->host_dptr != nullptr;
            if (ok) hdst[k] = (char *)b->host_dptr + b->ret_b0;
        }
        if (ok) {
            const int r = gpu_launch_copies((int)n, hdst.data(), (const void *const *)src.data(), sz.data(), ctx->num_sms,
                                            ctx->main, pdl_gather);
            if (r == -1) return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
            gathered = r >= 0;   // (-2: a span is not 16-byte aligned)
        }
    }
    if (!gathered)
        for (size_t k = 0; k < n; ++k)
            CK(ctx, cudaMemcpyAsync(dst[k], src[k], sz[k], cudaMemcpyDeviceToHost, ctx->main));
    for (size_t k = 0; k < n; ++k) {
        fcl_buffer b = ctx->lazy[k];
        b->ret_lazy = false;
        if (!at_finish) {
            CK(ctx, cudaEventRecord(b->d2h_ev, ctx->main));
            b->d2h_pending = true; b->d2h_on_main = true; b->d2h_on_race = false; b->d2h_gen = ctx->finish_gen.load();
        }
    }
    ctx->lazy.clear();
    return FCL_SUCCESS;
}

// ---- online profiling of alternate host bodies (C26, L22.s4-11) ----
// "It starts by running each kernel version for a small allocation size and measuring time
// taken for its completion.  The best performing kernel version is picked for the remaining
// subkernels."  The allocation is one host chunk per variant (the C11 chunk of that moment);
// the comparison is per work-group.
struct VariantPick {
    int nvar = 1, var = 0, next = 0;
    bool profiling = false;
    double ms_per_wg[4] = {0, 0, 0, 0};
};

std::array<int64_t, 6> variant_key(const Launch &L) {
    return {L.a.kernel, L.a.integer ? 1 : 0, L.a.n0, L.a.n1, L.g.lws[0], L.g.work_dim > 1 ? L.g.lws[1] : 1};
}

VariantPick pick_variant(fcl_context ctx, const Launch &L) {
    VariantPick vp;
    vp.nvar = host_num_variants(L.a.kernel);
    if (L.o.host_variant >= 0) { vp.var = std::min(L.o.host_variant, vp.nvar - 1); return vp; }
    if (vp.nvar == 1) return vp;
    std::lock_guard<std::mutex> lk(ctx->var_mu);
    auto it = ctx->variant_cache.find(variant_key(L));
    if (it != ctx->variant_cache.end()) vp.var = it->second;
    else vp.profiling = true;
    return vp;
}

// Variant for the next host chunk.
int chunk_variant(VariantPick &vp) {
    if (vp.profiling && vp.next < vp.nvar) return vp.next++;
    return vp.var;
}

// A chunk of `wgs` work-groups run with variant v took dt ms.
void variant_measured(fcl_context ctx, const Launch &L, VariantPick &vp, int v, double dt, int64_t wgs) {
    if (!vp.profiling || wgs <= 0 || v < 0 || v >= 4) return;
    vp.ms_per_wg[v] = dt / (double)wgs;
    for (int k = 0; k < vp.nvar; ++k)
        if (vp.ms_per_wg[k] <= 0) return;
    int best = 0;
    for (int k = 1; k < vp.nvar; ++k)
        if (vp.ms_per_wg[k] < vp.ms_per_wg[best]) best = k;
    vp.var = best;
    vp.profiling = false;
    std::lock_guard<std::mutex> lk(ctx->var_mu);
    ctx->variant_cache[variant_key(L)] = best;
}

void variant_info(const VariantPick &vp, fcl_launch_info &info) {
    info.host_variant = vp.var;
    info.n_host_variants = vp.nvar;
    for (int k = 0; k < 4; ++k) info.profile_ms_per_wg[k] = vp.ms_per_wg[k];
}

// Stats mode: stamp pair for the next plain grid (read and cleared by fcl_finish).
// ---- device selection from online profiles ----
// A free-running cooperative launch whose kernel and shape showed, in the last cooperative
// probe, that one device cannot contribute -- the host finished no work-group before the GPU
// exited, or it covered the whole range before the GPU did -- runs on the other device alone.
// Every select_period-th launch of the shape is a cooperative probe again.
// The shape, and whether an input has to reach the GPU first (a stale device copy, e.g. after a
// lazy non-blocking write): the same kernel is host- or GPU-favoured depending on that transfer.
std::array<int64_t, 9> select_key(const Launch &L) {
    int64_t stale = 0;
    for (int k = 0; k < L.a.nbuf; ++k) stale |= ((L.acc[k] & 1) && !L.bufs[k]->dev_valid) ? 1 : 0;
    return {L.a.kernel, L.a.integer ? 1 : 0, L.a.n0, L.a.n1, L.g.lws[0], L.g.work_dim > 1 ? L.g.lws[1] : 1, L.lo, L.hi, stale};
}

bool select_eligible(fcl_context ctx, const Launch &L) {
    const bool on = L.o.select == FCL_SELECT_ON || (L.o.select == FCL_SELECT_DEFAULT && ctx->select_on);
    return on && ctx->select_period > 0 && L.o.mode == FCL_MODE_COOP && L.o.forced_split < 0 && !L.o.defer_merge &&
           L.o.host_delay_us == 0 && L.o.gpu_delay_us <= 0 && !L.o.record_exec_counts && !L.o.drop_publish && L.hi > L.lo;
}

// Returns FCL_SELECTED_* for this launch; *probe: it runs cooperatively to refresh the profile.
int select_device(fcl_context ctx, const Launch &L, bool *probe) {
    std::lock_guard<std::mutex> lk(ctx->sel_mu);
    auto &e = ctx->sel[select_key(L)];
    const int64_t n = e.launches++;
    *probe = n >= e.next_probe || e.choice == FCL_SELECTED_COOP;
    return *probe ? FCL_SELECTED_COOP : e.choice;
}

void select_update(fcl_context ctx, const Job &j, bool gpu_done) {
    int c = FCL_SELECTED_COOP;
    // A lite launch (single wave, no polls) computes every work-group on the GPU: partial host
    // work can only shorten a host-bounded return copy, never with an eager or lazy return.
    const bool host_work_useless = j.lite && (j.eager || j.lazy);
    // The host covering the whole range first only shows it is the faster device when the probe's
    // grid did not have to wait for earlier GPU work (in a chain of kernels it always does).
    if (!gpu_done) c = j.probe_gpu_idle ? FCL_SELECTED_CPU : FCL_SELECTED_COOP;
    // The host's share must also pay for the cooperative path's fixed costs (host side, chunk
    // bookkeeping, a piecewise return): below min_share of the range it does not (CORR 1024's
    // reduce: 7 % of the work-groups, 0.39 vs 0.26 ms GPU-only).
    else if (gpu_done && (host_work_useless || (double)j.info.cpu_wgs < ctx->select_min_share * (double)(j.L.hi - j.L.lo)))
        c = FCL_SELECTED_GPU;
    // A launch whose inputs crossed PCIe while it ran (streamed) and of which the
    // host still covered most of the range: the GPU's part was bounded by the link, not by its
    // compute, and it held the link that the launches after it need for their own stale inputs.
    // The host alone costs at most 1/share of the cooperative time and leaves the link to them
    // (bench.py's e2e step: GESUMMV on the host while BICG's matrix crosses, 2.5 -> 1.4 ms).
    else if (gpu_done && j.stream && (double)j.info.cpu_wgs >= ctx->select_stream_share * (double)(j.L.hi - j.L.lo))
        c = FCL_SELECTED_CPU;
    std::lock_guard<std::mutex> lk(ctx->sel_mu);
    auto &e = ctx->sel[j.sel_key];
    // a probe that confirms the standing single-device choice backs the next one off; any change
    // (or a cooperative outcome) probes again at the base period
    const int64_t base = std::max<int64_t>(1, ctx->select_period);
    e.period = (c != FCL_SELECTED_COOP && c == e.choice && e.period > 0) ? std::min<int64_t>(2 * e.period, 16 * base) : base;
    // the GPU covered the range before the host completed even its first C11 chunk (2 % of the
    // range): the host is more than ~50x slower on this shape -- probe again only rarely
    if (c == FCL_SELECTED_GPU && j.info.cpu_wgs == 0) e.period = 16 * base;
    e.choice = c;
    e.next_probe = e.launches + e.period - 1;
    double best = -1;
    for (int q = 0; q < std::min<int32_t>(j.info.n_c11_chunks, 64); ++q)
        if (j.info.chunk_ms[q] > 0 && j.info.chunk_sizes[q] > 0) {
            const double r = j.info.chunk_ms[q] / (double)j.info.chunk_sizes[q];
            if (best < 0 || r < best) best = r;
        }
    e.host_ms_per_wg = best;
}

// ---- sequence selection (last item) ----
// Per-launch selection sees one launch's race, not what the caller waits for: a chain of small
// kernels whose GPU grids each win their race can still finish later on the GPU than on the
// host alone, once launch latencies, the return of the results and the synchronisation are
// counted (ATAX 256: 32 us GPU-alone, 26 us host-alone).  So the runtime also times whole
// sequences -- the eligible COOP launches from one fcl_finish to the next, first enqueue to the
// end of fcl_finish -- and, per signature, runs now and then the other way: the host alone for
// three sequences, when the probes' host rates predict it faster than the default (or, where no
// probe's host completed a chunk, when the sequence is small), or the default selection for one,
// when the host alone is the standing choice.  The better of each kind's last four wins.  A sequence whose launches
// do not follow the planned signature stops the plan (the launches already run on the host are
// correct either way: every host body reproduces the GPU's bits).
// The selection key with its stale-input bit counting only inputs that no earlier launch of the
// sequence wrote: a sequence whose first kernel ran on the host leaves the second one's input
// stale on the device, and that must not change the signature, while inputs the caller wrote
// (the e2e loop's non-blocking writes) do.
fcl_context_st::SeqKey seq_key(const Launch &L, const std::array<int64_t, 9> &k, const std::vector<const void *> &written) {
    fcl_context_st::SeqKey s;
    for (int q = 0; q < 8; ++q) s[q] = k[q];
    int64_t stale = 0;
    for (int b = 0; b < L.a.nbuf; ++b)
        if ((L.acc[b] & 1) && !L.bufs[b]->dev_valid &&
            std::find(written.begin(), written.end(), (const void *)L.bufs[b]) == written.end())
            stale = 1;
    s[7] = s[7] * 2 + stale;   // (s[7]: the range end, folded with the bit)
    return s;
}

// The best of the last (up to) four sequences of a kind: the first run of a signature on the
// host alone pays for waking the workers and touching the host copies (0.4 ms against 0.025 ms
// warm for ATAX 256), and one such outlier must not decide.
double seq_best(const double *t, int n) {
    double v = 0;
    for (int q = 0; q < std::min(n, 4); ++q) v = (q == 0 || t[q] < v) ? t[q] : v;
    return v;
}

// Multiply-adds of a launch's range (the order of magnitude of its host work; a probe whose
// host completed no chunk gives no rate, and then only small launches are worth a trial).
double host_madds(const Launch &L) {
    const double n0 = (double)L.a.n0, n1 = (double)L.a.n1;
    double m;
    switch (L.a.kernel) {
    case K_GESUMMV: m = 2 * n0 * n0; break;
    case K_SYRK: m = n0 * n0 * n1; break;
    case K_SYR2K: m = 2 * n0 * n0 * n1; break;
    case K_CORR_CORR: m = 0.5 * n1 * n1 * n0; break;
    case K_CONV2D: m = 9 * n0 * n1; break;
    default: m = n0 * n1; break;
    }
    const double nwg = (double)(L.g.ng[0] * L.g.ng[1] * L.g.ng[2]);
    return nwg > 0 ? m * (double)(L.hi - L.lo) / nwg : m;
}

// Called for every launch before device selection; returns true if it runs on the host alone.
bool seq_launch(fcl_context ctx, const Launch &L, bool eligible) {
    auto &c = ctx->seq;
    if (!ctx->seq_on) return false;
    if (!eligible) { c.ok = false; c.run = -1; return false; }
    if (!c.ok || c.keys.size() >= 64) { c.ok = false; c.run = -1; return false; }
    if (c.keys.empty()) c.written.clear();
    const auto k9 = select_key(L);
    const fcl_context_st::SeqKey k = seq_key(L, k9, c.written);
    for (int b = 0; b < L.a.nbuf; ++b)
        if (L.acc[b] & 2) c.written.push_back(L.bufs[b]);
    const size_t pos = c.keys.size();
    // a host plan past its first launch needs none of the shared tables: follow the plan's keys
    // (std::map nodes never move, and entries are never erased)
    if (c.run == 1 && pos > 0 && c.plan_keys) {
        c.keys.push_back(k);
        for (int64_t v : k) c.h = (c.h ^ (uint64_t)v) * 1099511628211ull;
        c.work += host_madds(L);
        if (pos < c.plan_keys->size() && (*c.plan_keys)[pos] == k) return true;
        c.ok = false;   // off the planned signature: the rest runs by per-launch selection
        c.run = -1;
        return false;
    }
    std::lock_guard<std::mutex> lk(ctx->sel_mu);
    if (c.keys.empty()) {
        c.t0 = now_ms();
        c.h = 1469598103934665603ull;
        c.est = 0;
        c.work = 0;
        c.run = -1;
        c.trial = false;
        c.plan_keys = nullptr;
        auto f = ctx->seq_first.find(k);
        if (f != ctx->seq_first.end()) {
            auto t = ctx->seq_tab.find(f->second);
            if (t != ctx->seq_tab.end() && t->second.inert > 0) {
                // nothing to decide for this signature for a while: run it untracked (no
                // bookkeeping on its launches or at its fcl_finish)
                t->second.inert -= 1;
                c.ok = false;
                c.keys.push_back(k);
                return false;
            }
            if (t != ctx->seq_tab.end()) {
                const auto &e = t->second;
                c.run = e.trial > 0 ? e.trial_kind : e.choice;
                c.trial = e.trial > 0;
                c.plan = f->second;
                c.plan_keys = &e.keys;
            }
        }
    }
    c.keys.push_back(k);
    for (int64_t v : k) c.h = (c.h ^ (uint64_t)v) * 1099511628211ull;   // FNV-1a over the keys
    c.work += host_madds(L);
    if (c.run != 1) {   // (the host-alone estimate is recorded for default sequences only)
        const auto se = ctx->sel.find(k9);
        const double r = se == ctx->sel.end() ? -1.0 : se->second.host_ms_per_wg;
        c.est = (c.est < 0 || r < 0) ? -1.0 : c.est + r * (double)(L.hi - L.lo);
    }
    if (c.run == 1) {
        if (c.plan_keys && pos < c.plan_keys->size() && (*c.plan_keys)[pos] == k) return true;
        c.ok = false;   // off the planned signature: the rest runs by per-launch selection
        c.run = -1;
    }
    return false;
}

// Called at the end of a successful fcl_finish.
void seq_end(fcl_context ctx) {
    auto &c = ctx->seq;
    if (!ctx->seq_on) return;
    const bool record = c.ok && !c.keys.empty();
    if (record) {
        const double wall = now_ms() - c.t0;
        std::lock_guard<std::mutex> lk(ctx->sel_mu);
        auto &e = ctx->seq_tab[c.h];
        if (e.keys.empty()) {
            e.keys = c.keys;
            ctx->seq_first[c.keys[0]] = c.h;
        }
        const int kind = c.run == 1 ? 1 : 0;
        // a sequence run as the other kind than planned (none: the first of its signature)
        double *ring = e.t_run[kind];
        for (int q = 3; q > 0; --q) ring[q] = ring[q - 1];
        ring[0] = wall;
        e.n_run[kind] = std::min(4, e.n_run[kind] + 1);
        if (kind == 0) e.est_host = c.est;
        e.work = c.work;
        e.seqs += 1;
        if (ctx->seq_debug)
            fprintf(stderr, "[fcl seq] sig %016llx n %zu run %d trial %d wall %.4f est %.4f work %.3g choice %d seqs %lld next %lld\n",
                    (unsigned long long)c.h, c.keys.size(), c.run, (int)c.trial, wall, c.est, c.work, e.choice, (long long)e.seqs,
                    (long long)e.next_trial);
        // a host trial whose two best sequences are both far slower than the default ends at once
        if (c.trial && e.trial > 0 && kind == 1 && e.n_run[0] > 0 && e.n_run[1] >= 2 &&
            std::max(e.t_run[1][0], e.t_run[1][1]) > 4.0 * seq_best(e.t_run[0], e.n_run[0]))
            e.trial = 1;
        if (c.trial && e.trial > 0) {
            if (--e.trial == 0) {
                const double d = seq_best(e.t_run[0], e.n_run[0]), h = seq_best(e.t_run[1], e.n_run[1]);
                const int win = (e.n_run[1] > 0 && e.n_run[0] > 0 && h < d) ? 1 : 0;
                if (win == e.choice && win == 0) {
                    e.loss_period = std::min<int64_t>(4096, e.loss_period * 8);
                    e.next_trial = e.seqs + e.loss_period;
                } else if (win == e.choice) {
                    e.period = std::min<int64_t>(1024, e.period * 2);
                    e.next_trial = e.seqs + e.period;
                } else {
                    // a new choice is re-checked after 64 sequences, then 128, ... 1024 while it
                    // holds (each re-check costs one sequence run the other way)
                    e.choice = win;
                    e.period = 64;
                    e.next_trial = e.seqs + e.period;
                }
            }
        } else if (e.trial == 0 && e.seqs >= e.next_trial) {
            const int other = 1 - e.choice;
            const double d = seq_best(e.t_run[0], e.n_run[0]);
            // the host alone is tried when the probes' best host rates predict it faster (2DCONV:
            // 21 ms predicted against 14.6 cooperative -- no trial), or -- no rate (the host
            // completed no chunk before the GPU was done) -- when the sequence is small (at most
            // 2^20 multiply-adds: well under a millisecond on the host)
            const bool worth = e.est_host >= 0 ? e.est_host <= d : e.work <= (double)(1 << 20);
            if (other == 1 && !worth) {
                e.next_trial = e.seqs + e.loss_period;   // the host cannot come close: do not try
            } else {
                e.trial = other == 1 ? 3 : 1;   // (a default re-check is one sequence: its last four stand)
                e.trial_kind = other;
                ctx->counts[FCL_COUNT_SEQ_TRIALS] += 1;
            }
        }
        // a default signature whose host alone is not worth a trial (no rate and not small, or a
        // predicted loss) runs its next 255 sequences untracked
        if (e.trial == 0 && e.choice == 0 && kind == 0) {
            const double d = seq_best(e.t_run[0], e.n_run[0]);
            const bool worth = e.est_host >= 0 ? e.est_host <= d : e.work <= (double)(1 << 20);
            if (!worth) e.inert = 255;
        }
    }
    c.keys.clear();
    c.ok = true;
    c.run = -1;
    c.trial = false;
}

unsigned long long *plain_stamp(fcl_context ctx) {
    if (!ctx->dpstamp || ctx->pst_n >= fcl_context_st::kPlainStamps) return nullptr;
    return ctx->dpstamp + 2 * ctx->pst_n++;
}

// PDL mode of the next plain grid on main (see fcl_context_st::pdl_chain).
int pdl_mode_impl(fcl_context ctx, const Launch &L);
int pdl_mode(fcl_context ctx, const Launch &L) {
    const int m = pdl_mode_impl(ctx, L);
    ctx->tr.add(m == PDL_OFF ? "pdl_off" : (m == PDL_WAIT ? "pdl_wait" : "pdl_nowait"), ctx->epoch);
    return m;
}
int pdl_mode_impl(fcl_context ctx, const Launch &L) {
    if (!ctx->pdl) return PDL_OFF;
    auto &ch = ctx->pdl_chain;
    if (ctx->main_fenced.exchange(0)) {   // an ordinary launch: it waits for everything before it
        ch.clear();
        ctx->pdl_chain_grids = 1;
        for (int a = 0; a < L.a.nbuf; ++a) ch.push_back({L.bufs[a], L.acc[a]});
        return PDL_OFF;
    }
    // at most 8 grids per chain: a grid can only be in flight together with the grids since the
    // last waiting one, which keeps the 16-entry write-through counter ring safe
    bool dep = ctx->pdl_chain_grids >= 8;
    for (int a = 0; a < L.a.nbuf && !dep; ++a)
        for (const auto &e : ch)
            if (e.b == L.bufs[a] && ((e.acc | L.acc[a]) & 2)) { dep = true; break; }
    if (dep) { ch.clear(); ctx->pdl_chain_grids = 0; }
    for (int a = 0; a < L.a.nbuf; ++a) ch.push_back({L.bufs[a], L.acc[a]});
    ctx->pdl_chain_grids += 1;
    return dep ? PDL_WAIT : PDL_NOWAIT;
}

Job *job_alloc(fcl_context ctx) {
    Job *j = nullptr;
    {
        std::lock_guard<std::mutex> lk(ctx->q_mu);
        if (!ctx->free_jobs.empty()) { j = ctx->free_jobs.back(); ctx->free_jobs.pop_back(); }
    }
    if (!j) {
        j = new Job();
        for (cudaEvent_t *pe : {&j->ev_k0, &j->ev_t1, &j->ev_m0, &j->ev_m1})
            if (cudaEventCreate(pe) != cudaSuccess) { cudaGetLastError(); return nullptr; }
        for (cudaEvent_t *pe : {&j->ev_start, &j->ev_k1, &j->ev_staged, &j->ev_ret, &j->ev_wm, &j->ev_d2h})
            if (cudaEventCreateWithFlags(pe, cudaEventDisableTiming) != cudaSuccess) { cudaGetLastError(); return nullptr; }
    }
    j->status = FCL_SUCCESS;
    j->done.store(0);
    j->kind = Job::JOB_COOP;
    j->host_seq = j->ticket = 0;
    j->nx = 0;
    j->have_k = j->have_m = j->wm_pending = false;
    j->gpu_launched = j->dev_merge = j->eager = j->forced = j->twin_alias = j->lite = j->exact_spans = false;
    j->lazy = false;
    j->stream = false;
    j->nstream = 0;
    j->unit = 1;
    std::memset(&j->info, 0, sizeof j->info);
    for (int q = 0; q < 6; ++q) j->twin[q] = j->stage[q] = nullptr;
    return j;
}

void job_release_buffers(fcl_context ctx, Job &j, bool staged) {
    if (staged) { ctx->hd_used.store(1, std::memory_order_relaxed); cudaEventRecord(ctx->ev_hd_release, ctx->hd); }
    for (int q = 0; q < j.L.nout; ++q) {
        if (j.twin[q]) pool_put(ctx, j.twin[q], staged);
        if (j.stage[q]) pool_put(ctx, j.stage[q], staged);
        j.twin[q] = j.stage[q] = nullptr;
    }
}

// ------------------------------------------------------------------------------------------
// Phase A (calling thread): everything the GPU does for a cooperative launch is queued here.
// ------------------------------------------------------------------------------------------
fcl_status coop_phase_a(fcl_context ctx, Job &j) {
    Launch &L = j.L;
    fcl_launch_info &info = j.info;
    const TaskSpace ts = gpu_task_space(L.a, L.g);
    j.t0 = first_task_at(L.a, L.g, ts.ntasks, L.lo);
    j.t1 = first_task_at(L.a, L.g, ts.ntasks, L.hi);
    info.gpu_tasks_total = j.t1 - j.t0;
    info.gpu_tasks = -1;
    j.forced = L.o.forced_split >= 0;
    j.s_forced = j.forced ? std::min<int64_t>(std::max<int64_t>(L.o.forced_split, L.lo), L.hi) : -1;
    constexpr int kSlots = fcl_context_st::kSlots;

    // a new kernel id (C14); stale status words are ignored by the dispatcher
    ctx->epoch += 1;
    j.epoch = ctx->epoch;
    j.slot = (int)(j.epoch % kSlots);
    if (ctx->slot_used[j.slot]) {
        // the dispatcher that used this status slot 16 launches ago must have finished
        const uint32_t prev = j.epoch - kSlots;
        while (__atomic_load_n(ctx->exit_host + j.slot, __ATOMIC_ACQUIRE) < prev &&
               ctx->main_done_epoch.load(std::memory_order_acquire) - prev >= 0x80000000u) {
            const cudaError_t q = cudaStreamQuery(ctx->main);
            if (q == cudaSuccess) break;
            if (q != cudaErrorNotReady) return cuda_fail(ctx, q, "slot reuse");
            _mm_pause();
        }
    }
    // main-stream position before this launch: this job's first staging copy (and the pieces
    // of streamed inputs) wait for it, so no pool buffer or input is overwritten while an
    // earlier kernel still reads it.  Always this job's own event: the previous dispatcher's
    // end event (used here before) belongs to a job that can be recycled and re-recorded --
    // behind this launch's own grid, or a later one -- while this launch still waits on it;
    // with streamed inputs that made the grid wait for pieces that waited for the grid.

    // Host chunk boundaries are aligned to the output span unit (1 work-group for 1-D kernels,
    // one work-group row for 2-D row-major ones).  The staged spans are then exactly the host's
    // footprint, and the only words the GPU can have written inside a merge domain are its own
    // redundant (bit-identical) copies of host work-groups, so the device copy itself is a
    // valid twin.  A twin is captured only when the footprint is not one span
    // (CORR symmat: a row plus a column) or a forced split point is not span-aligned.
    {
        long long uw = 0, ub = 0, tot = 0;
        bool contiguous = true;
        for (int q = 0; q < L.nout; ++q) {
            out_span_desc(L.a, L.g, L.out_idx[q], &uw, &ub, &tot);
            if (uw <= 0) contiguous = false;
            else j.unit = std::max<int64_t>(j.unit, uw);
        }
        const bool aligned_split = !j.forced || j.s_forced % j.unit == 0 || j.s_forced == L.hi;
        j.twin_alias = contiguous && aligned_split && !ctx->force_twin;
        j.exact_spans = contiguous;
    }
    // Single wave without in-task polls: every CTA runs exactly one task, unchecked (the first
    // task of a CTA never waits for the status), so no work-group can be skipped or aborted,
    // the GPU computes the whole range and no merge can be needed.  The dispatcher reduces to
    // the plain grid plus the exit signal, without status loads or arrival tail, and the host
    // neither stages nor publishes: its finished chunks only bound the return copy.
    int opt_period = L.o.abort_period;
    if (opt_period == 0 && ctx->env_abort_period != 0) opt_period = ctx->env_abort_period;   // FCL_ABORT_PERIOD
    const int abort_period = opt_period > 0 ? opt_period : (opt_period < 0 ? 0 : gpu_default_abort_period(L.a));
    j.lite = (j.t1 > j.t0) && !j.forced && !L.o.defer_merge && abort_period == 0 && !ctx->no_lite && !j.stream &&
             L.o.gpu_delay_us <= 0 &&
             (j.t1 - j.t0) <= gpu_coop_capacity(L.a, L.g, ctx->num_sms);
    // (a lite launch neither stages nor streams: nothing on hd waits for this position)
    if (!j.lite) CK(ctx, cudaEventRecord(j.ev_start, ctx->main));
    j.main_before = j.lite ? nullptr : j.ev_start;
    // twin (original data) and stage (CPU results) per OUT/INOUT buffer (C5, L16.s2-3)
    const void *srcs[6];
    size_t nbytes[6];
    bool hd_wait = false;
    if (j.lite) j.twin_alias = true;   // no twin and no stage
    for (int q = 0; q < L.nout && !j.lite; ++q) {
        fcl_buffer b = L.bufs[L.out_idx[q]];
        if (!j.twin_alias) j.twin[q] = pool_get(ctx, b->bytes, &hd_wait);
        j.stage[q] = pool_get(ctx, b->bytes, &hd_wait);
        if ((!j.twin_alias && !j.twin[q]) || !j.stage[q]) {
            job_release_buffers(ctx, j, false);
            return set_err(ctx, FCL_OUT_OF_RESOURCES, "twin/stage allocation of %zu bytes failed", b->bytes);
        }
        srcs[q] = b->dev;
        nbytes[q] = b->bytes;
    }
    ctx->tr.add("A_pool", j.epoch);
    if (hd_wait) {
        CK(ctx, cudaStreamWaitEvent(ctx->main, ctx->ev_hd_release, 0));
        ctx->main_fenced.store(1);
    }
    if (!j.twin_alias) {
        if (gpu_launch_copies(L.nout, j.twin, srcs, nbytes, ctx->num_sms, ctx->main) < 0) {
            for (int q = 0; q < L.nout; ++q)   // unaligned caller memory: per-buffer copies
                CK(ctx, cudaMemcpyAsync(j.twin[q], srcs[q], nbytes[q], cudaMemcpyDeviceToDevice, ctx->main));
        } else {
            info.gpu_launches += 1;
        }
    }

    if (j.forced) {
        // test hook: the GPU is told the split before it starts
        ctx->hd_used.store(1, std::memory_order_relaxed);
        CK(ctx, cudaStreamWaitEvent(ctx->hd, j.main_before, 0));
        fcl_status st = publish(ctx, j, (uint32_t)j.s_forced);
        if (st != FCL_SUCCESS) return st;
        CK(ctx, cudaEventRecord(j.ev_staged, ctx->hd));
        CK(ctx, cudaStreamWaitEvent(ctx->main, j.ev_staged, 0));
        ctx->main_fenced.store(1);
    }

    // GPU: the whole range, persistent dispatcher (C8)
    CoopCtl c;
    c.status = ctx->status_dptr + j.slot;
    c.epoch = j.epoch;
    c.w_default = (unsigned int)L.hi;
    c.claim = ctx->dclaim + j.slot;
    c.claim_next = ctx->dclaim + (j.slot + 1) % kSlots;
    c.tasks = ctx->stats ? ctx->dtasks + j.slot : nullptr;
    c.tasks_next = ctx->stats ? ctx->dtasks + (j.slot + 1) % kSlots : nullptr;
    c.wm_out = ctx->dwm;
    c.check_first = j.forced ? 1 : 0;
    c.status_mapped = ctx->status_location == FCL_STATUS_HOST_MAPPED ? 1 : 0;
    c.tstamp = ctx->stats ? ctx->dstamp + 4 * j.slot : nullptr;
    c.tstamp_next = ctx->stats ? ctx->dstamp + 4 * ((j.slot + 1) % kSlots) : nullptr;
    c.task_lo = j.t0; c.task_hi = j.t1;
    c.abort_period = abort_period;
    c.barrier = ctx->dbar + 32 * j.slot;
    c.barrier_next = ctx->dbar + 32 * ((j.slot + 1) % kSlots);
    c.merge_ctr = ctx->dmctr + j.slot;
    c.merge_ctr_next = ctx->dmctr + (j.slot + 1) % kSlots;
    c.exit_word = ctx->exit_dptr + j.slot;
    c.arrival = j.stream ? ctx->darrival + j.slot : nullptr;
    c.task_delay_ns = L.o.gpu_delay_us > 0 ? 1000ull * (unsigned long long)L.o.gpu_delay_us : 0ull;
    c.exec_cnt = L.o.record_exec_counts ? ctx->rec.d_cnt : nullptr;
    c.exec_w = L.o.record_exec_counts ? ctx->rec.d_w : nullptr;
    c.mg = DevMergeList{};
    c.mg.n = 0;

    // Free-running mode: the merge decides its domain on the device from the watermark the
    // dispatcher acted on and runs in the dispatcher's fused tail (or right behind it), and
    // small outputs are returned eagerly behind it -- no host round trip between the GPU
    // finishing and the result being coherent.
    j.dev_merge = (j.t1 > j.t0) && !j.forced && !L.o.defer_merge && !j.lite;
    size_t out_total = 0;
    for (int q = 0; q < L.nout; ++q) {
        size_t b0, b1;
        out_span(L.a, L.g, L.out_idx[q], L.lo, L.hi, &b0, &b1);
        out_total += b1 - b0;
    }
    // An INOUT buffer is read-modify-written in place by the host bodies: its return copy
    // must wait until the host workers have stopped (an abandoned chunk may still be running
    // when the GPU finishes), so only pure-OUT launches return eagerly.
    j.eager = (j.dev_merge || j.lite) && !L.any_inout && out_total <= ctx->eager_return_bytes;
    DevMergeList M{};
    size_t maxb = 0;
    if (j.dev_merge) {
        M.n = L.nout;
        for (int q = 0; q < L.nout; ++q) {
            fcl_buffer b = L.bufs[L.out_idx[q]];
            M.gpu[q] = (unsigned char *)b->dev;
            M.cpu[q] = (const unsigned char *)j.stage[q];
            M.twin[q] = (const unsigned char *)(j.twin_alias ? b->dev : j.twin[q]);
            M.es[q] = (int)b->elem_size;
            out_span_desc(L.a, L.g, L.out_idx[q], &M.unit_wgs[q], &M.unit_bytes[q], &M.total[q]);
            maxb = std::max(maxb, (size_t)M.total[q]);
        }
        M.wm_word = ctx->dwm;
        M.epoch = j.epoch;
        M.hi = L.hi;
        M.tstamp = ctx->stats ? ctx->dstamp + 4 * j.slot + 2 : nullptr;
        M.exit_word = ctx->exit_dptr + j.slot;
    }
    M.wm_word = ctx->dwm;
    M.epoch = j.epoch;
    M.hi = L.hi;
    c.fused = ctx->unfused ? 0 : 1;
    if (ctx->test_publish_zero_us > 0) M.n = 0;   // (exit-drain measurement: no merge, see the context)
    if (c.fused) c.mg = M;   // mg.n == 0 (forced / deferred): barrier + exit signal only
    c.mg.tstamp = ctx->stats ? ctx->dstamp + 4 * j.slot + 2 : nullptr;

    if (j.t1 > j.t0) {
        const bool timing = ctx->ktiming || (L.o.flags & FCL_LAUNCH_TIMING);
        if (timing) CK(ctx, cudaEventRecord(j.ev_k0, ctx->main));
        ctx->tr.add("A_prelaunch", j.epoch);
        if (j.lite) {
            const int nx = (j.slot + 1) % kSlots;
            SlotReset r{ctx->dclaim + nx, ctx->stats ? ctx->dtasks + nx : nullptr, ctx->dmctr + nx, ctx->dbar + 32 * nx,
                        ctx->dbar + 32 * j.slot, ctx->lite_exit_word ? ctx->exit_dptr + j.slot : nullptr, j.epoch,
                        plain_stamp(ctx), ctx->test_gpu_delay_ns,
                        L.o.record_exec_counts ? ctx->rec.d_cnt : nullptr};
            if (gpu_launch_plain(L.a, L.g, j.t0, j.t1, ctx->main, &r, pdl_mode(ctx, L)) < 0)
                return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
        } else {
            if (gpu_launch_coop(L.a, L.g, c, ctx->num_sms, ctx->main) < 0)
                return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
            ctx->pdl_chain.clear();   // an ordinary launch that never triggers early: the next
            ctx->pdl_chain_grids = 0;
                                      // grid starts after it (and everything before it) completed
        }
        ctx->tr.add("A_launched", j.epoch);
        if (timing) CK(ctx, cudaEventRecord(j.ev_t1, ctx->main));
        CK(ctx, cudaEventRecord(j.ev_k1, ctx->main));
        ctx->tr.add("A_k1", j.epoch);
        // GPU exit signal for the host executor (L18.s19): the fused tail (or, lite, the plain
        // grid's last CTA) stores the epoch to mapped host memory; unfused, a bare memop does it.
        if (!c.fused && !j.lite) {
            fcl_status xs = stream_store(ctx, ctx->exit_dptr + j.slot, (unsigned long long)j.epoch, ctx->main, false, &info);
            if (xs != FCL_SUCCESS) return xs;
        }
        // (a lite grid without an exit word uses nothing of its slot; a later launch of the
        // slot must not wait for a word it never stores)
        ctx->slot_used[j.slot] = !j.lite || ctx->lite_exit_word;
        ctx->main_tail = j.ev_k1;
        info.gpu_path = j.lite ? FCL_GPU_PATH_LITE : FCL_GPU_PATH_DISPATCHER;
        j.have_k = timing;
        info.gpu_launches += 1;
        j.gpu_launched = true;
    } else {
        // no dispatcher: reset the next launch's counters here
        CK(ctx, cudaMemsetAsync(ctx->dclaim + (j.slot + 1) % kSlots, 0, 8, ctx->main));
        CK(ctx, cudaMemsetAsync(ctx->dtasks + (j.slot + 1) % kSlots, 0, 8, ctx->main));
        CK(ctx, cudaMemsetAsync(ctx->dbar + 32 * ((j.slot + 1) % kSlots), 0, 128, ctx->main));
        CK(ctx, cudaMemsetAsync(ctx->dmctr + (j.slot + 1) % kSlots, 0, 8, ctx->main));
        ctx->main_tail = nullptr;
    }
    if (j.dev_merge && !c.fused) {
        if (gpu_launch_merge_dev(M, maxb, ctx->num_sms, ctx->main) < 0)
            return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
        info.gpu_launches += 1;
    }
    // Small pure-OUT outputs of a free-running launch return lazily (the device copy is
    // complete once the grid -- with its fused merge -- is; the return copies the whole span,
    // so host words an abandoned chunk of this launch wrote are overwritten with the same bits)
    if (j.eager && lazy_return(ctx, L, info)) { j.eager = false; j.lazy = true; }
    if (j.eager) {
        cudaEvent_t mark = j.ev_k1;
        if (!c.fused && !j.lite) { CK(ctx, cudaEventRecord(j.ev_ret, ctx->main)); mark = j.ev_ret; }
        fcl_status st = enqueue_d2h(ctx, L, L.lo, L.hi, info, mark);
        if (st != FCL_SUCCESS) return st;
    }
    return FCL_SUCCESS;
}

// ------------------------------------------------------------------------------------------
// Phase B (coordinator thread): descending adaptive chunks on the host (C9-C11), staged and
// published after each (C13), until the GPU exits or the host covers the range.
// ------------------------------------------------------------------------------------------
fcl_status coop_phase_b(fcl_context ctx, Job &j) {
    Launch &L = j.L;
    Executor &ex = ctx->ex;
    fcl_launch_info &info = j.info;
    // host copies of every argument must be current (pending returns of earlier launches)
    for (int k = 0; k < L.a.nbuf; ++k) {
        fcl_buffer b = L.bufs[k];
        // (the outputs of an eager / lazy launch are excluded before their state is read: the
        // API thread may be queueing their lazy return for a later launch right now)
        if (!((j.eager || j.lazy) && (L.acc[k] & 2)) && d2h_busy(ctx, b)) {
            CK(ctx, cudaEventSynchronize(b->d2h_ev));
        }
    }
    const int64_t nwg = L.hi - L.lo;
    const int nact = L.o.n_host_threads > 0 ? std::min(L.o.n_host_threads, ex.T) : ex.T;
    const int64_t lo_cpu = j.forced ? j.s_forced : L.lo;
    int64_t hi_cur = L.hi;
    int pct = std::max(1, L.o.init_chunk_pct);
    double prev_avg = -1.0, t_start = 0.0, busy = 0.0;
    int nch = 0;
    VariantPick vp = pick_variant(ctx, L);
    int cur_var = vp.var;
    bool in_flight = false, gpu_done = !j.gpu_launched, cpu_all = false, staged_any = false, hd_joined = false;
    int64_t cur_lo = 0, cur_hi = 0, cur_size = 0, cpu_done_wgs = 0;
    // The GPU may finish before the host side can start (a launch queued behind a busy
    // coordinator, or the pool still stopping an earlier launch's abandoned chunk -- which can
    // take a scheduler quantum when a worker thread has been preempted): then no chunk is
    // started at all, and the abandoned chunk is left to stop on its own.
    const bool event_exit = j.lite && !ctx->lite_exit_word;   // no exit word: the event (or finish) tells
    const unsigned qmask = event_exit ? ctx->lite_query_mask : ctx->exit_query_mask;
    auto exit_word_seen = [&]() {
        return __atomic_load_n(ctx->exit_host + j.slot, __ATOMIC_ACQUIRE) >= (unsigned long long)j.epoch ||
               ctx->main_done_epoch.load(std::memory_order_acquire) - j.epoch < 0x80000000u;
    };
    unsigned spin = 0;
    auto gpu_exited = [&]() {
        return !j.forced && j.gpu_launched &&
               (exit_word_seen() || (event_exit && (++spin & qmask) == 0 && cudaEventQuery(j.ev_k1) == cudaSuccess));
    };
    bool exited_before = gpu_exited();
    while (!exited_before && !quiesce_try(ctx)) {   // the pool must be idle before ours starts
        for (int k = 0; k < ctx->exit_poll_pauses; ++k) _mm_pause();
        exited_before = gpu_exited();
    }

    if (ctx->test_publish_zero_us > 0 && j.dev_merge && !exited_before) {
        // exit-drain measurement: publish W = lo after the given time, compute nothing
        std::this_thread::sleep_for(std::chrono::microseconds(ctx->test_publish_zero_us));
        ctx->hd_used.store(1, std::memory_order_relaxed);
        CK(ctx, cudaStreamWaitEvent(ctx->hd, j.main_before, 0));
        if (gpu_launch_store64(ctx->status_dptr + j.slot, ((unsigned long long)j.epoch << 32) | (uint32_t)L.lo, ctx->hd,
                               ctx->dpub + j.slot) < 0)
            return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
        while (!exit_word_seen()) _mm_pause();
        info.published_watermark = L.lo;
        j.wm_pending = true;
        job_release_buffers(ctx, j, true);
        return FCL_SUCCESS;
    }
    auto start_chunk = [&]() {
        int64_t size = ceil_pct(pct, nwg);
        const int64_t min_units = L.o.cpu_wg_split ? 1 : nact;   // L18.s31 without C23
        size = std::max<int64_t>(size, min_units);
        if (j.twin_alias) size = (size + j.unit - 1) / j.unit * j.unit;   // span-aligned chunks
        size = std::min<int64_t>(size, hi_cur - lo_cpu);
        cur_hi = hi_cur; cur_lo = hi_cur - size; cur_size = size;
        const int parts = (L.o.cpu_wg_split && size < nact) ? (int)((nact + size - 1) / size) : 1;
        if (L.o.host_delay_us > 0) std::this_thread::sleep_for(std::chrono::microseconds(L.o.host_delay_us));
        if (nch < 64) info.chunk_sizes[nch] = (int32_t)size;
        ++nch;
        t_start = now_ms();
        KArgs ka = L.a;
        ka.host_variant = cur_var = chunk_variant(vp);
        ex.submit(ka, L.g, cur_lo, cur_hi, parts, nact);
        in_flight = true;
    };
    auto stage_chunk = [&](int64_t clo, int64_t chi) -> fcl_status {
        if (j.lite) {   // the GPU computes everything: the finished chunk only bounds the return
            info.published_watermark = clo;
            return FCL_SUCCESS;
        }
        ctx->hd_used.store(1, std::memory_order_relaxed);
        if (!hd_joined) {
            CK(ctx, cudaStreamWaitEvent(ctx->hd, j.main_before, 0));
            hd_joined = true;
        }
        for (int q = 0; q < L.nout; ++q) {
            fcl_buffer b = L.bufs[L.out_idx[q]];
            size_t b0, b1;
            out_span(L.a, L.g, L.out_idx[q], clo, chi, &b0, &b1);
            if (b1 > b0) {
                CK(ctx, cudaMemcpyAsync((char *)j.stage[q] + b0, (char *)b->host + b0, b1 - b0, cudaMemcpyHostToDevice, ctx->hd));
                ctx->counts[FCL_COUNT_H2D_BYTES] += (int64_t)(b1 - b0);
                info.h2d_bytes += (int64_t)(b1 - b0);
            }
        }
        if (!j.forced && !L.o.drop_publish) {
            fcl_status st = publish(ctx, j, (uint32_t)clo);
            if (st != FCL_SUCCESS) return st;
        }
        CK(ctx, cudaEventRecord(j.ev_staged, ctx->hd));
        staged_any = true;
        info.published_watermark = clo;
        return FCL_SUCCESS;
    };

    // Streamed inputs (§6.7): row pieces of the stale matrices in ascending work-group order on
    // hd, each followed by the arrival front (a stream memop), never beyond the host's frontier
    // (the work-groups it has taken), at most two pieces outstanding.
    int64_t s_sent = L.lo;
    int s_head = 0, s_out = 0;
    unsigned s_spin = 0;
    int64_t s_piece = 1;
    if (j.stream) {
        size_t per_wg = 0;
        for (int q = 0; q < j.nstream; ++q) per_wg += (size_t)L.g.lws[0] * (size_t)L.a.n1 * L.bufs[j.sbuf[q]]->elem_size;
        s_piece = std::max<int64_t>(1, (int64_t)(ctx->stream_piece_bytes / std::max<size_t>(1, per_wg)));
    }
    auto pump = [&]() -> fcl_status {
        if (!j.stream || gpu_done) return FCL_SUCCESS;
        if (s_out > 0 && ((++s_spin & 15) == 0 || s_out >= 2)) {
            while (s_out > 0) {
                const cudaError_t q = cudaEventQuery(ctx->stream_ev[s_head & 3]);
                if (q == cudaErrorNotReady) break;
                if (q != cudaSuccess) return cuda_fail(ctx, q, "stream piece");
                ++s_head; --s_out;
            }
        }
        const int64_t frontier = in_flight ? cur_lo : hi_cur;
        while (s_out < 2 && s_sent < frontier) {
            const int64_t hi = std::min<int64_t>(s_sent + s_piece, frontier);
            ctx->hd_used.store(1, std::memory_order_relaxed);
            if (!hd_joined) {   // behind every earlier kernel that may still read the old device copy
                CK(ctx, cudaStreamWaitEvent(ctx->hd, j.main_before, 0));
                hd_joined = true;
            }
            const int64_t r0 = s_sent * L.g.lws[0], r1 = std::min<int64_t>(hi * L.g.lws[0], L.a.n0);
            for (int q = 0; q < j.nstream && r1 > r0; ++q) {
                fcl_buffer b = L.bufs[j.sbuf[q]];
                const size_t rb = (size_t)L.a.n1 * b->elem_size;
                CK(ctx, cudaMemcpyAsync((char *)b->dev + (size_t)r0 * rb, (char *)b->host + (size_t)r0 * rb,
                                        (size_t)(r1 - r0) * rb, cudaMemcpyHostToDevice, ctx->hd));
                ctx->counts[FCL_COUNT_H2D_BYTES] += (int64_t)((size_t)(r1 - r0) * rb);
                info.h2d_bytes += (int64_t)((size_t)(r1 - r0) * rb);
            }
            fcl_status st = stream_store(ctx, ctx->darrival + j.slot, ((unsigned long long)j.epoch << 32) | (uint32_t)hi,
                                         ctx->hd, true, &info);
            if (st != FCL_SUCCESS) return st;
            CK(ctx, cudaEventRecord(ctx->stream_ev[(s_head + s_out) & 3], ctx->hd));
            ++s_out;
            s_sent = hi;
            info.streamed_wgs = s_sent - L.lo;
        }
        return FCL_SUCCESS;
    };

    info.published_watermark = L.hi;
    if (exited_before) {
        gpu_done = true;
        ctx->tr.add("gpu_exit_seen", j.epoch);
    } else if (hi_cur > lo_cpu) {
        start_chunk();
    } else {
        cpu_all = true;
    }
    {
        fcl_status st = pump();
        if (st != FCL_SUCCESS) { ex.abort_flag = 1; ex.wait(); return st; }
    }
    while (in_flight) {
        {
            fcl_status st = pump();
            if (st != FCL_SUCCESS) { ex.abort_flag = 1; ex.wait(); return st; }
        }
        if (!j.forced && !gpu_done && j.gpu_launched && exit_word_seen()) {
            gpu_done = true;   // GPU exit (L18.s19)
            ctx->tr.add("gpu_exit_seen", j.epoch);
            break;
        }
        if ((++spin & qmask) == 0 && j.gpu_launched) {   // a failed dispatcher never signals
            const cudaError_t q = cudaEventQuery(j.ev_k1);
            if (q == cudaSuccess && event_exit) {   // (no exit word: the event is the signal)
                gpu_done = true;
                ctx->tr.add("gpu_exit_seen", j.epoch);
                break;
            }
            if (q != cudaSuccess && q != cudaErrorNotReady) { ex.abort_flag = 1; ex.wait(); return cuda_fail(ctx, q, "dispatcher"); }
        }
        if (ex.finished()) {
            const double dt = now_ms() - t_start;
            busy += dt;
            if (nch - 1 < 64) info.chunk_ms[nch - 1] = dt;   // (the C11 input, exported for its pin)
            in_flight = false;
            cpu_done_wgs += cur_size;
            variant_measured(ctx, L, vp, cur_var, dt, cur_size);
            const double avg = dt / (double)cur_size;
            if (nch == 1 || avg < prev_avg) pct += std::max(0, L.o.step_pct);   // C11
            prev_avg = avg;
            const int64_t clo = cur_lo, chi = cur_hi;
            hi_cur = clo;
            const bool more = hi_cur > lo_cpu;
            if (more) start_chunk();          // keep the workers busy while this chunk is staged
            fcl_status st = stage_chunk(clo, chi);
            if (st != FCL_SUCCESS) { ex.abort_flag = 1; ex.wait(); return st; }
            if (!more) { cpu_all = true; break; }
        } else {
            // back off between polls: the exit word is written by the GPU over PCIe, and a core
            // hammering that line slows the device's posted writes (and the return copies queued
            // behind them)
            for (int k = 0; k < ctx->exit_poll_pauses; ++k) _mm_pause();
        }
    }
    // Return race: the GPU finished first (its copy is complete: it ran every work-group it did
    // not skip, and the skipped ones were merged in its tail), but the host still needs the
    // device's results below its own frontier hi_cur.  Instead of abandoning the running chunk
    // and copying everything, the result comes back in ascending pieces on dh while the host
    // goes on computing chunks from the top; the two meet in the middle.  A piece never
    // overlaps a running chunk (INOUT outputs are updated in place on the host); when the copy
    // front reaches the running chunk, that chunk is abandoned and its range copied too.
    auto out_bytes = [&](int64_t a, int64_t b) -> size_t {
        size_t t = 0;
        for (int q = 0; q < L.nout; ++q) {
            size_t b0, b1;
            out_span(L.a, L.g, L.out_idx[q], a, b, &b0, &b1);
            t += b1 - b0;
        }
        return t;
    };
    // (only for exact spans: a piece of work-groups must map to its own bytes, not to a
    // conservative cover such as CORR's row-plus-column symmat footprint)
    const bool race = gpu_done && !j.forced && (j.dev_merge || j.lite) && !j.eager && !j.lazy && !ctx->no_race && j.exact_spans &&
                      hi_cur > L.lo && out_bytes(L.lo, hi_cur) >= ctx->race_min_bytes;
    info.n_c11_chunks = nch;
    if (race) {
        ctx->tr.add("race_begin", j.epoch);
        info.race = 1;
        quiesce(ctx);   // an earlier launch's abandoned chunk may still read a host copy written below
        ctx->dr_used.store(1, std::memory_order_relaxed);
        CK(ctx, cudaStreamWaitEvent(ctx->dr, j.ev_k1, 0));
        for (int q = 0; q < L.nout; ++q) {   // behind any earlier return of the same buffers
            fcl_buffer ob = L.bufs[L.out_idx[q]];
            if (d2h_busy(ctx, ob) && !ob->d2h_on_main) CK(ctx, cudaStreamWaitEvent(ctx->dr, ob->d2h_ev, 0));
        }
        const size_t unit_b = std::max<size_t>(1, out_bytes(L.lo, std::min<int64_t>(L.lo + j.unit, L.hi)));
        const int64_t piece = j.unit * std::max<int64_t>(1, (int64_t)(ctx->race_piece_bytes / unit_b));
        int64_t F = L.lo;   // end of the prefix whose return is queued
        int qh = 0, qn = 0;
        auto race_chunk = [&]() {
            // never while an abandoned chunk of an earlier launch may still run (the GPU may have
            // finished before this host side started, so the pool was never quiesced)
            if (!quiesce_try(ctx)) return;
            const double per_wg = cpu_done_wgs > 0 ? busy / (double)cpu_done_wgs : -1.0;
            int64_t size = per_wg > 0 ? (int64_t)(ctx->race_chunk_ms / per_wg) : ceil_pct(pct, nwg);
            size = std::max<int64_t>(size, nact);
            size = (size + j.unit - 1) / j.unit * j.unit;
            const int64_t room = (hi_cur - (F + piece)) / j.unit * j.unit;   // leave the next piece alone
            if (room < j.unit) return;
            size = std::min(size, room);
            cur_hi = hi_cur; cur_lo = hi_cur - size; cur_size = size;
            if (nch < 64) info.chunk_sizes[nch] = (int32_t)size;
            ++nch;
            t_start = now_ms();
            KArgs ka = L.a;
            ka.host_variant = cur_var = chunk_variant(vp);
            ex.submit(ka, L.g, cur_lo, cur_hi, 1, nact);
            in_flight = true;
        };
        for (;;) {
            if (in_flight && ex.finished()) {
                busy += now_ms() - t_start;
                if (nch - 1 < 64) info.chunk_ms[nch - 1] = now_ms() - t_start;
                in_flight = false;
                cpu_done_wgs += cur_size;
                hi_cur = cur_lo;
                info.published_watermark = hi_cur;   // the host's frontier
                race_chunk();
            }
            const int64_t limit = in_flight ? cur_lo : hi_cur;
            if (F >= limit) {
                if (!in_flight) break;   // everything below the host's frontier is on its way
                ex.abort_flag = 1;       // the copy front reached the running chunk
                ex.wait();
                busy += now_ms() - t_start;
                ex.abort_flag = 0;
                in_flight = false;
                continue;
            }
            if (qn < 2) {
                const int64_t b = std::min<int64_t>(F + piece, limit);
                for (int q = 0; q < L.nout; ++q) {
                    fcl_buffer ob = L.bufs[L.out_idx[q]];
                    size_t b0, b1;
                    out_span(L.a, L.g, L.out_idx[q], F, b, &b0, &b1);
                    if (b1 <= b0) continue;
                    CK(ctx, cudaMemcpyAsync((char *)ob->host + b0, (char *)ob->dev + b0, b1 - b0, cudaMemcpyDeviceToHost, ctx->dr));
                    ctx->counts[FCL_COUNT_D2H_BYTES] += (int64_t)(b1 - b0);
                    info.d2h_bytes += (int64_t)(b1 - b0);
                }
                CK(ctx, cudaEventRecord(ctx->race_ev[(qh + qn) & 3], ctx->dr));
                ++qn;
                F = b;
            } else {
                const cudaError_t q = cudaEventQuery(ctx->race_ev[qh & 3]);
                if (q == cudaSuccess) { ++qh; --qn; }
                else if (q != cudaErrorNotReady) return cuda_fail(ctx, q, "return race");
                else for (int k = 0; k < 64; ++k) _mm_pause();
            }
        }
        for (int q = 0; q < L.nout; ++q) {   // the buffers' return events follow the last piece
            fcl_buffer ob = L.bufs[L.out_idx[q]];
            CK(ctx, cudaEventRecord(ob->d2h_ev, ctx->dr));
            ob->d2h_pending = true; ob->d2h_on_main = false; ob->d2h_on_race = true; ob->d2h_gen = ctx->finish_gen.load();
        }
        ctx->tr.add("race_end", j.epoch);
    } else if (in_flight && (j.eager || j.lazy) && gpu_done) {
        // GPU finished first and the (pure-OUT) result is already on its way back: abandon the
        // chunk without waiting for it (L18.s19).  Its workers only write words bit-identical to
        // the returned ones; whatever could change what they read or write waits in quiesce().
        std::lock_guard<std::mutex> lk(ctx->qz_mu);
        ex.abort_flag = 1;
        ctx->qz_n = 0;
        for (int k = 0; k < L.a.nbuf; ++k) ctx->qz_bufs[ctx->qz_n++] = L.bufs[k];
        ctx->quiescing.store(1, std::memory_order_release);
        busy += now_ms() - t_start;
    } else if (in_flight) {   // GPU finished first: abandon the running chunk (L18.s19)
        ex.abort_flag = 1;
        ex.wait();
        busy += now_ms() - t_start;
        ex.abort_flag = 0;
    }
    if (j.stream && s_sent > L.lo) {   // up to two pieces may still be in flight on hd
        CK(ctx, cudaEventRecord(ctx->ev_stream_done, ctx->hd));
        ctx->stream_pending = true;
    }
    info.t_host_ms = busy;
    info.n_chunks = nch;
    variant_info(vp, info);
    if (nch == 0) info.host_variant = -1;
    info.cpu_wgs = cpu_done_wgs;
    info.gpu_watermark = L.hi;
    fcl_status st = FCL_SUCCESS;
    if (j.probe) select_update(ctx, j, gpu_done);

    if (j.dev_merge || j.lite) {
        // the merge is already queued (or, lite, cannot be needed); only the precise return
        // of large outputs is left
        if (gpu_done) {
            if (!j.eager && !j.lazy && !race) {
                // The host copy already holds every published chunk, and the GPU acted on some
                // watermark >= the lowest one published, so returning the device copy (merged
                // by the fused tail) below the host's own published watermark is complete --
                // no device read of the GPU's watermark on this path.
                quiesce(ctx);   // (an earlier launch's abandoned chunk may still read these host copies)
                st = enqueue_d2h(ctx, L, L.lo, info.published_watermark, info, j.ev_k1);
            }
            j.wm_pending = !j.lite;   // info.gpu_watermark resolved lazily by fcl_get_launch_info
        } else {
            info.cpu_did_all = 1;      // host authoritative (L16.s21); device merged behind
            info.gpu_watermark = j.lite ? L.hi : L.lo;   // lite: the GPU computes every work-group
            info.merged = j.lite ? 0 : 1;
        }
    } else {
        // Forced split / deferred merge: the host decides merge domain and return (C15/C17)
        int64_t merge_lo = L.hi;
        bool wait_staged = false;
        if (j.forced) {
            merge_lo = j.s_forced;
            wait_staged = staged_any;
        } else if (cpu_all && !gpu_done) {
            merge_lo = L.lo;
            wait_staged = staged_any;
        } else if (j.gpu_launched) {
            int64_t wm = L.hi;
            st = read_gpu_watermark(ctx, j, &wm);
            if (st != FCL_SUCCESS) return st;
            merge_lo = wm;
            wait_staged = staged_any && wm < L.hi;
        }
        if (merge_lo <= L.lo) info.cpu_did_all = 1;
        info.gpu_watermark = merge_lo;
        if (merge_lo < L.hi) {
            info.merged = 1;
            if (wait_staged) {
                CK(ctx, cudaStreamWaitEvent(ctx->main, j.ev_staged, 0));
                ctx->main_fenced.store(1);
            }
            st = enqueue_merges(ctx, j, merge_lo, L.hi);
            if (st != FCL_SUCCESS) return st;
        }
        if (L.o.defer_merge && merge_lo < L.hi) {
            for (int q = 0; q < L.nout; ++q) {   // the return copy must follow the deferred merge
                fcl_buffer b = L.bufs[L.out_idx[q]];
                out_span(L.a, L.g, L.out_idx[q], L.lo, merge_lo, &b->r_b0, &b->r_b1);
            }
        } else {
            CK(ctx, cudaEventRecord(j.ev_ret, ctx->main));   // after the host-side merges
            quiesce(ctx);
            st = enqueue_d2h(ctx, L, L.lo, merge_lo, info, j.ev_ret);
        }
    }
    job_release_buffers(ctx, j, staged_any);
    return st;
}

fcl_status run_cpu_only(fcl_context ctx, Launch &L, fcl_launch_info &info);

// A CPU-only launch in queue order (C22: the host side of every earlier launch has run): its
// inputs' host copies must hold the expected versions -- every return copy of an earlier launch
// has landed (the paper's CPU scheduler waits "until the most recent data arrives from the
// GPU", L20.s7) -- then the executor runs the whole range.
fcl_status cpu_job(fcl_context ctx, Job &j) {
    Launch &L = j.L;
    for (int k = 0; k < L.a.nbuf; ++k) {
        fcl_buffer b = L.bufs[k];
        if (d2h_busy(ctx, b)) {
            CK(ctx, cudaEventSynchronize(b->d2h_ev));
        }
    }
    if (L.o.host_delay_us > 0) std::this_thread::sleep_for(std::chrono::microseconds(L.o.host_delay_us));
    return run_cpu_only(ctx, L, j.info);
}

// Host->device copies of the host copies a pending CPU-only job produced, ordered after the GPU
// work queued before the launch that needs them (xt waits for that main-stream position), then
// the ticket: the launch's grid waits on the device until the ticket has landed (C18: "the GPU
// ... discarding stale data", here: never reading it).
fcl_status xfer_job(fcl_context ctx, Job &j) {
    ctx->xt_used.store(1, std::memory_order_relaxed);
    auto fail = [&](cudaError_t e, const char *what) {   // (the waiting grid must still be released)
        const fcl_status st = cuda_fail(ctx, e, what);
        stream_store(ctx, ctx->d_xfer, (unsigned long long)j.ticket, ctx->xt, false);
        return st;
    };
    cudaError_t e = cudaStreamWaitEvent(ctx->xt, j.ev_start, 0);
    if (e != cudaSuccess) return fail(e, "transfer wait");
    for (int q = 0; q < j.nx; ++q) {
        fcl_buffer b = j.xb[q];
        e = cudaMemcpyAsync(b->dev, b->host, b->bytes, cudaMemcpyHostToDevice, ctx->xt);
        if (e != cudaSuccess) return fail(e, "transfer copy");
        ctx->counts[FCL_COUNT_H2D_BYTES] += (int64_t)b->bytes;
        j.info.h2d_bytes += (int64_t)b->bytes;
    }
    return stream_store(ctx, ctx->d_xfer, (unsigned long long)j.ticket, ctx->xt, true, &j.info);
}

// ------------------------------------------------------------------------------------------
// Coordinator thread and the launch queue
// ------------------------------------------------------------------------------------------
void coordinator(fcl_context ctx) {
    cudaSetDevice(ctx->device);
    if (ctx->coord_core >= 0) {   // its own core: it spins on the GPU exit word and the workers
        cpu_set_t cs;
        CPU_ZERO(&cs);
        CPU_SET(ctx->coord_core, &cs);
        sched_setaffinity(0, sizeof cs, &cs);
    }
    for (;;) {
        Job *j = nullptr;
        // spin for work for a while (launches come in bursts), then sleep on the condvar
        auto t0 = Clock::now();
        while (ctx->q_len.load(std::memory_order_acquire) == 0 && !ctx->q_stop_flag.load(std::memory_order_relaxed)) {
            _mm_pause();
            if (std::chrono::duration_cast<std::chrono::nanoseconds>(Clock::now() - t0).count() > ctx->ex.spin_ns) {
                std::unique_lock<std::mutex> lk(ctx->q_mu);
                ctx->coord_sleeping.store(1);
                ctx->q_cv.wait(lk, [&] { return ctx->q_stop || !ctx->queue.empty(); });
                ctx->coord_sleeping.store(0);
                t0 = Clock::now();
            }
        }
        {
            std::lock_guard<std::mutex> lk(ctx->q_mu);
            if (ctx->queue.empty()) {
                if (ctx->q_stop) return;   // stop requested and nothing pending
                continue;
            }
            j = ctx->queue.front();
            ctx->running = j;
        }
        fcl_status st = FCL_SUCCESS;
        ctx->tr.add("phaseB_begin", j->epoch);
        if (ctx->sticky.load() != FCL_SUCCESS) {
            st = ctx->sticky.load();
            // a GPU launch waits on the device for this ticket: store it anyway (the context is
            // lost; the grid must still be able to finish so that the caller's sync returns)
            if (j->kind == Job::JOB_XFER) stream_store(ctx, ctx->d_xfer, (unsigned long long)j->ticket, ctx->xt, false);
        }
        else if (j->kind == Job::JOB_CPU) st = cpu_job(ctx, *j);
        else if (j->kind == Job::JOB_XFER) st = xfer_job(ctx, *j);
        else {
            st = coop_phase_b(ctx, *j);
            if (j->stream) ctx->stream_jobs.fetch_sub(1, std::memory_order_acq_rel);
        }
        if (j->kind == Job::JOB_CPU) ctx->host_done_seq.store(j->host_seq, std::memory_order_release);
        ctx->tr.add("phaseB_end", j->epoch);
        {
            std::lock_guard<std::mutex> lk(ctx->q_mu);
            j->status = st;
            if (st != FCL_SUCCESS && ctx->sticky.load() == FCL_SUCCESS) ctx->sticky = st;
            ctx->queue.erase(ctx->queue.begin());
            ctx->q_len.fetch_sub(1, std::memory_order_release);
            ctx->running = nullptr;
            j->done.store(1, std::memory_order_release);
            if (j != ctx->last) ctx->free_jobs.push_back(j);
        }
        if (ctx->drain_sleeping.load()) ctx->q_cv.notify_all();
    }
}

// Wait until every queued launch's host side is done (spin first, then sleep).
void drain(fcl_context ctx) {
    auto t0 = Clock::now();
    while (ctx->q_len.load(std::memory_order_acquire) > 0) {
        _mm_pause();
        if (std::chrono::duration_cast<std::chrono::nanoseconds>(Clock::now() - t0).count() > ctx->ex.spin_ns) {
            std::unique_lock<std::mutex> lk(ctx->q_mu);
            ctx->drain_sleeping.fetch_add(1);
            ctx->q_cv.wait(lk, [&] { return ctx->queue.empty(); });
            ctx->drain_sleeping.fetch_sub(1);
            return;
        }
    }
    std::lock_guard<std::mutex> lk(ctx->q_mu);   // acquire the coordinator's last critical section
}

// A new launch conflicts with a pending one if either writes a buffer the other touches --
// except a pure read-after-write on a free-running pending launch (device merge in its
// dispatcher, or lite): its device copy is complete in stream order before the new kernel
// on main, and the new launch's host side runs after the pending one's (FIFO) and waits for
// the buffer's return copy before reading the host copy.  So a dependent kernel is not held
// back by the host side of the one before it (e.g. a return race still in progress).
//
// Buffer versions make more of these safe without waiting (C18, L20.s1-9):
//  * RAW on a pending CPU-only job: its host side runs after the job (queue order), and a GPU
//    read waits on the device for the transfer of the job's result (JOB_XFER);
//  * WAR, when the pending launch (free-running, or a CPU-only job) only reads the buffer, does
//    not stream it to the device, and the new launch is cooperative and updates the buffer in
//    place (INOUT): its device writes follow the pending grid on main, and every write to the
//    host copy happens in its own host side -- after the pending one's (queue order), and after
//    any chunk of it that is still stopping (phase B quiesces before returning data).
bool conflicts_with_pending(fcl_context ctx, const Launch &L) {
    std::lock_guard<std::mutex> lk(ctx->q_mu);
    for (Job *p : ctx->queue) {
        if (p->kind == Job::JOB_XFER) {   // reads host copies, writes device copies of xb
            for (int a = 0; a < L.a.nbuf; ++a)
                for (int q = 0; q < p->nx; ++q)
                    if (L.bufs[a] == p->xb[q] && (L.acc[a] & 2)) return true;
            continue;
        }
        const bool cpu_job = p->kind == Job::JOB_CPU;
        const bool free_running = !cpu_job && (p->dev_merge || p->lite);
        for (int a = 0; a < L.a.nbuf; ++a)
            for (int b = 0; b < p->L.a.nbuf; ++b) {
                if (L.bufs[a] != p->L.bufs[b]) continue;
                const bool we_write = (L.acc[a] & 2) != 0, they_write = (p->L.acc[b] & 2) != 0;
                if (we_write) {
                    bool streamed = false;
                    for (int q = 0; q < p->nstream; ++q) streamed |= p->sbuf[q] == b;
                    const bool war_ok = !they_write && (free_running || cpu_job) && !streamed &&
                                        L.o.mode == FCL_MODE_COOP && L.acc[a] == 3;
                    if (!war_ok) return true;                     // WAR / WAW
                    continue;
                }
                if (they_write && !free_running && !cpu_job) return true;   // RAW on a host-decided merge
            }
    }
    return false;
}

fcl_status check_ctx(fcl_context ctx) {
    if (!ctx) return FCL_INVALID_CONTEXT;
    if (ctx->sticky.load() != FCL_SUCCESS) return ctx->sticky.load();
    cudaSetDevice(ctx->device);
    return FCL_SUCCESS;
}

// ---- single-device modes (run with the queue drained) ----
fcl_status run_gpu_only(fcl_context ctx, Launch &L, fcl_launch_info &info) {
    const TaskSpace ts = gpu_task_space(L.a, L.g);
    const int64_t t0 = first_task_at(L.a, L.g, ts.ntasks, L.lo), t1 = first_task_at(L.a, L.g, ts.ntasks, L.hi);
    const bool timing = ctx->ktiming || (L.o.flags & FCL_LAUNCH_TIMING);
    if (timing) CK(ctx, cudaEventRecord(ctx->ev_k0, ctx->main));
    SlotReset r{};
    r.tstamp = plain_stamp(ctx);
    r.exec_cnt = L.o.record_exec_counts ? ctx->rec.d_cnt : nullptr;
    if (gpu_launch_plain(L.a, L.g, t0, t1, ctx->main, &r, pdl_mode(ctx, L)) < 0)
        return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
    if (timing) CK(ctx, cudaEventRecord(ctx->ev_t1, ctx->main));
    CK(ctx, cudaEventRecord(ctx->ev_k1, ctx->main));
    ctx->sync_have_k = timing;
    info.gpu_launches += 1;
    info.gpu_path = FCL_GPU_PATH_PLAIN;
    info.gpu_tasks = info.gpu_tasks_total = t1 - t0;
    if (lazy_return(ctx, L, info)) return FCL_SUCCESS;
    return enqueue_d2h(ctx, L, L.lo, L.hi, info, ctx->ev_k1);
}

fcl_status run_cpu_only(fcl_context ctx, Launch &L, fcl_launch_info &info) {
    info.n_wg = L.hi - L.lo; info.wg_lo = L.lo; info.wg_hi = L.hi;
    info.gpu_watermark = L.hi;
    Executor &ex = ctx->ex;
    const int nact = L.o.n_host_threads > 0 ? L.o.n_host_threads : ex.T;
    const int64_t nwg = L.hi - L.lo;
    const int parts = (L.o.cpu_wg_split && nwg < nact) ? (int)((nact + nwg - 1) / nwg) : 1;
    const double t0 = now_ms();
    quiesce(ctx);
    VariantPick vp = pick_variant(ctx, L);
    int64_t hi = L.hi;
    int nch = 0;
    if (vp.profiling) {   // wake the pool first: no variant's sample pays for sleeping workers
        ex.submit(L.a, L.g, L.lo, L.lo, 1, nact);
        ex.wait();
    }
    // online profiling: one small allocation per variant, from the top, then the winner
    while (vp.profiling && vp.next < vp.nvar && hi > L.lo) {
        const int v = chunk_variant(vp);
        const int64_t size = std::min<int64_t>(hi - L.lo, std::max<int64_t>(L.o.cpu_wg_split ? 1 : nact,
                                                                           ceil_pct(std::max(1, L.o.init_chunk_pct), nwg)));
        const int p = (L.o.cpu_wg_split && size < nact) ? (int)((nact + size - 1) / size) : 1;
        KArgs ka = L.a;
        ka.host_variant = v;
        const double tc = now_ms();
        ex.submit(ka, L.g, hi - size, hi, p, nact);
        ex.wait();
        variant_measured(ctx, L, vp, v, now_ms() - tc, size);
        if (nch < 64) info.chunk_sizes[nch] = (int32_t)size;
        ++nch;
        hi -= size;
    }
    if (hi > L.lo) {
        KArgs ka = L.a;
        ka.host_variant = vp.var;
        const int64_t rest = hi - L.lo;
        const int p = (L.o.cpu_wg_split && rest < nact) ? (int)((nact + rest - 1) / rest) : 1;
        ex.submit(ka, L.g, L.lo, hi, p, nact);
        ex.wait();
        if (nch < 64) info.chunk_sizes[nch] = (int32_t)rest;
        ++nch;
    }
    (void)parts;
    variant_info(vp, info);
    info.t_host_ms = now_ms() - t0;
    info.cpu_wgs = nwg;
    info.n_chunks = nch;
    info.n_c11_chunks = 0;   // (CPU-only: profiling allocations, then the rest in one job)
    info.cpu_did_all = 1;
    info.published_watermark = L.lo;
    return FCL_SUCCESS;   // (the outputs' device copies were marked stale at enqueue: program order)
}

}  // namespace

// ==========================================================================================
// C-ABI
// ==========================================================================================
extern "C" {

const char *fcl_version(void) { return "fcl-b200 0.2 sm_100a"; }

const char *fcl_status_string(fcl_status s) {
    switch (s) {
    case FCL_SUCCESS: return "FCL_SUCCESS";
    case FCL_DEVICE_NOT_AVAILABLE: return "FCL_DEVICE_NOT_AVAILABLE";
    case FCL_OUT_OF_RESOURCES: return "FCL_OUT_OF_RESOURCES";
    case FCL_INVALID_VALUE: return "FCL_INVALID_VALUE";
    case FCL_INVALID_CONTEXT: return "FCL_INVALID_CONTEXT";
    case FCL_INVALID_MEM_OBJECT: return "FCL_INVALID_MEM_OBJECT";
    case FCL_INVALID_KERNEL_NAME: return "FCL_INVALID_KERNEL_NAME";
    case FCL_INVALID_KERNEL: return "FCL_INVALID_KERNEL";
    case FCL_INVALID_KERNEL_ARGS: return "FCL_INVALID_KERNEL_ARGS";
    case FCL_INVALID_WORK_DIMENSION: return "FCL_INVALID_WORK_DIMENSION";
    case FCL_INVALID_WORK_GROUP_SIZE: return "FCL_INVALID_WORK_GROUP_SIZE";
    case FCL_INVALID_GLOBAL_WORK_SIZE: return "FCL_INVALID_GLOBAL_WORK_SIZE";
    case FCL_CONTEXT_LOST: return "FCL_CONTEXT_LOST";
    case FCL_CUDA_ERROR: return "FCL_CUDA_ERROR";
    case FCL_NOT_SUPPORTED: return "FCL_NOT_SUPPORTED";
    default: return "FCL_UNKNOWN_STATUS";
    }
}

const char *fcl_last_error(fcl_context ctx) {
    if (!ctx) return "no context";
    std::lock_guard<std::mutex> lk(ctx->err_mu);
    static thread_local std::string copy;
    copy = ctx->err;
    return copy.c_str();
}

fcl_status fcl_default_launch_opts(fcl_launch_opts *o) {
    if (!o) return FCL_INVALID_VALUE;
    std::memset(o, 0, sizeof *o);
    o->mode = FCL_MODE_COOP;
    o->forced_split = -1;
    o->init_chunk_pct = 2;
    o->step_pct = 2;
    o->cpu_wg_split = 1;
    o->abort_period = 0;
    o->wg_lo = 0;
    o->wg_hi = -1;
    o->blocking = 0;
    o->host_variant = -1;
    return FCL_SUCCESS;
}

// FCL_SEGV_TRACE=1: a native backtrace on SIGSEGV/SIGBUS/SIGABRT (diagnostics on the GPU box)
static void segv_trace(int sig) {
    void *frames[64];
    const int n = backtrace(frames, 64);
    char msg[64];
    const int len = snprintf(msg, sizeof msg, "fcl: signal %d, native backtrace:\n", sig);
    if (len > 0) { ssize_t w = write(2, msg, (size_t)len); (void)w; }
    backtrace_symbols_fd(frames, n, 2);
    signal(sig, SIG_DFL);
    raise(sig);
}

// The CPUs of the GPU's NUMA node (/sys/bus/pci/devices/<bus id>/local_cpulist), empty if unknown:
// a host pool next to its GPU reads and writes the pinned mirrors in local DRAM (SURVEY §8b:
// "all local-NUMA cores").
static std::vector<int> gpu_local_cpus(int device) {
    std::vector<int> out;
    char bus[32] = {0};
    if (cudaDeviceGetPCIBusId(bus, sizeof bus, device) != cudaSuccess) { cudaGetLastError(); return out; }
    for (char *c = bus; *c; ++c) *c = (char)tolower(*c);
    std::string path = std::string("/sys/bus/pci/devices/") + bus + "/local_cpulist";
    FILE *f = fopen(path.c_str(), "r");
    if (!f) return out;
    char line[4096] = {0};
    if (fgets(line, sizeof line, f)) {
        for (char *tok = strtok(line, ",\n"); tok; tok = strtok(nullptr, ",\n")) {
            int a = -1, b = -1;
            if (sscanf(tok, "%d-%d", &a, &b) == 2) { for (int c = a; c <= b; ++c) out.push_back(c); }
            else if (sscanf(tok, "%d", &a) == 1) out.push_back(a);
        }
    }
    fclose(f);
    return out;
}

fcl_status fcl_create_context(const fcl_context_desc *desc, fcl_context *out) {
    if (getenv("FCL_SEGV_TRACE") && atoi(getenv("FCL_SEGV_TRACE")) != 0) {
        signal(SIGSEGV, segv_trace);
        signal(SIGBUS, segv_trace);
        signal(SIGABRT, segv_trace);
    }
    if (!out) return FCL_INVALID_VALUE;
    *out = nullptr;
    fcl_context_desc d{};
    if (desc) d = *desc;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) { cudaGetLastError(); return FCL_DEVICE_NOT_AVAILABLE; }
    if (d.device < 0 || d.device >= ndev) return FCL_INVALID_VALUE;
    if (d.status_location != FCL_STATUS_HOST_MAPPED && d.status_location != FCL_STATUS_DEVICE) return FCL_INVALID_VALUE;
    fcl_context ctx = new fcl_context_st();
    ctx->device = d.device;
    ctx->status_location = d.status_location;
    if ((d.dev_alloc == nullptr) != (d.dev_free == nullptr)) { delete ctx; return FCL_INVALID_VALUE; }
    ctx->dev_alloc = d.dev_alloc;
    ctx->dev_free = d.dev_free;
    ctx->alloc_user = d.alloc_user;
    auto fail = [&](cudaError_t e, const char *what) {
        fprintf(stderr, "fcl_create_context: %s: %s\n", what, cudaGetErrorString(e));
        delete ctx;
        return FCL_CUDA_ERROR;
    };
    cudaError_t e;
    if ((e = cudaSetDevice(d.device)) != cudaSuccess) return fail(e, "cudaSetDevice");
    if ((e = cudaFree(nullptr)) != cudaSuccess) return fail(e, "context init");
    cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, d.device);
    auto mk = [&](void *given, cudaStream_t *s, bool *own) -> cudaError_t {
        if (given) { *s = (cudaStream_t)given; *own = false; return cudaSuccess; }
        *own = true;
        return cudaStreamCreateWithFlags(s, cudaStreamNonBlocking);
    };
    if ((e = mk(d.main_stream, &ctx->main, &ctx->own_main)) != cudaSuccess) return fail(e, "main stream");
    if ((e = mk(d.hd_stream, &ctx->hd, &ctx->own_hd)) != cudaSuccess) return fail(e, "hd stream");
    if ((e = mk(d.dh_stream, &ctx->dh, &ctx->own_dh)) != cudaSuccess) return fail(e, "dh stream");
    if ((e = cudaStreamCreateWithFlags(&ctx->xt, cudaStreamNonBlocking)) != cudaSuccess) return fail(e, "transfer stream");
    if ((e = cudaStreamCreateWithFlags(&ctx->dr, cudaStreamNonBlocking)) != cudaSuccess) return fail(e, "race stream");
    // status words (one per launch slot), GPU-exit word, pinned copy of the wm word
    void *hp = nullptr, *dp = nullptr;
    if ((e = cudaHostAlloc(&hp, 64, cudaHostAllocPortable)) != cudaSuccess) return fail(e, "pinned scratch");
    std::memset(hp, 0, 64);
    ctx->wm_host = (unsigned long long *)hp;
    if ((e = cudaHostAlloc(&hp, 8 * fcl_context_st::kSlots, cudaHostAllocMapped | cudaHostAllocPortable)) != cudaSuccess) return fail(e, "exit word");
    std::memset(hp, 0, 8 * fcl_context_st::kSlots);
    ctx->exit_host = (unsigned long long *)hp;
    if ((e = cudaHostGetDevicePointer(&dp, hp, 0)) != cudaSuccess) return fail(e, "exit word mapping");
    ctx->exit_dptr = (unsigned long long *)dp;
    if (d.status_location == FCL_STATUS_HOST_MAPPED) {
        if ((e = cudaHostAlloc(&hp, 8 * fcl_context_st::kSlots, cudaHostAllocMapped | cudaHostAllocPortable)) != cudaSuccess) return fail(e, "status word");
        std::memset(hp, 0, 8 * fcl_context_st::kSlots);
        ctx->status_host = (unsigned long long *)hp;
        if ((e = cudaHostGetDevicePointer(&dp, hp, 0)) != cudaSuccess) return fail(e, "status mapping");
        ctx->status_dptr = (unsigned long long *)dp;
    } else {
        if ((e = cudaMalloc(&dp, 8 * fcl_context_st::kSlots)) != cudaSuccess) return fail(e, "status word");
        cudaMemset(dp, 0, 8 * fcl_context_st::kSlots);
        ctx->status_dptr = (unsigned long long *)dp;
    }
    // device counters: claim[kSlots], tasks[kSlots], wm word, stamps[4 * kSlots], merge chunk
    // counters[kSlots], then barrier counters (32 u32 per slot: root + 16 leaves)
    if ((e = cudaMalloc(&dp, 8 * (7 * fcl_context_st::kSlots + 2) + 128 * fcl_context_st::kSlots)) != cudaSuccess) return fail(e, "counters");
    cudaMemset(dp, 0, 8 * (7 * fcl_context_st::kSlots + 2) + 128 * fcl_context_st::kSlots);
    ctx->dclaim = (unsigned long long *)dp;
    ctx->dtasks = ctx->dclaim + fcl_context_st::kSlots;
    ctx->dwm = ctx->dtasks + fcl_context_st::kSlots;
    ctx->dstamp = ctx->dwm + 2;
    ctx->dmctr = ctx->dstamp + 4 * fcl_context_st::kSlots;
    ctx->dbar = (unsigned int *)(ctx->dmctr + fcl_context_st::kSlots);
    if (getenv("FCL_STATS") && atoi(getenv("FCL_STATS")) != 0) {
        if ((e = cudaMalloc(&dp, 16 * fcl_context_st::kPlainStamps)) != cudaSuccess) return fail(e, "stamps");
        cudaMemset(dp, 0, 16 * fcl_context_st::kPlainStamps);
        ctx->dpstamp = (unsigned long long *)dp;
    }
    for (cudaEvent_t *pe : {&ctx->ev_k0, &ctx->ev_t1})
        if ((e = cudaEventCreate(pe)) != cudaSuccess) return fail(e, "events");
    if ((e = cudaMalloc(&dp, 8 * fcl_context_st::kSlots)) != cudaSuccess) return fail(e, "arrival words");
    cudaMemset(dp, 0, 8 * fcl_context_st::kSlots);
    ctx->darrival = (unsigned long long *)dp;
    for (cudaEvent_t *pe : {&ctx->ev_k1, &ctx->ev_mark, &ctx->ev_hd_release, &ctx->ev_gd2h, &ctx->race_ev[0], &ctx->race_ev[1],
                            &ctx->race_ev[2], &ctx->race_ev[3], &ctx->stream_ev[0], &ctx->stream_ev[1], &ctx->stream_ev[2],
                            &ctx->stream_ev[3], &ctx->ev_stream_done})
        if ((e = cudaEventCreateWithFlags(pe, cudaEventDisableTiming)) != cudaSuccess) return fail(e, "events");
    // stream memory operations for publication (driver entry point; fall back to a kernel store)
    {
        void *fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue64", &fn, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess && fn)
            ctx->write64 = (PFN_writeValue64)fn;
        else
            cudaGetLastError();
    }
    {
        void *fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue64", &fn, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess && fn)
            ctx->wait64 = (PFN_waitValue64)fn;
        else
            cudaGetLastError();
    }
    if (getenv("FCL_NO_MEMOPS")) { ctx->write64 = nullptr; ctx->wait64 = nullptr; }
    ctx->no_version_wait = getenv("FCL_NO_VERSION_WAIT") && atoi(getenv("FCL_NO_VERSION_WAIT")) != 0;
    if (getenv("FCL_TEST_PUBLISH_ZERO_US") && getenv("FCL_STATS") && atoi(getenv("FCL_STATS")) != 0) {
        ctx->test_publish_zero_us = atoll(getenv("FCL_TEST_PUBLISH_ZERO_US"));
        if ((e = cudaMalloc(&dp, 8 * fcl_context_st::kSlots)) != cudaSuccess) return fail(e, "publish stamps");
        cudaMemset(dp, 0, 8 * fcl_context_st::kSlots);
        ctx->dpub = (unsigned long long *)dp;
    }
    if ((e = cudaMalloc(&dp, 8)) != cudaSuccess) return fail(e, "transfer word");
    cudaMemset(dp, 0, 8);
    ctx->d_xfer = (unsigned long long *)dp;
    if (getenv("FCL_EAGER_RETURN_BYTES")) ctx->eager_return_bytes = (size_t)atoll(getenv("FCL_EAGER_RETURN_BYTES"));
    ctx->stats = getenv("FCL_STATS") && atoi(getenv("FCL_STATS")) != 0;
    ctx->tr.on = getenv("FCL_TRACE") && atoi(getenv("FCL_TRACE")) != 0;
    ctx->pdl = !(getenv("FCL_NO_PDL") && atoi(getenv("FCL_NO_PDL")) != 0);
    if (getenv("FCL_LITE_EXIT")) ctx->lite_exit_word = atoi(getenv("FCL_LITE_EXIT")) != 0;
    if (getenv("FCL_POOL_KEEP")) ctx->pool_keep = (uint32_t)std::max(0, atoi(getenv("FCL_POOL_KEEP")));
    if (getenv("FCL_POOL_CAP_MB")) ctx->pool_cap = (size_t)atoll(getenv("FCL_POOL_CAP_MB")) << 20;
    ctx->stream_on = !(getenv("FCL_NO_STREAM") && atoi(getenv("FCL_NO_STREAM")) != 0);
    if (getenv("FCL_STREAM_PIECE_BYTES")) ctx->stream_piece_bytes = std::max<size_t>(1 << 16, (size_t)atoll(getenv("FCL_STREAM_PIECE_BYTES")));
    if (getenv("FCL_SELECT")) ctx->select_on = atoi(getenv("FCL_SELECT")) != 0;
    if (getenv("FCL_TEST_GPU_DELAY_US")) ctx->test_gpu_delay_ns = 1000ull * (unsigned long long)atoll(getenv("FCL_TEST_GPU_DELAY_US"));
    if (getenv("FCL_SELECT_MIN_SHARE")) ctx->select_min_share = atof(getenv("FCL_SELECT_MIN_SHARE"));
    if (getenv("FCL_SELECT_STREAM_SHARE")) ctx->select_stream_share = atof(getenv("FCL_SELECT_STREAM_SHARE"));
    if (getenv("FCL_SEQ_DEBUG")) ctx->seq_debug = atoi(getenv("FCL_SEQ_DEBUG")) != 0;
    if (getenv("FCL_SEQ_SELECT")) ctx->seq_on = atoi(getenv("FCL_SEQ_SELECT")) != 0;
    if (getenv("FCL_SELECT_PERIOD")) ctx->select_period = std::max(0, atoi(getenv("FCL_SELECT_PERIOD")));
    if (getenv("FCL_LAZY_BYTES")) ctx->lazy_max_bytes = (size_t)atoll(getenv("FCL_LAZY_BYTES"));
    ctx->force_twin = getenv("FCL_FORCE_TWIN") && atoi(getenv("FCL_FORCE_TWIN")) != 0;
    ctx->unfused = getenv("FCL_UNFUSED_MERGE") && atoi(getenv("FCL_UNFUSED_MERGE")) != 0;
    ctx->no_lite = getenv("FCL_NO_LITE") && atoi(getenv("FCL_NO_LITE")) != 0;
    ctx->no_sym = getenv("FCL_NO_SYM") && atoi(getenv("FCL_NO_SYM")) != 0;
    ctx->no_race = getenv("FCL_NO_RACE") && atoi(getenv("FCL_NO_RACE")) != 0;
    if (getenv("FCL_ABORT_PERIOD")) ctx->env_abort_period = atoi(getenv("FCL_ABORT_PERIOD"));
    if (getenv("FCL_EXIT_POLL_PAUSES")) ctx->exit_poll_pauses = std::max(1, atoi(getenv("FCL_EXIT_POLL_PAUSES")));
    if (getenv("FCL_RACE_MIN_BYTES")) ctx->race_min_bytes = (size_t)atoll(getenv("FCL_RACE_MIN_BYTES"));
    if (getenv("FCL_RACE_PIECE_BYTES")) ctx->race_piece_bytes = std::max<size_t>(4096, (size_t)atoll(getenv("FCL_RACE_PIECE_BYTES")));
    if (getenv("FCL_RACE_CHUNK_MS")) ctx->race_chunk_ms = atof(getenv("FCL_RACE_CHUNK_MS"));
    if (getenv("FCL_KTIMING")) ctx->ktiming = atoi(getenv("FCL_KTIMING")) != 0;
    if ((e = cudaDeviceSynchronize()) != cudaSuccess) return fail(e, "init sync");
    // (FCL_NO_PRELOAD=1: keep CUDA's lazy loading -- only to show what the preload prevents)
    if (!(getenv("FCL_NO_PRELOAD") && atoi(getenv("FCL_NO_PRELOAD")) != 0) && gpu_preload_kernels() != 0)
        return fail(cudaErrorInvalidDeviceFunction, "kernel preload");
    const char *pin = getenv("FCL_PIN_THREADS");
    const bool do_pin = d.pin_threads ? true : (pin ? atoi(pin) != 0 : true);
    int nthr = d.n_host_threads;
    if (nthr <= 0 && getenv("FCL_HOST_THREADS")) nthr = atoi(getenv("FCL_HOST_THREADS"));
    ctx->ex.start(nthr, do_pin, gpu_local_cpus(d.device));
    ctx->coord_core = (do_pin && !ctx->ex.cores.empty()) ? ctx->ex.cores[0] : -1;
    ctx->coord = std::thread(coordinator, ctx);
    *out = ctx;
    return FCL_SUCCESS;
}

fcl_status fcl_release_context(fcl_context ctx) {
    if (!ctx) return FCL_INVALID_CONTEXT;
    cudaSetDevice(ctx->device);
    drain(ctx);
    quiesce(ctx);
    if (ctx->tr.on) {
        const char *path = getenv("FCL_TRACE_FILE");
        FILE *f = path ? fopen(path, "w") : stderr;
        if (f) {
            for (auto &r : ctx->tr.recs) fprintf(f, "%.4f %s %u\n", r.t, r.tag, r.epoch);
            if (f != stderr) fclose(f);
        }
    }
    {
        std::lock_guard<std::mutex> lk(ctx->q_mu);
        ctx->q_stop = true;
        ctx->q_stop_flag.store(1);
    }
    ctx->q_cv.notify_all();
    if (ctx->coord.joinable()) ctx->coord.join();
    cudaDeviceSynchronize();
    ctx->ex.shutdown();
    for (auto &pe : ctx->pool) dfree(ctx, pe.p);
    for (Job *j : ctx->free_jobs) {
        for (cudaEvent_t e : {j->ev_start, j->ev_k0, j->ev_t1, j->ev_k1, j->ev_m0, j->ev_m1, j->ev_staged, j->ev_ret, j->ev_wm, j->ev_d2h})
            if (e) cudaEventDestroy(e);
        delete j;
    }
    if (ctx->last && ctx->last->done.load()) {
        Job *j = ctx->last;
        for (cudaEvent_t e : {j->ev_start, j->ev_k0, j->ev_t1, j->ev_k1, j->ev_m0, j->ev_m1, j->ev_staged, j->ev_ret, j->ev_wm, j->ev_d2h})
            if (e) cudaEventDestroy(e);
        delete j;
    }
    for (cudaEvent_t e : {ctx->ev_k0, ctx->ev_t1, ctx->ev_k1, ctx->ev_mark, ctx->ev_hd_release, ctx->ev_gd2h, ctx->race_ev[0],
                          ctx->race_ev[1], ctx->race_ev[2], ctx->race_ev[3], ctx->stream_ev[0], ctx->stream_ev[1],
                          ctx->stream_ev[2], ctx->stream_ev[3], ctx->ev_stream_done})
        if (e) cudaEventDestroy(e);
    if (ctx->status_host) cudaFreeHost(ctx->status_host);
    else if (ctx->status_dptr) cudaFree(ctx->status_dptr);
    if (ctx->wm_host) cudaFreeHost(ctx->wm_host);
    if (ctx->exit_host) cudaFreeHost(ctx->exit_host);
    if (ctx->dclaim) cudaFree(ctx->dclaim);
    if (ctx->rec.d_cnt) cudaFree(ctx->rec.d_cnt);
    if (ctx->rec.d_w) cudaFree(ctx->rec.d_w);
    if (ctx->darrival) cudaFree(ctx->darrival);
    if (ctx->d_xfer) cudaFree(ctx->d_xfer);
    if (ctx->dpub) cudaFree(ctx->dpub);
    if (ctx->own_main) cudaStreamDestroy(ctx->main);
    if (ctx->own_hd) cudaStreamDestroy(ctx->hd);
    if (ctx->own_dh) cudaStreamDestroy(ctx->dh);
    if (ctx->xt) cudaStreamDestroy(ctx->xt);
    if (ctx->dr) cudaStreamDestroy(ctx->dr);
    delete ctx;
    return FCL_SUCCESS;
}

static fcl_status create_buffer_impl(fcl_context ctx, uint32_t flags, size_t bytes, uint32_t elem_size,
                                     const void *host_init, void *host_ptr, void *device_ptr, fcl_buffer *out) {
    fcl_status s = check_ctx(ctx);
    if (s != FCL_SUCCESS) return s;
    if (!out || bytes == 0) return set_err(ctx, FCL_INVALID_VALUE, "bytes must be > 0");
    if (!(elem_size == 1 || elem_size == 2 || elem_size == 4 || elem_size == 8) || bytes % elem_size)
        return set_err(ctx, FCL_INVALID_VALUE, "elem_size %u invalid for %zu bytes", elem_size, bytes);
    if ((flags & FCL_MEM_USE_HOST_PTR) && !host_ptr) return set_err(ctx, FCL_INVALID_VALUE, "USE_HOST_PTR without host_ptr");
    if ((flags & FCL_MEM_USE_DEVICE_PTR) && !device_ptr) return set_err(ctx, FCL_INVALID_VALUE, "USE_DEVICE_PTR without device_ptr");
    if (ctx->stream_jobs.load(std::memory_order_acquire) > 0) drain(ctx);   // (allocations below: see stream_jobs)
    fcl_buffer b = new fcl_buffer_st();
    b->ctx = ctx; b->bytes = bytes; b->elem_size = elem_size; b->flags = flags;
    cudaError_t e;
    if (flags & FCL_MEM_USE_DEVICE_PTR) { b->dev = device_ptr; b->own_dev = false; }
    else {
        if (!(b->dev = dmalloc(ctx, bytes))) { delete b; return set_err(ctx, FCL_OUT_OF_RESOURCES, "device allocation of %zu bytes", bytes); }
        b->own_dev = true;
    }
    if (flags & FCL_MEM_USE_HOST_PTR) { b->host = host_ptr; b->own_host = false; }
    else {
        if ((e = cudaHostAlloc(&b->host, bytes, cudaHostAllocPortable | cudaHostAllocMapped)) != cudaSuccess) {
            cudaGetLastError();
            if (b->own_dev) dfree(ctx, b->dev);
            delete b;
            return set_err(ctx, FCL_OUT_OF_RESOURCES, "cudaHostAlloc(%zu)", bytes);
        }
        b->own_host = true;
    }
    if ((e = cudaEventCreateWithFlags(&b->d2h_ev, cudaEventDisableTiming)) != cudaSuccess) { delete b; return cuda_fail(ctx, e, "event"); }
    // device-visible address of the host mirror (write-through returns); caller memory that is
    // not pinned and mapped has none
    {
        void *dp = nullptr;
        if (cudaHostGetDevicePointer(&dp, b->host, 0) == cudaSuccess) b->host_dptr = dp;
        else { cudaGetLastError(); b->host_dptr = nullptr; }
    }
    const bool ext_host = (flags & FCL_MEM_USE_HOST_PTR) != 0, ext_dev = (flags & FCL_MEM_USE_DEVICE_PTR) != 0;
    if (host_init) {
        std::memcpy(b->host, host_init, bytes);
        if ((e = cudaMemcpy(b->dev, b->host, bytes, cudaMemcpyHostToDevice)) != cudaSuccess) return cuda_fail(ctx, e, "initial H2D");
    } else if (ext_host && !ext_dev) {
        if ((e = cudaMemcpy(b->dev, b->host, bytes, cudaMemcpyHostToDevice)) != cudaSuccess) return cuda_fail(ctx, e, "initial H2D");
    } else if (ext_dev && !ext_host) {
        if ((e = cudaMemcpy(b->host, b->dev, bytes, cudaMemcpyDeviceToHost)) != cudaSuccess) return cuda_fail(ctx, e, "initial D2H");
    } else if (!ext_host && !ext_dev) {
        std::memset(b->host, 0, bytes);
        if ((e = cudaMemset(b->dev, 0, bytes)) != cudaSuccess) return cuda_fail(ctx, e, "memset");
    }
    b->host_valid = b->dev_valid = true;
    *out = b;
    return FCL_SUCCESS;
}

fcl_status fcl_create_buffer(fcl_context ctx, uint32_t flags, size_t bytes, uint32_t elem_size,
                             const void *host_init, fcl_buffer *out) {
    if (flags & (FCL_MEM_USE_HOST_PTR | FCL_MEM_USE_DEVICE_PTR))
        return set_err(ctx, FCL_INVALID_VALUE, "use fcl_create_buffer_ext for caller-owned memory");
    return create_buffer_impl(ctx, flags, bytes, elem_size, host_init, nullptr, nullptr, out);
}

fcl_status fcl_create_buffer_ext(fcl_context ctx, uint32_t flags, size_t bytes, uint32_t elem_size,
                                 void *host_ptr, void *device_ptr, fcl_buffer *out) {
    if (host_ptr) flags |= FCL_MEM_USE_HOST_PTR;
    if (device_ptr) flags |= FCL_MEM_USE_DEVICE_PTR;
    return create_buffer_impl(ctx, flags, bytes, elem_size, nullptr, host_ptr, device_ptr, out);
}

fcl_status fcl_release_buffer(fcl_buffer b) {
    if (!b) return FCL_INVALID_MEM_OBJECT;
    fcl_context ctx = b->ctx;
    cudaSetDevice(ctx->device);
    drain(ctx);
    quiesce(ctx);   // no abandoned chunk may still touch the mirror being freed
    if (b->ret_lazy) {   // its pending return is dropped with it
        b->ret_lazy = false;
        ctx->lazy.erase(std::remove(ctx->lazy.begin(), ctx->lazy.end(), b), ctx->lazy.end());
    }
    cudaStreamSynchronize(ctx->main);
    cudaStreamSynchronize(ctx->hd);
    cudaStreamSynchronize(ctx->dh);
    cudaStreamSynchronize(ctx->dr);
    cudaStreamSynchronize(ctx->xt);
    if (b->merge_pending) {
        if (b->twin) pool_put(ctx, b->twin, false);
        if (b->stage) pool_put(ctx, b->stage, false);
        ctx->defer_list.erase(std::remove(ctx->defer_list.begin(), ctx->defer_list.end(), b), ctx->defer_list.end());
    }
    if (b->own_dev) dfree(ctx, b->dev);
    if (b->own_host) cudaFreeHost(b->host);
    cudaEventDestroy(b->d2h_ev);
    delete b;
    return FCL_SUCCESS;
}

fcl_status fcl_write_buffer(fcl_context ctx, fcl_buffer b, size_t offset, size_t n, const void *src, int32_t blocking) {
    fcl_status s = check_ctx(ctx);
    if (s != FCL_SUCCESS) return s;
    if (!b || b->ctx != ctx) return FCL_INVALID_MEM_OBJECT;
    if (!src || offset > b->bytes || n > b->bytes - offset) return set_err(ctx, FCL_INVALID_VALUE, "write range");
    drain(ctx);
    quiesce(ctx);   // an abandoned chunk may still read or write this mirror
    if (b->ret_lazy && (s = flush_returns(ctx, false)) != FCL_SUCCESS) return s;
    if (d2h_busy(ctx, b)) { CK(ctx, cudaEventSynchronize(b->d2h_ev)); b->d2h_pending = false; }
    char *h = (char *)b->host + offset;
    if (n < b->bytes) {
        s = make_valid(ctx, b, true, true, nullptr);
        if (s != FCL_SUCCESS) return s;
    }
    // overwriting the pinned mirror: no queued copy may still read its old contents (main, and
    // the pieces of a streamed launch on hd)
    if (src != h) CK(ctx, cudaStreamSynchronize(ctx->main));
    if (src != h && ctx->xt_used.load()) CK(ctx, cudaStreamSynchronize(ctx->xt));   // transfers read mirrors
    if (ctx->stream_pending) {
        CK(ctx, cudaEventSynchronize(ctx->ev_stream_done));
        ctx->stream_pending = false;
    }
    if (src != h) std::memcpy(h, src, n);
    b->ver_expected = b->ver_host = ++ctx->kid;   // a write is a new version of the buffer
    if (!blocking && n == b->bytes) {
        // a non-blocking write of the whole buffer refreshes the device copy lazily, when a
        // launch first needs it on the GPU -- never, if the data is consumed on the host alone
        // (device selection)
        b->host_valid = true;
        b->dev_valid = false;
        return FCL_SUCCESS;
    }
    b->ver_dev = b->ver_host;
    CK(ctx, cudaMemcpyAsync((char *)b->dev + offset, h, n, cudaMemcpyHostToDevice, ctx->main));
    ctx->counts[FCL_COUNT_H2D_BYTES] += (int64_t)n;
    b->host_valid = b->dev_valid = true;
    if (blocking) CK(ctx, cudaStreamSynchronize(ctx->main));
    return FCL_SUCCESS;
}

fcl_status fcl_read_buffer(fcl_context ctx, fcl_buffer b, size_t offset, size_t n, void *dst, int32_t blocking) {
    fcl_status s = check_ctx(ctx);
    if (s != FCL_SUCCESS) return s;
    if (!b || b->ctx != ctx) return FCL_INVALID_MEM_OBJECT;
    if (!dst || offset > b->bytes || n > b->bytes - offset) return set_err(ctx, FCL_INVALID_VALUE, "read range");
    (void)blocking;
    drain(ctx);
    quiesce(ctx);
    if (b->ret_lazy && (s = flush_returns(ctx, false)) != FCL_SUCCESS) return s;
    if (d2h_busy(ctx, b)) { CK(ctx, cudaEventSynchronize(b->d2h_ev)); b->d2h_pending = false; }
    if (b->host_valid) {   // location tracking (L20.s31-33): no transfer when the host is current
        const char *h = (const char *)b->host + offset;
        if (dst != h) std::memcpy(dst, h, n);
        return FCL_SUCCESS;
    }
    CK(ctx, cudaStreamSynchronize(ctx->main));
    CK(ctx, cudaMemcpy((char *)b->host + offset, (char *)b->dev + offset, n, cudaMemcpyDeviceToHost));
    if (n == b->bytes) { b->host_valid = true; b->ver_host = b->ver_dev; }
    const char *h = (const char *)b->host + offset;
    if (dst != h) std::memcpy(dst, h, n);
    return FCL_SUCCESS;
}

fcl_status fcl_buffer_versions(fcl_buffer b, uint64_t *expected, uint64_t *host, uint64_t *device) {
    if (!b) return FCL_INVALID_MEM_OBJECT;
    if (expected) *expected = b->ver_expected;
    if (host) *host = b->host_valid ? b->ver_host : 0;
    if (device) *device = b->dev_valid ? b->ver_dev : 0;
    return FCL_SUCCESS;
}

fcl_status fcl_buffer_info(fcl_buffer b, void **host_ptr, void **device_ptr, size_t *bytes, uint32_t *elem_size) {
    if (!b) return FCL_INVALID_MEM_OBJECT;
    if (host_ptr) *host_ptr = b->host;
    if (device_ptr) *device_ptr = b->dev;
    if (bytes) *bytes = b->bytes;
    if (elem_size) *elem_size = b->elem_size;
    return FCL_SUCCESS;
}

fcl_status fcl_get_kernel(fcl_context ctx, const char *name, fcl_kernel *out) {
    (void)ctx;
    if (!name || !out) return FCL_INVALID_VALUE;
    static fcl_kernel_st handles[kNumKernels];
    for (int k = 0; k < kNumKernels; ++k)
        if (!std::strcmp(kKernels[k].name, name)) {
            handles[k].def = &kKernels[k];
            *out = &handles[k];
            return FCL_SUCCESS;
        }
    return FCL_INVALID_KERNEL_NAME;
}

fcl_status fcl_kernel_host_variants(fcl_kernel k, int32_t *n, const char **names, int32_t max_names) {
    if (!k || !k->def) return FCL_INVALID_KERNEL;
    if (!n) return FCL_INVALID_VALUE;
    const int kid = k->def->id;
    *n = host_num_variants(kid);
    if (names)
        for (int v = 0; v < *n && v < max_names; ++v) names[v] = host_variant_name(kid, v);
    return FCL_SUCCESS;
}

fcl_status fcl_kernel_signature(fcl_kernel k, char *buf, size_t len) {
    if (!k || !buf || len == 0) return FCL_INVALID_VALUE;
    std::string s;
    for (int a = 0; a < k->def->nargs; ++a) {
        const ArgSpec &sp = k->def->args[a];
        if (a) s += ' ';
        s += sp.name;
        s += ':';
        if (sp.kind == 'b') s += (sp.acc == 1 ? "in" : sp.acc == 2 ? "out" : "inout");
        else s += (sp.kind == 'i' ? "i" : "f");
    }
    std::snprintf(buf, len, "%s", s.c_str());
    return s.size() < len ? FCL_SUCCESS : FCL_INVALID_VALUE;
}

// opts.record_exec_counts: reset the record for launch L (device counters zeroed on main, ahead
// of L's grid) and point L's host bodies at the per-work-group host counters.
static fcl_status exec_rec_begin(fcl_context ctx, Launch &L) {
    auto &r = ctx->rec;
    const TaskSpace ts = gpu_task_space(L.a, L.g);
    r.valid = true;
    r.g = L.g;
    r.lo = L.lo; r.hi = L.hi;
    r.t0 = first_task_at(L.a, L.g, ts.ntasks, L.lo);
    r.t1 = first_task_at(L.a, L.g, ts.ntasks, L.hi);
    r.cpu_done.assign((size_t)L.g.n_wg, 0);
    r.cpu_parts.assign((size_t)L.g.n_wg, 0);
    const size_t need = (size_t)std::max<int64_t>(1, r.t1 - r.t0) * sizeof(unsigned int);
    if (need > r.d_cap) {
        if (r.d_cnt) cudaFree(r.d_cnt);
        if (r.d_w) cudaFree(r.d_w);
        r.d_cnt = r.d_w = nullptr;
        r.d_cap = 0;
        if (cudaMalloc(&r.d_cnt, need) != cudaSuccess || cudaMalloc(&r.d_w, need) != cudaSuccess) {
            cudaGetLastError();
            r.valid = false;
            return set_err(ctx, FCL_OUT_OF_RESOURCES, "exec-count record of %zu bytes", need);
        }
        r.d_cap = need;
    }
    ctx->main_fenced.store(1);
    CK(ctx, cudaMemsetAsync(r.d_cnt, 0, need, ctx->main));
    CK(ctx, cudaMemsetAsync(r.d_w, 0xFF, need, ctx->main));   // plain grids: no mask
    L.a.rec_cpu_done = r.cpu_done.data();
    L.a.rec_cpu_parts = r.cpu_parts.data();
    r.a = L.a;
    return FCL_SUCCESS;
}

static fcl_status build_launch(fcl_context ctx, fcl_kernel kernel, uint32_t work_dim, const size_t gws[3],
                               const size_t lws[3], const fcl_arg *args, uint32_t n_args, const fcl_launch_opts *opts,
                               Launch &L) {
    if (!kernel) return FCL_INVALID_KERNEL;
    const KernelDef *kd = kernel->def;
    if (work_dim < 1 || work_dim > 3) return set_err(ctx, FCL_INVALID_WORK_DIMENSION, "work_dim %u", work_dim);
    if (!gws || !lws) return set_err(ctx, FCL_INVALID_VALUE, "gws/lws required");
    Geom g{};
    g.work_dim = (int)work_dim;
    int64_t lprod = 1;
    g.n_wg = 1;
    for (uint32_t d = 0; d < 3; ++d) {
        g.gws[d] = d < work_dim ? (int64_t)gws[d] : 1;
        g.lws[d] = d < work_dim ? (int64_t)lws[d] : 1;
        if (g.lws[d] <= 0 || g.gws[d] <= 0) return set_err(ctx, FCL_INVALID_WORK_GROUP_SIZE, "zero size in dim %u", d);
        if (g.gws[d] % g.lws[d]) return set_err(ctx, FCL_INVALID_WORK_GROUP_SIZE, "gws %% lws != 0 in dim %u", d);
        g.ng[d] = g.gws[d] / g.lws[d];
        lprod *= g.lws[d];
        g.n_wg *= g.ng[d];
    }
    if (lprod > 1024) return set_err(ctx, FCL_INVALID_WORK_GROUP_SIZE, "work-group of %lld > 1024 items", (long long)lprod);
    if (g.n_wg >= 0xFFFFFFFFll) return set_err(ctx, FCL_INVALID_GLOBAL_WORK_SIZE, "too many work-groups");
    if ((int)n_args != kd->nargs || !args) return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "%s takes %d args", kd->name, kd->nargs);
    KArgs a{};
    a.kernel = kd->id;
    a.integer = kd->integer;
    a.alpha = 1.5f; a.beta = 1.2f; a.eps = 0.1f; a.ialpha = 3; a.ibeta = 2;
    int nb = 0, ni = 0;
    int64_t ints[2] = {0, 0};
    L.nout = 0;
    L.any_inout = false;
    for (int k = 0; k < kd->nargs; ++k) {
        const ArgSpec &sp = kd->args[k];
        const fcl_arg &ar = args[k];
        if (sp.kind == 'b') {
            if (ar.kind != FCL_ARG_BUFFER || !ar.buffer || ar.buffer->ctx != ctx)
                return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "arg %d (%s) must be a buffer of this context", k, sp.name);
            const int acc = ar.access ? ar.access : sp.acc;
            if ((sp.acc & 2) && !(acc & 2))
                return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "arg %s is written by %s: access must be OUT/INOUT", sp.name, kd->name);
            if (ar.buffer->elem_size != 4) return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "arg %s: elem_size must be 4", sp.name);
            L.bufs[nb] = ar.buffer;
            L.acc[nb] = sp.acc;
            a.dev[nb] = ar.buffer->dev;
            a.host[nb] = ar.buffer->host;
            if (sp.acc & 2) L.out_idx[L.nout++] = nb;
            if (sp.acc == 3) L.any_inout = true;
            ++nb;
        } else if (sp.kind == 'i') {
            if (ar.kind != FCL_ARG_INT) return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "arg %d (%s) must be an int", k, sp.name);
            if (!std::strcmp(sp.name, "alpha")) a.ialpha = (int32_t)ar.i;
            else if (!std::strcmp(sp.name, "beta")) a.ibeta = (int32_t)ar.i;
            else if (ni < 2) ints[ni++] = ar.i;
        } else {
            if (ar.kind != FCL_ARG_FLOAT) return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "arg %d (%s) must be a float", k, sp.name);
            if (!std::strcmp(sp.name, "alpha")) a.alpha = (float)ar.f;
            else if (!std::strcmp(sp.name, "beta")) a.beta = (float)ar.f;
            else if (!std::strcmp(sp.name, "eps")) a.eps = (float)ar.f;
        }
    }
    a.nbuf = nb;
    a.n0 = ints[0];
    a.n1 = ni >= 2 ? ints[1] : ints[0];
    if (a.n0 <= 0 || a.n1 <= 0) return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "problem sizes must be > 0");
    for (int k = 0; k < nb; ++k) {
        const int64_t need = required_elems(a.kernel, k, a.n0, a.n1) * 4;
        if ((int64_t)L.bufs[k]->bytes < need)
            return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "buffer arg %d holds %zu bytes, needs %lld", k, L.bufs[k]->bytes, (long long)need);
    }
    for (int x = 0; x < nb; ++x)
        for (int y = x + 1; y < nb; ++y)
            if (L.bufs[x] == L.bufs[y] && ((L.acc[x] & 2) || (L.acc[y] & 2)))
                return set_err(ctx, FCL_INVALID_KERNEL_ARGS, "a written buffer is passed twice (args alias)");
    int64_t ext[3];
    required_extent(a.kernel, a.n0, a.n1, ext);
    for (uint32_t d = 0; d < work_dim; ++d)
        if (g.gws[d] < ext[d] || g.gws[d] >= ext[d] + g.lws[d])
            return set_err(ctx, FCL_INVALID_GLOBAL_WORK_SIZE, "gws[%u]=%lld must be the extent %lld padded to lws", d,
                           (long long)g.gws[d], (long long)ext[d]);
    const char *why = nullptr;
    if (!gpu_geometry_ok(a, g, &why)) return set_err(ctx, FCL_INVALID_WORK_GROUP_SIZE, "%s: %s", kd->name, why);
    fcl_launch_opts o;
    fcl_default_launch_opts(&o);
    if (opts) o = *opts;
    if (o.mode < FCL_MODE_COOP || o.mode > FCL_MODE_CPU_ONLY) return set_err(ctx, FCL_INVALID_VALUE, "mode");
    if (o.host_variant >= host_num_variants(a.kernel))
        return set_err(ctx, FCL_INVALID_VALUE, "host_variant %d: %s has %d", o.host_variant, kd->name, host_num_variants(a.kernel));
    // wg_hi < 0: the whole NDRange; wg_lo == wg_hi: an empty slice (nothing runs)
    int64_t lo = o.wg_lo, hi = o.wg_hi >= 0 ? o.wg_hi : g.n_wg;
    if (lo < 0 || hi > g.n_wg || lo > hi) return set_err(ctx, FCL_INVALID_VALUE, "wg range [%lld, %lld)", (long long)lo, (long long)hi);
    const int64_t al = gpu_slice_align(a, g);
    if ((lo % al) || (hi % al && hi != g.n_wg))
        return set_err(ctx, FCL_INVALID_VALUE, "wg range must be aligned to %lld work-groups (fcl_slice_range)", (long long)al);
    // (the whole range only: a slice's mirror blocks would land in rows outside it and update
    // the device copy of C there -- a later slice on the same buffer would read them final)
    a.sym = (a.kernel == K_SYRK || a.kernel == K_SYR2K) && lo == 0 && hi == g.n_wg && !ctx->no_sym;
    L.ctx = ctx; L.kd = kd; L.a = a; L.g = g; L.lo = lo; L.hi = hi; L.o = o;
    return FCL_SUCCESS;
}

fcl_status fcl_enqueue_ndrange(fcl_context ctx, fcl_kernel kernel, uint32_t work_dim, const size_t gws[3],
                               const size_t lws[3], const fcl_arg *args, uint32_t n_args, const fcl_launch_opts *opts,
                               fcl_launch_info *info_out) {
    fcl_status s = check_ctx(ctx);
    if (s != FCL_SUCCESS) return s;
    const double t_call = now_ms();
    Launch L{};
    s = build_launch(ctx, kernel, work_dim, gws, lws, args, n_args, opts, L);
    if (s != FCL_SUCCESS) return s;
    if (L.hi == L.lo) {   // an empty slice (a rank with no work-groups): nothing to run
        if (info_out) {
            std::memset(info_out, 0, sizeof *info_out);
            info_out->wg_lo = info_out->wg_hi = info_out->gpu_watermark = info_out->published_watermark = L.lo;
            info_out->host_variant = -1;
        }
        return FCL_SUCCESS;
    }
    if (L.o.record_exec_counts) {   // test hook: a fresh record (the previous one's launch must be done)
        drain(ctx);
        quiesce(ctx);
        s = exec_rec_begin(ctx, L);
        if (s != FCL_SUCCESS) return s;
    }
    if (!ctx->defer_list.empty()) {
        drain(ctx);
        if (!ctx->defer_list.empty()) return set_err(ctx, FCL_INVALID_VALUE, "a deferred merge is pending (call fcl_merge)");
    }
    int selected = FCL_SELECTED_COOP;
    bool probe = false;
    int seq_host = 0;
    {
        const bool eligible = select_eligible(ctx, L);
        if (seq_launch(ctx, L, eligible)) {   // sequence selection: the host alone (§6.6)
            selected = FCL_SELECTED_CPU;
            L.o.mode = FCL_MODE_CPU_ONLY;
            seq_host = 1;
            ctx->counts[FCL_COUNT_SEQ_HOST] += 1;
        } else if (eligible) {
            selected = select_device(ctx, L, &probe);
            if (selected == FCL_SELECTED_GPU) L.o.mode = FCL_MODE_GPU_ONLY;
            else if (selected == FCL_SELECTED_CPU) L.o.mode = FCL_MODE_CPU_ONLY;
        }
    }
    const bool coop = L.o.mode == FCL_MODE_COOP;
    const bool cpu_only = L.o.mode == FCL_MODE_CPU_ONLY;
    ctx->tr.add("enq_begin", ctx->epoch + 1);
    // Buffer versions (C18, L20.s1-9) and location tracking (C22, L20.s31-33) order launches
    // without waiting for the pending host sides:
    //  * a host-side reader (a cooperative launch's chunks, a CPU-only launch -- both run by the
    //    coordinator in queue order) finds every earlier host-side writer done, and waits for
    //    the return copies of earlier GPU work on its inputs;
    //  * a GPU-side reader of a buffer a pending CPU-only launch writes waits ON THE DEVICE for a
    //    transfer the coordinator issues after that launch (JOB_XFER + a stream memory wait);
    //  * the remaining hazards (conflicts_with_pending, a host copy written on the device by the
    //    caller, streamed inputs) still wait for the queue -- counted in FCL_COUNT_LAUNCH_DRAINS.
    const uint64_t host_done = ctx->host_done_seq.load(std::memory_order_acquire);
    bool need_drain = L.o.blocking || conflicts_with_pending(ctx, L);
    int nxfer = 0;
    fcl_buffer xfer[6];
    for (int k = 0; k < L.a.nbuf; ++k) {
        fcl_buffer b = L.bufs[k];
        if (cpu_only) {
            need_drain |= !b->host_valid;   // device-written: refreshed synchronously below
            continue;
        }
        if (!b->dev_valid) {
            // a pending host-only job writes it: transfer after that job, wait on the device
            if (b->host_seq > host_done && ctx->write64 && ctx->wait64 && !need_drain) xfer[nxfer++] = b;
            else if (b->host_seq > host_done) need_drain = true;
            // (otherwise the host copy is final: refreshed on main below -- except for a launch
            // that streams its stale rows, which starts on an empty queue)
            else if (coop && ctx->stream_on && (L.a.kernel == K_GESUMMV || L.a.kernel == K_ATAX_TMP || L.a.kernel == K_BICG_Q))
                need_drain = true;
        }
        if (!b->host_valid && coop && (L.acc[k] & 1)) need_drain = true;
    }
    if (need_drain) nxfer = 0;   // (drained: the host copies are final, make_valid refreshes)
    if (need_drain) {
        if (ctx->q_len.load(std::memory_order_acquire) > 0) ctx->counts[FCL_COUNT_LAUNCH_DRAINS] += 1;
        drain(ctx);
    }
    if (conflicts_with_quiescing(ctx, L) || (cpu_only && need_drain)) quiesce(ctx);
    if (ctx->sticky.load() != FCL_SUCCESS) return ctx->sticky.load();
    const uint64_t kid = ++ctx->kid;
    if (nxfer > 0) {
        // the host copies of a pending CPU-only launch go to the device after it, on hd behind
        // the GPU work queued so far (which may still read the old device copies); this launch's
        // GPU work waits on main until the ticket has landed
        Job *t = job_alloc(ctx);
        if (!t) return set_err(ctx, FCL_OUT_OF_RESOURCES, "job allocation");
        t->kind = Job::JOB_XFER;
        t->ticket = ++ctx->xfer_seq;
        t->nx = nxfer;
        for (int q = 0; q < nxfer; ++q) t->xb[q] = xfer[q];
        CK(ctx, cudaEventRecord(t->ev_start, ctx->main));
        {
            std::lock_guard<std::mutex> lk(ctx->q_mu);
            ctx->queue.push_back(t);
            ctx->q_len.fetch_add(1, std::memory_order_release);
        }
        if (ctx->coord_sleeping.load()) ctx->q_cv.notify_all();
        if (!ctx->no_version_wait) {
            const CUresult r = ctx->wait64((CUstream)ctx->main, (CUdeviceptr)ctx->d_xfer, (cuuint64_t)t->ticket,
                                           CU_STREAM_WAIT_VALUE_GEQ);
            if (r != CUDA_SUCCESS) return set_err(ctx, FCL_CUDA_ERROR, "cuStreamWaitValue64 failed (%d)", (int)r);
        }
        ctx->main_fenced.store(1);
        for (int q = 0; q < nxfer; ++q) { xfer[q]->dev_valid = true; xfer[q]->ver_dev = xfer[q]->ver_host; }
    }
    for (int k = 0; k < L.a.nbuf; ++k)   // (the versions this launch produces)
        if (L.acc[k] & 2) L.bufs[k]->ver_expected = kid;

    if (cpu_only && !need_drain) {
        // A CPU-only launch runs in queue order on the coordinator (JOB_CPU).  The host copies it
        // reads must not be overwritten by a lazy return flushed later: flush them now (the job
        // waits for their copies).  Its outputs' device copies are stale from here on.
        for (int k = 0; k < L.a.nbuf; ++k)
            if (L.bufs[k]->ret_lazy) {
                s = flush_returns(ctx, false);
                if (s != FCL_SUCCESS) return s;
                break;
            }
        Job *j = job_alloc(ctx);
        if (!j) return set_err(ctx, FCL_OUT_OF_RESOURCES, "job allocation");
        j->kind = Job::JOB_CPU;
        j->L = L;
        j->host_seq = ++ctx->host_seq;
        j->epoch = (uint32_t)kid;
        fcl_launch_info &info = j->info;
        info.n_wg = L.hi - L.lo; info.wg_lo = L.lo; info.wg_hi = L.hi;
        info.gpu_watermark = info.published_watermark = L.hi;
        info.selected = selected;
        info.seq_host = seq_host;
        for (int k = 0; k < L.a.nbuf; ++k)
            if (L.acc[k] & 2) {
                fcl_buffer b = L.bufs[k];
                b->dev_valid = false;   // lazy H2D (or a JOB_XFER) on the next GPU use
                b->host_seq = j->host_seq;
                b->ver_host = kid;      // (once the job has run: queue order)
            }
        ctx->counts[selected == FCL_SELECTED_CPU ? FCL_COUNT_SEL_CPU : FCL_COUNT_CPU_ONLY] += 1;
        info.t_call_ms = now_ms() - t_call;
        if (info_out) *info_out = info;
        {
            std::lock_guard<std::mutex> lk(ctx->q_mu);
            if (ctx->last && ctx->last != j && ctx->last->done.load()) ctx->free_jobs.push_back(ctx->last);
            ctx->last = j;
            ctx->queue.push_back(j);
            ctx->q_len.fetch_add(1, std::memory_order_release);
        }
        if (ctx->coord_sleeping.load()) ctx->q_cv.notify_all();
        return FCL_SUCCESS;
    }

    if (!coop) {
        ctx->main_tail = nullptr;   // later launches record their own main position
        fcl_launch_info &info = ctx->sync_info;
        std::memset(&info, 0, sizeof info);
        info.n_wg = L.hi - L.lo; info.wg_lo = L.lo; info.wg_hi = L.hi;
        info.gpu_watermark = info.published_watermark = L.hi;
        ctx->sync_have_k = false;
        for (int k = 0; k < L.a.nbuf; ++k) {
            const bool is_out = (L.acc[k] & 2) != 0;
            // GPU-only: the host copy of an output is only rewritten by the return copy (which
            // is ordered behind earlier ones on dh), so it need not be current; CPU-only reads
            // and writes host copies
            const bool need_host = cpu_only;
            const bool need_dev = !cpu_only;
            s = make_valid(ctx, L.bufs[k], need_host, need_dev, &info, is_out);
            if (s != FCL_SUCCESS) return s;
            if (!cpu_only && is_out && (L.acc[k] & 1) && !L.bufs[k]->host_valid) {
                // partially returned in-place outputs: the rest of the host copy must be current
                // first (a pure-OUT one stays stale on the host: the device copy is authoritative)
                s = make_valid(ctx, L.bufs[k], true, true, &info);
                if (s != FCL_SUCCESS) return s;
            }
        }
        if (cpu_only)
            for (int k = 0; k < L.a.nbuf; ++k)
                if (L.acc[k] & 2) { L.bufs[k]->dev_valid = false; L.bufs[k]->ver_host = kid; }
        s = (L.o.mode == FCL_MODE_GPU_ONLY) ? run_gpu_only(ctx, L, info) : run_cpu_only(ctx, L, info);
        for (int k = 0; k < L.a.nbuf && !cpu_only; ++k)
            if (L.acc[k] & 2) { L.bufs[k]->ver_dev = kid; L.bufs[k]->ver_host = kid; }
        info.selected = selected;
        info.seq_host = seq_host;
        ctx->counts[selected == FCL_SELECTED_GPU ? FCL_COUNT_SEL_GPU
                    : selected == FCL_SELECTED_CPU ? FCL_COUNT_SEL_CPU
                    : L.o.mode == FCL_MODE_GPU_ONLY ? FCL_COUNT_GPU_ONLY : FCL_COUNT_CPU_ONLY] += 1;
        info.t_call_ms = now_ms() - t_call;
        {
            std::lock_guard<std::mutex> lk(ctx->q_mu);
            if (ctx->last && ctx->last->done.load()) ctx->free_jobs.push_back(ctx->last);
            ctx->last = nullptr;
        }
        if (info_out) *info_out = info;
        return s;
    }
    for (int k = 0; k < L.a.nbuf; ++k)
        if (L.acc[k] & 2) { L.bufs[k]->ver_dev = kid; L.bufs[k]->ver_host = kid; }

    // lazy returns of buffers whose host copy this launch's host side reads (or that a
    // host-decided merge may change) are queued first; phase B waits for them
    for (int k = 0; k < L.a.nbuf; ++k)
        if (L.bufs[k]->ret_lazy && ((L.acc[k] & 1) || L.o.defer_merge || L.o.forced_split >= 0)) {
            s = flush_returns(ctx, false);
            if (s != FCL_SUCCESS) return s;
            break;
        }

    // cooperative launch: both copies of every argument must be current
    Job *j = job_alloc(ctx);
    if (!j) return set_err(ctx, FCL_OUT_OF_RESOURCES, "job allocation");
    j->L = L;
    j->probe = probe;
    j->probe_gpu_idle = false;
    ctx->counts[FCL_COUNT_COOP] += 1;
    if (probe) ctx->counts[FCL_COUNT_PROBE] += 1;
    if (probe) {
        j->sel_key = select_key(L);
        j->probe_gpu_idle = cudaStreamQuery(ctx->main) == cudaSuccess;
    }
    fcl_launch_info &info = j->info;
    info.selected = FCL_SELECTED_COOP;
    info.probe = probe ? 1 : 0;
    info.n_wg = L.hi - L.lo; info.wg_lo = L.lo; info.wg_hi = L.hi;
    info.gpu_watermark = info.published_watermark = L.hi;
    // Streamed inputs (§6.7): the row-partitioned matrices of a row-dot kernel whose device copy
    // is stale go to the GPU in ascending row pieces while the host computes from the top.
    // (the arrival front must be a stream memop: a store kernel could wait for an SM the
    // grid it signals occupies)
    if (ctx->stream_on && ctx->write64 && (L.a.kernel == K_GESUMMV || L.a.kernel == K_ATAX_TMP || L.a.kernel == K_BICG_Q) &&
        L.g.work_dim == 1 && L.g.lws[0] % 4 == 0 && L.o.forced_split < 0 && !L.o.defer_merge &&
        !L.o.drop_publish) {   // (the GPU waits for pieces or for the watermark: both must come)
        for (int k = 0; k < L.a.nbuf; ++k) {
            fcl_buffer b = L.bufs[k];
            if (L.acc[k] == 1 && !b->dev_valid && required_elems(L.a.kernel, k, L.a.n0, L.a.n1) == L.a.n0 * L.a.n1 &&
                L.a.n1 > 1)
                j->sbuf[j->nstream++] = k;
        }
        j->stream = j->nstream > 0;
        if (j->stream) ctx->stream_jobs.fetch_add(1, std::memory_order_acq_rel);
        j->L.a.streamed = j->stream;
    }
    for (int k = 0; k < L.a.nbuf; ++k) {
        fcl_buffer b = L.bufs[k];
        bool streamed = false;
        for (int q = 0; q < j->nstream; ++q) streamed |= j->sbuf[q] == k;
        // A host copy left stale by a device-side update (fcl_buffer_device_written) is refreshed
        // first when the host side reads it (IN / INOUT; the queue is drained above).  A pure-OUT
        // buffer stays stale on the host: the device copy is complete after the launch, and a
        // read refreshes the host copy from it.
        if (!b->host_valid && (L.acc[k] & 1)) {
            s = make_valid(ctx, b, true, false, &info);
            if (s != FCL_SUCCESS) break;
        }
        // A device copy left stale by a CPU-only launch is refreshed first (lazy H2D; the
        // queue is drained above whenever a copy is stale).
        if (!b->dev_valid && !streamed) {
            s = make_valid(ctx, b, false, true, &info);
            if (s != FCL_SUCCESS) break;
        }
        // A pending return copy of a buffer this launch writes still reads its device copy:
        // order the overwrite behind it on the device; the host side of the hazard is
        // resolved in phase B.
        if (d2h_busy(ctx, b) && (L.acc[k] & 2) && !b->d2h_on_main) {
            const cudaError_t e = cudaStreamWaitEvent(ctx->main, b->d2h_ev, 0);
            ctx->main_fenced.store(1);
            if (e != cudaSuccess) { s = cuda_fail(ctx, e, "stream wait"); break; }
        }
    }
    ctx->tr.add("phaseA_begin", ctx->epoch + 1);
    if (s == FCL_SUCCESS) s = coop_phase_a(ctx, *j);
    ctx->tr.add("phaseA_end", j->epoch);
    if (s != FCL_SUCCESS) {
        job_release_buffers(ctx, *j, false);
        std::lock_guard<std::mutex> lk(ctx->q_mu);
        ctx->free_jobs.push_back(j);
        return s;
    }
    // what is known at return, copied before the coordinator may start writing the job's info
    info.t_call_ms = now_ms() - t_call;
    if (info_out && !L.o.blocking) *info_out = info;
    {
        std::lock_guard<std::mutex> lk(ctx->q_mu);
        if (ctx->last && ctx->last != j && ctx->last->done.load()) ctx->free_jobs.push_back(ctx->last);
        ctx->last = j;
        ctx->queue.push_back(j);
        ctx->q_len.fetch_add(1, std::memory_order_release);
    }
    if (ctx->coord_sleeping.load()) ctx->q_cv.notify_all();
    // (no pool_trim here: cudaFree synchronises the device, and with this job queued the device
    // may be waiting for the coordinator -- a streamed grid for its input pieces, a stream wait
    // for a transfer ticket -- while the coordinator's own CUDA calls wait behind the cudaFree;
    // that deadlock hit the 5 s stream guard.  fcl_finish trims, with nothing in flight.)
    if (L.o.blocking) {
        drain(ctx);
        s = j->status;
        info.t_call_ms = now_ms() - t_call;
        if (info_out) *info_out = info;   // (complete: the host side is done)
    }
    return s;
}

fcl_status fcl_merge(fcl_context ctx, fcl_buffer b) {
    fcl_status s = check_ctx(ctx);
    if (s != FCL_SUCCESS) return s;
    if (!b || b->ctx != ctx) return FCL_INVALID_MEM_OBJECT;
    drain(ctx);
    quiesce(ctx);
    if (!b->merge_pending) return FCL_SUCCESS;
    const char *tw = b->twin ? (const char *)b->twin : (const char *)b->dev;
    if (gpu_launch_merge((char *)b->dev + b->m_b0, (char *)b->stage + b->m_b0, tw + b->m_b0,
                         b->m_b1 - b->m_b0, (int)b->elem_size, ctx->num_sms, ctx->main) < 0)
        return set_err(ctx, FCL_CUDA_ERROR, "%s", gpu_last_error_string());
    ctx->main_tail = nullptr;
    CK(ctx, cudaEventRecord(ctx->ev_mark, ctx->main));
    CK(ctx, cudaStreamWaitEvent(ctx->hd, ctx->ev_mark, 0));   // pool reuse is ordered after the merge
    if (b->r_b1 > b->r_b0) {
        ctx->dh_used.store(1, std::memory_order_relaxed);
        CK(ctx, cudaStreamWaitEvent(ctx->dh, ctx->ev_mark, 0));
        if (d2h_busy(ctx, b) && b->d2h_on_race) CK(ctx, cudaStreamWaitEvent(ctx->dh, b->d2h_ev, 0));
        ctx->counts[FCL_COUNT_D2H_BYTES] += (int64_t)(b->r_b1 - b->r_b0);
        CK(ctx, cudaMemcpyAsync((char *)b->host + b->r_b0, (char *)b->dev + b->r_b0, b->r_b1 - b->r_b0,
                                cudaMemcpyDeviceToHost, ctx->dh));
        CK(ctx, cudaEventRecord(b->d2h_ev, ctx->dh));
        b->d2h_pending = true; b->d2h_on_main = false; b->d2h_on_race = false; b->d2h_gen = ctx->finish_gen.load();
    }
    b->r_b0 = b->r_b1 = 0;
    if (b->twin) pool_put(ctx, b->twin, false);
    pool_put(ctx, b->stage, false);
    b->twin = b->stage = nullptr;
    b->merge_pending = false;
    ctx->defer_list.erase(std::remove(ctx->defer_list.begin(), ctx->defer_list.end(), b), ctx->defer_list.end());
    return FCL_SUCCESS;
}

fcl_status fcl_merge_raw(void *gpu, const void *cpu, const void *twin, size_t bytes, uint32_t elem_size, void *stream) {
    if (!(elem_size == 1 || elem_size == 2 || elem_size == 4 || elem_size == 8) || bytes % elem_size) return FCL_INVALID_VALUE;
    if (bytes && (!gpu || !cpu || !twin)) return FCL_INVALID_VALUE;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (gpu_launch_merge(gpu, cpu, twin, bytes, (int)elem_size, sms, stream) < 0) return FCL_CUDA_ERROR;
    return FCL_SUCCESS;
}

fcl_status fcl_buffer_device_written(fcl_context ctx, fcl_buffer b, size_t offset, size_t n, void *stream) {
    fcl_status s = check_ctx(ctx);
    if (s != FCL_SUCCESS) return s;
    if (!b || b->ctx != ctx) return FCL_INVALID_MEM_OBJECT;
    if (offset > b->bytes || n > b->bytes - offset) return set_err(ctx, FCL_INVALID_VALUE, "range");
    drain(ctx);
    quiesce(ctx);
    if (n == 0) return FCL_SUCCESS;
    if (b->ret_lazy) {   // a registered lazy return would copy the old device words over the new
        b->ret_lazy = false;
        ctx->lazy.erase(std::remove(ctx->lazy.begin(), ctx->lazy.end(), b), ctx->lazy.end());
    }
    if (stream && (cudaStream_t)stream != ctx->main) {   // later work on main follows the writes
        CK(ctx, cudaEventRecord(ctx->ev_mark, (cudaStream_t)stream));
        CK(ctx, cudaStreamWaitEvent(ctx->main, ctx->ev_mark, 0));
    }
    ctx->main_fenced.store(1);
    b->dev_valid = true;
    b->host_valid = false;   // refreshed on demand (make_valid / fcl_read_buffer)
    b->ver_expected = b->ver_dev = ++ctx->kid;
    return FCL_SUCCESS;
}

fcl_status fcl_mirror_upper(void *a, size_t n, uint32_t elem_size, void *stream) {
    if (!(elem_size == 4 || elem_size == 8) || (n > 1 && !a)) return FCL_INVALID_VALUE;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (gpu_launch_mirror_upper(a, (long long)n, (int)elem_size, sms, stream) < 0) return FCL_CUDA_ERROR;
    return FCL_SUCCESS;
}

fcl_status fcl_finish(fcl_context ctx) {
    if (!ctx) return FCL_INVALID_CONTEXT;
    cudaSetDevice(ctx->device);
    ctx->tr.add("finish_begin", ctx->epoch);
    // one batched copy of every lazy return, queued on main right behind the last grid (before
    // the host sides are drained: the device copies it reads are final in stream order, and a
    // host chunk still running only writes the same bits)
    {
        fcl_status f = flush_returns(ctx, true);
        if (f != FCL_SUCCESS) return f;
    }
    // Host sides of lite launches never queue work on main and end when their grid has: with
    // only those pending, main is synchronised first and its completion handed to the
    // coordinator (main_done_epoch), which is how they learn it without an exit word.
    bool all_lite = true, all_returned = true;   // returned: outputs queued at enqueue (eager / lazy)
    {
        std::lock_guard<std::mutex> lk(ctx->q_mu);
        for (Job *p : ctx->queue) {
            all_lite = all_lite && p->lite;
            all_returned = all_returned && (p->eager || p->lazy);
        }
    }
    if (all_lite) {
        CK(ctx, cudaStreamSynchronize(ctx->main));
        ctx->main_done_epoch.store(ctx->epoch, std::memory_order_release);
        ctx->tr.add("finish_main_first", ctx->epoch);
    }
    // Lite host sides still queued end without effect on any buffer (the GPU computed every
    // work-group and their outputs are in the gather just synchronised, or on dh below): they
    // are not waited for -- every call that needs the queue empty drains it, and a chunk one of
    // them may still abandon is quiesced like any other (DESIGN.md §6.4 item 13).
    if (!all_lite || !all_returned) drain(ctx);
    ctx->tr.add("finish_drained", ctx->epoch);
    if (ctx->sticky.load() != FCL_SUCCESS) return ctx->sticky.load();
    // dh first: its return copies are ordered behind the kernels, so by the time it is done
    // main and hd usually are too and their syncs are cheap checks
    if (ctx->dh_used.exchange(0)) CK(ctx, cudaStreamSynchronize(ctx->dh));
    if (ctx->dr_used.exchange(0)) CK(ctx, cudaStreamSynchronize(ctx->dr));
    ctx->finish_gen.fetch_add(1, std::memory_order_acq_rel);   // every queued return copy is done
    ctx->tr.add("finish_dh", ctx->epoch);
    if (!all_lite) {
        CK(ctx, cudaStreamSynchronize(ctx->main));
        ctx->main_done_epoch.store(ctx->epoch, std::memory_order_release);
    }
    ctx->pdl_chain.clear();   // every grid on main has completed
    ctx->pdl_chain_grids = 0;
    ctx->tr.add("finish_main", ctx->epoch);
    if (ctx->hd_used.exchange(0)) CK(ctx, cudaStreamSynchronize(ctx->hd));
    if (ctx->xt_used.exchange(0)) CK(ctx, cudaStreamSynchronize(ctx->xt));
    ctx->tr.add("finish_hd", ctx->epoch);
    // An abandoned chunk of a free-running launch may still be stopping: it only writes words
    // identical to the returned ones, so every host copy is already coherent.  Whatever could
    // change what it reads or writes (buffer I/O, a conflicting or host-side launch, release)
    // waits for it (quiesce); fcl_finish does not.
    CK(ctx, cudaGetLastError());
    // "At the end of each kernel execution, older unused buffers are freed" (L20.s29): here, where
    // every queued launch is done and the device idle, so cudaFree's synchronisation costs nothing
    // and cannot wait for work that waits for the host
    if (ctx->q_len.load(std::memory_order_acquire) == 0) pool_trim(ctx);
    seq_end(ctx);
    ctx->tr.add("finish_end", ctx->epoch);
    if (ctx->tr.on && ctx->stats) {
        unsigned long long st[4 * fcl_context_st::kSlots];
        if (cudaMemcpy(st, ctx->dstamp, sizeof st, cudaMemcpyDeviceToHost) == cudaSuccess) {
            std::lock_guard<std::mutex> lk(ctx->tr.mu);
            for (int k = 0; k < fcl_context_st::kSlots; ++k) {
                static const char *names[4] = {"gpu_disp_start_ns", "gpu_disp_end_ns", "gpu_merge_start_ns", "gpu_merge_end_ns"};
                if (ctx->dpub) {
                    unsigned long long pst = 0;
                    if (cudaMemcpy(&pst, ctx->dpub + k, 8, cudaMemcpyDeviceToHost) == cudaSuccess && pst)
                        ctx->tr.recs.push_back({(double)(pst % 1000000000000ull) * 1e-6, "gpu_publish_ns", (uint32_t)k});
                }
                for (int q = 0; q < 4; ++q)
                    if (st[4 * k + q] && st[4 * k + q] != ~0ull)
                        ctx->tr.recs.push_back({(double)(st[4 * k + q] % 1000000000000ull) * 1e-6, names[q], (uint32_t)k});
            }
        }
        if (ctx->dpstamp && ctx->pst_n > 0) {
            std::vector<unsigned long long> ps(2 * (size_t)ctx->pst_n);
            if (cudaMemcpy(ps.data(), ctx->dpstamp, 16 * (size_t)ctx->pst_n, cudaMemcpyDeviceToHost) == cudaSuccess) {
                std::lock_guard<std::mutex> lk(ctx->tr.mu);
                for (int k = 0; k < ctx->pst_n; ++k) {
                    ctx->tr.recs.push_back({(double)(ps[2 * k] % 1000000000000ull) * 1e-6, "gpu_plain_start_ns", (uint32_t)k});
                    ctx->tr.recs.push_back({(double)(ps[2 * k + 1] % 1000000000000ull) * 1e-6, "gpu_plain_end_ns", (uint32_t)k});
                }
            }
            cudaMemset(ctx->dpstamp, 0, 16 * (size_t)ctx->pst_n);
            cudaDeviceSynchronize();
            ctx->pst_n = 0;
        }
    }
    return FCL_SUCCESS;
}

fcl_status fcl_get_counters(fcl_context ctx, int64_t *counts, int32_t n) {
    if (!ctx) return FCL_INVALID_CONTEXT;
    if (!counts || n < 0) return FCL_INVALID_VALUE;
    for (int32_t k = 0; k < n && k < FCL_COUNT_N; ++k) counts[k] = ctx->counts[k];
    return FCL_SUCCESS;
}

fcl_status fcl_get_launch_info(fcl_context ctx, fcl_launch_info *info) {
    if (!ctx) return FCL_INVALID_CONTEXT;
    if (!info) return FCL_INVALID_VALUE;
    cudaSetDevice(ctx->device);
    drain(ctx);
    Job *j = ctx->last;
    if (!j) {   // the last launch was a single-device one
        if (ctx->sync_have_k) {
            float ms = 0.f;
            if (cudaEventSynchronize(ctx->ev_t1) == cudaSuccess && cudaEventElapsedTime(&ms, ctx->ev_k0, ctx->ev_t1) == cudaSuccess)
                ctx->sync_info.t_gpu_kernel_ms = ms;
        }
        cudaGetLastError();
        *info = ctx->sync_info;
        return FCL_SUCCESS;
    }
    if (j->have_k) {
        float ms = 0.f;
        if (cudaEventSynchronize(j->ev_t1) == cudaSuccess && cudaEventElapsedTime(&ms, j->ev_k0, j->ev_t1) == cudaSuccess)
            j->info.t_gpu_kernel_ms = ms;
    }
    // the watermark of a cooperative launch whose host side did not need it (valid while no
    // later dispatcher has run: this is the most recent launch and the queue is drained) --
    // resolved for every launch, timed or not
    if (j->wm_pending) {
        int64_t wm = j->L.hi;
        if (read_gpu_watermark(ctx, *j, &wm) == FCL_SUCCESS) {
            j->info.gpu_watermark = wm;
            j->info.merged = wm < j->L.hi;
            if (wm <= j->L.lo) j->info.cpu_did_all = 1;
        }
        j->wm_pending = false;
    }
    if (ctx->stats && j->gpu_launched && j->info.gpu_tasks < 0) {
        unsigned long long nt = 0;
        if (cudaMemcpy(&nt, ctx->dtasks + j->slot, 8, cudaMemcpyDeviceToHost) == cudaSuccess)
            j->info.gpu_tasks = (int64_t)nt;
    }
    if (j->have_m) {
        float ms = 0.f;
        if (cudaEventSynchronize(j->ev_m1) == cudaSuccess && cudaEventElapsedTime(&ms, j->ev_m0, j->ev_m1) == cudaSuccess)
            j->info.t_merge_ms = ms;
    }
    cudaGetLastError();
    *info = j->info;
    return FCL_SUCCESS;
}

fcl_status fcl_get_exec_counts(fcl_context ctx, int64_t n, int32_t *gpu_done, int32_t *gpu_frags, int32_t *cpu_done) {
    if (!ctx) return FCL_INVALID_CONTEXT;
    cudaSetDevice(ctx->device);
    drain(ctx);
    quiesce(ctx);
    auto &r = ctx->rec;
    if (!r.valid) return set_err(ctx, FCL_INVALID_VALUE, "no launch recorded execution counts");
    if (n < r.g.n_wg) return set_err(ctx, FCL_INVALID_VALUE, "n %lld < %lld work-groups", (long long)n, (long long)r.g.n_wg);
    CK(ctx, cudaStreamSynchronize(ctx->main));
    const int64_t nt = r.t1 - r.t0;
    std::vector<unsigned int> cnt((size_t)std::max<int64_t>(0, nt)), wm((size_t)std::max<int64_t>(0, nt));
    if (nt > 0) {
        CK(ctx, cudaMemcpy(cnt.data(), r.d_cnt, (size_t)nt * 4, cudaMemcpyDeviceToHost));
        CK(ctx, cudaMemcpy(wm.data(), r.d_w, (size_t)nt * 4, cudaMemcpyDeviceToHost));
    }
    if (gpu_done) std::memset(gpu_done, 0, (size_t)n * 4);
    if (gpu_frags) std::memset(gpu_frags, 0, (size_t)n * 4);
    std::vector<int64_t> wgs;
    for (int64_t t = 0; t < nt; ++t) {
        wgs.clear();
        gpu_task_wgs(r.a, r.g, r.t0 + t, wgs);
        for (int64_t f : wgs) {
            if (f < 0 || f >= r.g.n_wg) continue;
            if (gpu_frags) gpu_frags[f] += 1;
            // a task stores only the work-groups below the watermark it was checked against
            if (gpu_done && cnt[(size_t)t] && (wm[(size_t)t] == 0xFFFFFFFFu || f < (int64_t)wm[(size_t)t]))
                gpu_done[f] += (int32_t)cnt[(size_t)t];
        }
    }
    if (cpu_done) {
        std::memset(cpu_done, 0, (size_t)n * 4);
        for (int64_t f = 0; f < r.g.n_wg; ++f) cpu_done[f] = __atomic_load_n(&r.cpu_done[(size_t)f], __ATOMIC_RELAXED);
    }
    return FCL_SUCCESS;
}

fcl_status fcl_slice_range(fcl_kernel kernel, uint32_t work_dim, const size_t gws[3], const size_t lws[3],
                           int32_t rank, int32_t nranks, int64_t *wg_lo, int64_t *wg_hi) {
    if (!kernel || !gws || !lws || !wg_lo || !wg_hi || nranks < 1 || rank < 0 || rank >= nranks) return FCL_INVALID_VALUE;
    if (work_dim < 1 || work_dim > 3) return FCL_INVALID_WORK_DIMENSION;
    Geom g{};
    g.work_dim = (int)work_dim;
    g.n_wg = 1;
    for (uint32_t d = 0; d < 3; ++d) {
        g.gws[d] = d < work_dim ? (int64_t)gws[d] : 1;
        g.lws[d] = d < work_dim ? (int64_t)lws[d] : 1;
        if (g.lws[d] <= 0 || g.gws[d] % g.lws[d]) return FCL_INVALID_WORK_GROUP_SIZE;
        g.ng[d] = g.gws[d] / g.lws[d];
        g.n_wg *= g.ng[d];
    }
    KArgs a{};
    a.kernel = kernel->def->id;
    a.integer = kernel->def->integer;
    const int64_t al = gpu_slice_align(a, g);
    const int64_t units = (g.n_wg + al - 1) / al;
    const int64_t u0 = units * rank / nranks, u1 = units * (rank + 1) / nranks;
    *wg_lo = std::min<int64_t>(u0 * al, g.n_wg);
    *wg_hi = std::min<int64_t>(u1 * al, g.n_wg);
    return FCL_SUCCESS;
}

}  // extern "C"
