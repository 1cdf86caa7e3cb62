// tsan_driver.cpp -- ThreadSanitizer run over the host side of the runtime (race
// detection): the calling thread, the coordinator thread and the executor's workers exchange
// jobs, claims, abort flags, watermarks and buffer state.  The runtime (runtime.cpp,
// host_bodies.cpp) is compiled with -fsanitize=thread and linked with the sm_100a kernels into
// this driver (scripts/tsan_build.sh); it exercises cooperative launches (free-running with host
// and GPU delays, forced splits, the return race, abandoned chunks, back-to-back asynchronous
// launches with dependencies), CPU-only launches with online profiling and GPU-only launches,
// and checks every result against the GPU-only one bit for bit.
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <vector>

#include "fcl.h"

#define CHECK(x)                                                                                  \
    do {                                                                                          \
        fcl_status s_ = (x);                                                                      \
        if (s_ != FCL_SUCCESS) {                                                                  \
            std::fprintf(stderr, "%s:%d %s -> %s (%s)\n", __FILE__, __LINE__, #x,                 \
                         fcl_status_string(s_), fcl_last_error(ctx));                            \
            std::exit(1);                                                                         \
        }                                                                                         \
    } while (0)

static fcl_context ctx;

struct Prob {
    const char *kernel;
    uint32_t wd;
    size_t gws[3], lws[3];
    std::vector<std::vector<float>> init;   // buffers in signature order
    std::vector<int> out;                   // output buffer indices
    std::vector<int64_t> ints;              // trailing int args
    std::vector<double> floats;             // trailing float args
};

static std::vector<float> rnd(size_t n, unsigned seed) {
    std::mt19937 g(seed);
    std::uniform_real_distribution<float> u(0.f, 1.f);
    std::vector<float> v(n);
    for (auto &x : v) x = u(g);
    return v;
}

// Run p once in `mode` with opts tweaks; returns the host copies of the outputs.
static std::vector<std::vector<float>> run(const Prob &p, int mode, int64_t split, int host_delay, int gpu_delay,
                                           int repeat_async = 1) {
    std::vector<fcl_buffer> bufs;
    for (auto &b : p.init) {
        fcl_buffer h;
        CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, b.size() * 4, 4, b.data(), &h));
        bufs.push_back(h);
    }
    fcl_kernel k;
    CHECK(fcl_get_kernel(ctx, p.kernel, &k));
    std::vector<fcl_arg> args;
    for (size_t q = 0; q < bufs.size(); ++q) {
        fcl_arg a{};
        a.kind = FCL_ARG_BUFFER;
        a.buffer = bufs[q];
        bool is_out = false;
        for (int o : p.out) is_out |= (o == (int)q);
        a.access = is_out ? FCL_ACCESS_INOUT : FCL_ACCESS_IN;
        if (is_out && std::strstr(p.kernel, "syr") == nullptr) a.access = FCL_ACCESS_OUT;
        args.push_back(a);
    }
    for (int64_t v : p.ints) { fcl_arg a{}; a.kind = FCL_ARG_INT; a.i = v; args.push_back(a); }
    for (double v : p.floats) { fcl_arg a{}; a.kind = FCL_ARG_FLOAT; a.f = v; args.push_back(a); }
    fcl_launch_opts o;
    CHECK(fcl_default_launch_opts(&o));
    o.mode = mode;
    o.forced_split = split;
    o.host_delay_us = host_delay;
    o.gpu_delay_us = gpu_delay;
    o.select = FCL_SELECT_OFF;
    for (int r = 0; r < repeat_async; ++r)   // (pure-OUT kernels: the same result every time)
        CHECK(fcl_enqueue_ndrange(ctx, k, p.wd, p.gws, p.lws, args.data(), (uint32_t)args.size(), &o, nullptr));
    CHECK(fcl_finish(ctx));
    std::vector<std::vector<float>> outs;
    for (int oi : p.out) {
        std::vector<float> v(p.init[(size_t)oi].size());
        CHECK(fcl_read_buffer(ctx, bufs[(size_t)oi], 0, v.size() * 4, v.data(), 1));
        outs.push_back(v);
    }
    for (auto b : bufs) CHECK(fcl_release_buffer(b));
    return outs;
}

static int compare(const std::vector<std::vector<float>> &a, const std::vector<std::vector<float>> &b, const char *what) {
    for (size_t q = 0; q < a.size(); ++q)
        if (std::memcmp(a[q].data(), b[q].data(), a[q].size() * 4) != 0) {
            std::fprintf(stderr, "MISMATCH %s output %zu\n", what, q);
            return 1;
        }
    return 0;
}

int main() {
    fcl_context_desc d{};
    d.n_host_threads = 6;
    d.pin_threads = 1;
    CHECK(fcl_create_context(&d, &ctx));
    std::vector<Prob> probs;
    {   // GESUMMV 1024, lws 64: 16 work-groups of row dots, two outputs
        Prob p{"gesummv_f32", 1, {1024, 1, 1}, {64, 1, 1}, {}, {3, 4}, {1024}, {1.5, 1.2}};
        p.init = {rnd(1024 * 1024, 1), rnd(1024 * 1024, 2), rnd(1024, 3), std::vector<float>(1024), std::vector<float>(1024)};
        probs.push_back(p);
    }
    {   // 2DCONV 1000 x 1200: tiles of work-groups, the return race for a large output
        Prob p{"conv2d_f32", 2, {1216, 1000, 1}, {32, 8, 1}, {}, {1}, {1000, 1200}, {}};
        p.init = {rnd(1000 * 1200, 4), std::vector<float>(1000 * 1200)};
        probs.push_back(p);
    }
    {   // SYRK 384 x 96: in place, upper-triangle tiles with mirrors, in-task polls
        Prob p{"syrk_f32", 2, {384, 384, 1}, {32, 8, 1}, {}, {1}, {384, 96}, {1.5, 1.2}};
        p.init = {rnd(384 * 96, 5), rnd(384 * 384, 6)};
        probs.push_back(p);
    }
    {   // column dots: online profiling of two host bodies
        Prob p{"bicg_s_f32", 1, {768, 1, 1}, {32, 1, 1}, {}, {2}, {640, 768}, {}};
        p.init = {rnd(640 * 768, 7), rnd(640, 8), std::vector<float>(768)};
        probs.push_back(p);
    }
    int bad = 0;
    for (auto &p : probs) {
        const auto ref = run(p, FCL_MODE_GPU_ONLY, -1, 0, 0);
        bad += compare(run(p, FCL_MODE_CPU_ONLY, -1, 0, 0), ref, p.kernel);
        for (int rep = 0; rep < 3; ++rep) {
            bad += compare(run(p, FCL_MODE_COOP, -1, 0, 0), ref, p.kernel);
            bad += compare(run(p, FCL_MODE_COOP, -1, 50 * rep, 0), ref, p.kernel);
            bad += compare(run(p, FCL_MODE_COOP, -1, 0, 300 * (rep + 1)), ref, p.kernel);
            bad += compare(run(p, FCL_MODE_COOP, 1 + rep, 0, 0), ref, p.kernel);
        }
        if (p.out.size() && std::strstr(p.kernel, "syr") == nullptr)   // back-to-back asynchronous launches
            bad += compare(run(p, FCL_MODE_COOP, -1, 0, 0, 4), ref, p.kernel);
        std::printf("done %s\n", p.kernel);
        std::fflush(stdout);
    }
    {   // a chain across devices without fcl_finish in between (queued CPU-only jobs, transfers
        // with device-side waits, GPU-only launches ordered like cooperative ones)
        const int64_t n = 512;
        std::vector<float> A = rnd(n * n, 9), x = rnd(n, 10), zero(n);
        fcl_kernel k1, k2;
        CHECK(fcl_get_kernel(ctx, "atax_tmp_f32", &k1));
        CHECK(fcl_get_kernel(ctx, "atax_y_f32", &k2));
        size_t gws[3] = {(size_t)n, 1, 1}, lws[3] = {64, 1, 1};
        std::vector<float> want;
        const int modes[4][2] = {{FCL_MODE_GPU_ONLY, FCL_MODE_GPU_ONLY}, {FCL_MODE_CPU_ONLY, FCL_MODE_GPU_ONLY},
                                 {FCL_MODE_GPU_ONLY, FCL_MODE_CPU_ONLY}, {FCL_MODE_CPU_ONLY, FCL_MODE_COOP}};
        for (auto &md : modes) {
            fcl_buffer bA, bx, bt, by;
            CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, A.size() * 4, 4, A.data(), &bA));
            CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, n * 4, 4, x.data(), &bx));
            CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, n * 4, 4, zero.data(), &bt));
            CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, n * 4, 4, zero.data(), &by));
            fcl_arg a1[5] = {}, a2[5] = {};
            a1[0].kind = a1[1].kind = a1[2].kind = FCL_ARG_BUFFER;
            a1[0].buffer = bA; a1[1].buffer = bx; a1[2].buffer = bt;
            a1[0].access = a1[1].access = FCL_ACCESS_IN; a1[2].access = FCL_ACCESS_OUT;
            a1[3].kind = a1[4].kind = FCL_ARG_INT; a1[3].i = a1[4].i = n;
            std::memcpy(a2, a1, sizeof a1);
            a2[1].buffer = bt; a2[2].buffer = by;
            fcl_launch_opts o;
            CHECK(fcl_default_launch_opts(&o));
            o.select = FCL_SELECT_OFF;
            o.mode = md[0];
            o.host_delay_us = 2000;
            CHECK(fcl_enqueue_ndrange(ctx, k1, 1, gws, lws, a1, 5, &o, nullptr));
            o.mode = md[1];
            o.host_delay_us = 0;
            CHECK(fcl_enqueue_ndrange(ctx, k2, 1, gws, lws, a2, 5, &o, nullptr));
            CHECK(fcl_finish(ctx));
            std::vector<float> y(n);
            CHECK(fcl_read_buffer(ctx, by, 0, n * 4, y.data(), 1));
            if (want.empty()) want = y;
            else if (std::memcmp(want.data(), y.data(), n * 4) != 0) { std::fprintf(stderr, "MISMATCH chain\n"); ++bad; }
            for (auto b : {bA, bx, bt, by}) CHECK(fcl_release_buffer(b));
        }
        std::printf("done chain\n");
    }
    {   // sequence selection: the ATAX 256 chain with device selection on, 60
        // sequences -- host-alone trials, probes on the coordinator, buffer versions between them
        const int64_t n = 256;
        const size_t gws[3] = {256, 1, 1}, lws[3] = {16, 1, 1};
        std::vector<float> A = rnd(n * n, 91), x = rnd(n, 92), zero(n, 0.f), want;
        fcl_kernel k1, k2;
        CHECK(fcl_get_kernel(ctx, "atax_tmp_f32", &k1));
        CHECK(fcl_get_kernel(ctx, "atax_y_f32", &k2));
        fcl_buffer bA, bx, bt, by;
        CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, A.size() * 4, 4, A.data(), &bA));
        CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, n * 4, 4, x.data(), &bx));
        CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, n * 4, 4, zero.data(), &bt));
        CHECK(fcl_create_buffer(ctx, FCL_MEM_READ_WRITE, n * 4, 4, zero.data(), &by));
        fcl_arg a1[5] = {}, a2[5] = {};
        a1[0].kind = a1[1].kind = a1[2].kind = FCL_ARG_BUFFER;
        a1[0].buffer = bA; a1[1].buffer = bx; a1[2].buffer = bt;
        a1[0].access = a1[1].access = FCL_ACCESS_IN; a1[2].access = FCL_ACCESS_OUT;
        a1[3].kind = a1[4].kind = FCL_ARG_INT; a1[3].i = a1[4].i = n;
        std::memcpy(a2, a1, sizeof a1);
        a2[1].buffer = bt; a2[2].buffer = by;
        fcl_launch_opts o;
        CHECK(fcl_default_launch_opts(&o));
        o.select = FCL_SELECT_ON;
        for (int q = 0; q < 60; ++q) {
            CHECK(fcl_enqueue_ndrange(ctx, k1, 1, gws, lws, a1, 5, &o, nullptr));
            CHECK(fcl_enqueue_ndrange(ctx, k2, 1, gws, lws, a2, 5, &o, nullptr));
            CHECK(fcl_finish(ctx));
            std::vector<float> y(n);
            CHECK(fcl_read_buffer(ctx, by, 0, n * 4, y.data(), 1));
            if (want.empty()) want = y;
            else if (std::memcmp(want.data(), y.data(), n * 4) != 0) { std::fprintf(stderr, "MISMATCH sequence %d\n", q); ++bad; }
        }
        int64_t cnt[FCL_COUNT_N];
        CHECK(fcl_get_counters(ctx, cnt, FCL_COUNT_N));
        std::printf("done sequences (seq_host %lld, seq_trials %lld)\n", (long long)cnt[FCL_COUNT_SEQ_HOST],
                    (long long)cnt[FCL_COUNT_SEQ_TRIALS]);
        for (auto b : {bA, bx, bt, by}) CHECK(fcl_release_buffer(b));
    }
    CHECK(fcl_release_context(ctx));
    std::printf(bad ? "tsan driver: %d MISMATCHES\n" : "tsan driver ok\n", bad);
    return bad ? 1 : 0;
}
