// host_bodies.cpp -- the host (CPU) work-group bodies of every built-in kernel.
//
// Fig 7 / L16.s24-25: a CPU work-group executes its kernel code iff its flattened id lies in
// the subkernel's range; the executor (runtime.cpp) only hands in-range ids to these bodies.
// C23 / L20.s34-39: a work-group may be split into `nparts` parts run by different threads;
// the in-scope kernels have no barriers or local memory, so a part is simply a disjoint subset
// of the work-group's work-items (output elements).
//
// Bit-identity with the GPU bodies (kernels.cu): the same IEEE operations in the same order
// (see fcl_internal.h).  This file is compiled with -ffp-contract=off, so `a * b + c` is a
// rounded multiply and a rounded add, and every fused multiply-add is an explicit fmaf().
// Integer instantiations use uint32 arithmetic (two's-complement wraparound, reading R6).
#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "fcl_internal.h"

namespace fcl {

namespace {

inline float op_fma(float a, float b, float c) { return std::fmaf(a, b, c); }
inline uint32_t op_fma(uint32_t a, uint32_t b, uint32_t c) { return a * b + c; }
inline float op_add(float a, float b) { return a + b; }
inline uint32_t op_add(uint32_t a, uint32_t b) { return a + b; }
inline float op_mul(float a, float b) { return a * b; }
inline uint32_t op_mul(uint32_t a, uint32_t b) { return a * b; }

inline bool aborted(const AbortFlag *f) { return f && f->load(std::memory_order_relaxed); }

// [lo, hi) of `n` items for part `part` of `nparts` (contiguous, balanced).
inline void part_range(int64_t n, int part, int nparts, int64_t &lo, int64_t &hi) {
    lo = n * part / nparts;
    hi = n * (part + 1) / nparts;
}

// ---------------------------------------------------------------- row-dot (ATAX k1, BICG k2, GESUMMV)
// Canonical order: 128 column partitions (q = j % 128, ascending j), per-lane fold of 4
// partials, xor-butterfly over 32 lanes.  Mirrors RowDotBody in kernels.cu.
// Returns false (and no value) when the abort flag is seen: it is polled every 1024 columns,
// so an abandoned chunk stops within a fraction of a microsecond.
template <typename T>
bool rowdot(const T *Ar, const T *x, int64_t ncols, const AbortFlag *ab, T *res) {
    T p[kRowPartitions];
    for (int q = 0; q < kRowPartitions; ++q) p[q] = 0;
    for (int64_t j0 = 0; j0 < ncols; j0 += kRowPartitions) {
        if ((j0 & 1023) == 0 && aborted(ab)) return false;
        const int w = (int)std::min<int64_t>(kRowPartitions, ncols - j0);
        const T *a = Ar + j0;
        const T *xv = x + j0;
        for (int q = 0; q < w; ++q) p[q] = op_fma(a[q], xv[q], p[q]);
    }
    T v[32];
    for (int l = 0; l < 32; ++l) v[l] = op_add(op_add(op_add(p[4 * l], p[4 * l + 1]), p[4 * l + 2]), p[4 * l + 3]);
    for (int off = 16; off > 0; off >>= 1)
        for (int l = 0; l < off; ++l) v[l] = op_add(v[l], v[l + off]);
    *res = v[0];
    return true;
}

template <typename T>
bool wg_rowdot(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t lws = g.lws[0];
    const bool ges = (a.kernel == K_GESUMMV);
    const int64_t nrows = a.n0, ncols = ges ? a.n0 : a.n1;
    const int64_t r0 = fgid * lws, r1 = std::min<int64_t>(r0 + lws, nrows);
    if (r0 >= r1) return true;
    int64_t lo, hi;
    part_range(r1 - r0, part, nparts, lo, hi);
    const T *A = (const T *)a.host[0];
    if (!ges) {
        const T *x = (const T *)a.host[1];
        T *out = (T *)a.host[2];
        for (int64_t i = r0 + lo; i < r0 + hi; ++i) {
            T v;
            if (!rowdot<T>(A + i * ncols, x, ncols, ab, &v)) return false;
            out[i] = v;
        }
    } else {
        const T *B = (const T *)a.host[1];
        const T *x = (const T *)a.host[2];
        T *tmp = (T *)a.host[3], *y = (T *)a.host[4];
        const T alpha = a.integer ? (T)(uint32_t)a.ialpha : (T)a.alpha;
        const T beta = a.integer ? (T)(uint32_t)a.ibeta : (T)a.beta;
        for (int64_t i = r0 + lo; i < r0 + hi; ++i) {
            T va, vb;
            if (!rowdot<T>(A + i * ncols, x, ncols, ab, &va) || !rowdot<T>(B + i * ncols, x, ncols, ab, &vb)) return false;
            tmp[i] = va;
            y[i] = op_add(op_mul(alpha, va), op_mul(beta, vb));
        }
    }
    return true;
}

// ---------------------------------------------------------------- col-dot (ATAX k2, BICG k1, CORR mean/std)
// Canonical order: 32 row partitions (q = i % 32, ascending i), then a sequential sum
// q = 0..31.  Mirrors ColDotBody in kernels.cu.
enum { COL_DOT = 0, COL_SUM = 1, COL_SQDEV = 2 };

template <typename T, int MODE>
bool wg_coldot(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t lws = g.lws[0];
    const int64_t nrows = a.n0, ncols = a.n1;
    const int64_t c0 = fgid * lws, c1 = std::min<int64_t>(c0 + lws, ncols);
    if (c0 >= c1) return true;
    int64_t lo, hi;
    part_range(c1 - c0, part, nparts, lo, hi);
    if (lo >= hi) return true;
    const int64_t pc0 = c0 + lo, w = hi - lo;
    const T *A = (const T *)a.host[0];
    const T *v = (MODE == COL_DOT) ? (const T *)a.host[1] : nullptr;
    const T *mean = (MODE == COL_SQDEV) ? (const T *)a.host[1] : nullptr;
    T *out = (T *)a.host[(MODE == COL_SUM) ? 1 : 2];
    thread_local std::vector<T> P;
    P.assign((size_t)kColPartitions * (size_t)w, T(0));
    for (int64_t i = 0; i < nrows; ++i) {
        if ((i & 31) == 0 && aborted(ab)) return false;
        T *pq = P.data() + (size_t)(i & (kColPartitions - 1)) * (size_t)w;
        const T *ar = A + i * ncols + pc0;
        if (MODE == COL_DOT) {
            const T vi = v[i];
            for (int64_t jj = 0; jj < w; ++jj) pq[jj] = op_fma(ar[jj], vi, pq[jj]);
        } else if (MODE == COL_SUM) {
            for (int64_t jj = 0; jj < w; ++jj) pq[jj] = op_add(pq[jj], ar[jj]);
        } else {
            const T *mj = mean + pc0;
            for (int64_t jj = 0; jj < w; ++jj) {
                const T c = op_add(ar[jj], -mj[jj]);
                pq[jj] = op_fma(c, c, pq[jj]);
            }
        }
    }
    for (int64_t jj = 0; jj < w; ++jj) {
        T tot = P[(size_t)jj];
        for (int q = 1; q < kColPartitions; ++q) tot = op_add(tot, P[(size_t)q * (size_t)w + (size_t)jj]);
        if (MODE == COL_DOT) {
            out[pc0 + jj] = tot;
        } else if (MODE == COL_SUM) {
            out[pc0 + jj] = (T)((float)tot / (float)nrows);
        } else {
            const float s = std::sqrt((float)tot / (float)nrows);
            out[pc0 + jj] = (T)((s <= a.eps) ? 1.0f : s);
        }
    }
    return true;
}

// ---------------------------------------------------------------- 2-D work-group geometry helpers
struct Wg2D { int64_t r0, r1, c0, c1; };
inline Wg2D wg2d(const Geom &g, int64_t fgid, int64_t nrows, int64_t ncols) {
    const int64_t gx = fgid % g.ng[0], gy = fgid / g.ng[0];
    Wg2D w;
    w.c0 = gx * g.lws[0]; w.c1 = std::min<int64_t>(w.c0 + g.lws[0], ncols);
    w.r0 = gy * g.lws[1]; w.r1 = std::min<int64_t>(w.r0 + g.lws[1], nrows);
    return w;
}

// ---------------------------------------------------------------- CORR reduce (in place)
// Rectangle [r0, r1) x [c0, c1) of the output (a work-group, or a batch of work-groups of one
// work-group row: wide rows stream and vectorize).
bool corr_reduce_rect(const KArgs &a, int64_t r0, int64_t r1, int64_t c0, int64_t c1, const AbortFlag *ab) {
    const int64_t n = a.n0, m = a.n1;
    float *d = (float *)a.host[0];
    const float *mean = (const float *)a.host[1], *sd = (const float *)a.host[2];
    const float sqrtn = std::sqrt((float)n);
    for (int64_t i = r0; i < r1; ++i) {
        if (aborted(ab)) return false;
        for (int64_t j = c0; j < c1; ++j) {
            const float den = sqrtn * sd[j];
            d[i * m + j] = (d[i * m + j] + (-mean[j])) / den;
        }
    }
    return true;
}

bool wg_corr_reduce(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    Wg2D w = wg2d(g, fgid, a.n0, a.n1);
    if (w.r0 >= w.r1 || w.c0 >= w.c1) return true;
    int64_t lo, hi;
    part_range(w.r1 - w.r0, part, nparts, lo, hi);
    return corr_reduce_rect(a, w.r0 + lo, w.r0 + hi, w.c0, w.c1, ab);
}

// ---------------------------------------------------------------- 2DCONV
// Rectangle [r0, r1) x [c0, c1) of the output, border excluded by the caller.
template <typename T>
bool conv2d_rect(const KArgs &a, int64_t r0, int64_t r1, int64_t c0, int64_t c1, const AbortFlag *ab) {
    const int64_t nj = a.n1;
    const T *A = (const T *)a.host[0];
    T *B = (T *)a.host[1];
    T c[9];
    if (a.integer) {
        const int32_t ci[9] = {2, 5, -8, -3, 6, -9, 4, 7, 1};
        for (int q = 0; q < 9; ++q) c[q] = (T)(uint32_t)ci[q];
    } else {
        const float cf[9] = {0.2f, 0.5f, -0.8f, -0.3f, 0.6f, -0.9f, 0.4f, 0.7f, 0.10f};
        for (int q = 0; q < 9; ++q) c[q] = (T)cf[q];
    }
    for (int64_t i = r0; i < r1; ++i) {
        if (aborted(ab)) return false;
        const T *um = A + (i - 1) * nj, *u0 = A + i * nj, *up = A + (i + 1) * nj;
        for (int64_t j = c0; j < c1; ++j) {
            T s = op_mul(c[0], um[j - 1]);
            s = op_fma(c[3], u0[j - 1], s);
            s = op_fma(c[6], up[j - 1], s);
            s = op_fma(c[1], um[j], s);
            s = op_fma(c[4], u0[j], s);
            s = op_fma(c[7], up[j], s);
            s = op_fma(c[2], um[j + 1], s);
            s = op_fma(c[5], u0[j + 1], s);
            s = op_fma(c[8], up[j + 1], s);
            B[i * nj + j] = s;
        }
    }
    return true;
}

template <typename T>
bool wg_conv2d(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t ni = a.n0, nj = a.n1;
    Wg2D w = wg2d(g, fgid, ni, nj);
    const int64_t r0 = std::max<int64_t>(w.r0, 1), r1 = std::min<int64_t>(w.r1, ni - 1);
    const int64_t c0 = std::max<int64_t>(w.c0, 1), c1 = std::min<int64_t>(w.c1, nj - 1);
    if (r0 >= r1 || c0 >= c1) return true;
    int64_t lo, hi;
    part_range(r1 - r0, part, nparts, lo, hi);
    return conv2d_rect<T>(a, r0 + lo, r0 + hi, c0, c1, ab);
}

// ---------------------------------------------------------------- SYRK / SYR2K
// Each output accumulates its k-chain in ascending k, one fma per term, then
// C = fma(alpha, acc, beta * C).  SYR2K's per-k pair order is symmetric: for i <= j A_i*B_j then
// B_i*A_j, for i > j the mirror's B_i*A_j then A_i*B_j -- so acc(i, j) == acc(j, i) bit for bit
// (DESIGN.md §6.1).  Mirrors GemmBody in kernels.cu.
template <typename T, bool TWO>
bool wg_syrk(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t n = a.n0, m = a.n1;
    Wg2D w = wg2d(g, fgid, n, n);
    if (w.r0 >= w.r1 || w.c0 >= w.c1) return true;
    const int64_t nr = w.r1 - w.r0, nc = w.c1 - w.c0;
    // split the work-group's outputs into (row group x column group) parts
    const int nrg = (int)std::min<int64_t>(nparts, nr);
    const int ncg = (int)std::max<int64_t>(1, std::min<int64_t>(nparts / nrg, (nc + 7) / 8));
    if (part >= nrg * ncg) return true;
    int64_t rlo, rhi, clo, chi;
    part_range(nr, part / ncg, nrg, rlo, rhi);
    part_range(nc, part % ncg, ncg, clo, chi);
    const int64_t j0 = w.c0 + clo, wc = chi - clo;
    if (rlo >= rhi || wc <= 0) return true;
    const T *A = (const T *)a.host[0];
    const T *B = TWO ? (const T *)a.host[1] : nullptr;
    T *C = (T *)a.host[TWO ? 2 : 1];
    const T alpha = a.integer ? (T)(uint32_t)a.ialpha : (T)a.alpha;
    const T beta = a.integer ? (T)(uint32_t)a.ibeta : (T)a.beta;
    // transposed column operands: Xt[k * wc + jj] = X[j0 + jj][k]
    thread_local std::vector<T> At, Bt, acc;
    At.resize((size_t)m * (size_t)wc);
    for (int64_t jj = 0; jj < wc; ++jj) {
        if (aborted(ab)) return false;
        for (int64_t k = 0; k < m; ++k) At[(size_t)(k * wc + jj)] = A[(j0 + jj) * m + k];
    }
    if (TWO) {
        Bt.resize((size_t)m * (size_t)wc);
        for (int64_t jj = 0; jj < wc; ++jj) {
            if (aborted(ab)) return false;
            for (int64_t k = 0; k < m; ++k) Bt[(size_t)(k * wc + jj)] = B[(j0 + jj) * m + k];
        }
    }
    acc.resize((size_t)wc);
    for (int64_t i = w.r0 + rlo; i < w.r0 + rhi; ++i) {
        if (aborted(ab)) return false;
        std::fill(acc.begin(), acc.end(), T(0));
        T *ac = acc.data();
        const T *ai = A + i * m;
        const T *bi = TWO ? B + i * m : nullptr;
        // SYR2K: columns jj < split lie below the diagonal (j < i) and take the mirror's order
        const int64_t split = TWO ? std::min<int64_t>(std::max<int64_t>(i - j0, 0), wc) : 0;
        for (int64_t k = 0; k < m; ++k) {
            if ((k & 511) == 511 && aborted(ab)) return false;   // write-once: nothing stored yet
            const T aik = ai[k];
            if (TWO) {
                const T bik = bi[k];
                const T *bt = Bt.data() + k * wc, *at = At.data() + k * wc;
                for (int64_t jj = 0; jj < split; ++jj) {
                    ac[jj] = op_fma(bik, at[jj], ac[jj]);   // B[i][k] * A[j][k]
                    ac[jj] = op_fma(aik, bt[jj], ac[jj]);   // A[i][k] * B[j][k]
                }
                for (int64_t jj = split; jj < wc; ++jj) {
                    ac[jj] = op_fma(aik, bt[jj], ac[jj]);   // A[i][k] * B[j][k]
                    ac[jj] = op_fma(bik, at[jj], ac[jj]);   // B[i][k] * A[j][k]
                }
            } else {
                const T *at = At.data() + k * wc;
                for (int64_t jj = 0; jj < wc; ++jj) ac[jj] = op_fma(aik, at[jj], ac[jj]);
            }
        }
        T *ci = C + i * n + j0;
        for (int64_t jj = 0; jj < wc; ++jj) ci[jj] = op_fma(alpha, ac[jj], op_mul(beta, ci[jj]));
    }
    return true;
}

// ---------------------------------------------------------------- CORR symmat
// symmat[j1][j2] = symmat[j2][j1] = sum_i d[i][j1] * d[i][j2] (j2 > j1, ascending i, fma
// chain); symmat[j1][j1] = 1.  Work-items j1 processed in blocks of 8 for row reuse.
bool wg_corr_corr(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t n = a.n0, m = a.n1;
    const int64_t lws = g.lws[0];
    const int64_t c0 = fgid * lws, c1 = std::min<int64_t>(c0 + lws, m);
    if (c0 >= c1) return true;
    int64_t lo, hi;
    part_range(c1 - c0, part, nparts, lo, hi);
    const float *d = (const float *)a.host[0];
    float *sym = (float *)a.host[1];
    constexpr int JB = 8;
    thread_local std::vector<float> acc;
    for (int64_t jb = c0 + lo; jb < c0 + hi; jb += JB) {
        const int nb = (int)std::min<int64_t>(JB, c0 + hi - jb);
        const int64_t jstart = jb + 1;               // smallest j2 any member of the block needs
        const int64_t width = m - jstart;
        if (width > 0) {
            acc.assign((size_t)nb * (size_t)width, 0.0f);
            for (int64_t i = 0; i < n; ++i) {
                if ((i & 63) == 0 && aborted(ab)) return false;
                const float *row = d + i * m;
                for (int b = 0; b < nb; ++b) {
                    const int64_t j1 = jb + b;
                    const float a1 = row[j1];
                    float *ac = acc.data() + (size_t)b * (size_t)width;
                    for (int64_t j2 = j1 + 1; j2 < m; ++j2) ac[j2 - jstart] = std::fmaf(a1, row[j2], ac[j2 - jstart]);
                }
            }
        }
        for (int b = 0; b < nb; ++b) {
            const int64_t j1 = jb + b;
            sym[j1 * m + j1] = 1.0f;
            const float *ac = acc.data() + (size_t)b * (size_t)(width > 0 ? width : 0);
            for (int64_t j2 = j1 + 1; j2 < m; ++j2) {
                sym[j1 * m + j2] = ac[j2 - jstart];
                sym[j2 * m + j1] = ac[j2 - jstart];
            }
        }
    }
    return true;
}

// ---------------------------------------------------------------- work-item-order variants
// Alternate host bodies (C26, L22.s4-11): the kernel as written for the GPU, run work-item by
// work-item -- each output element computed on its own with the canonical chain, walking the
// input in the device kernel's (coalescing) order, which strides through host memory.  They
// stand for the unmodified OpenCL kernel a CPU runtime would execute; the bodies above are the
// CPU-oriented versions with interchanged loops (the paper's hand-written CORR kernel, L26.s5-7).
// Both produce bit-identical outputs: loop interchange leaves every output's chain unchanged.

// col-dot: work-item j walks its column, partition by partition
template <typename T, int MODE>
bool wg_coldot_wi(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t lws = g.lws[0];
    const int64_t nrows = a.n0, ncols = a.n1;
    const int64_t c0 = fgid * lws, c1 = std::min<int64_t>(c0 + lws, ncols);
    if (c0 >= c1) return true;
    int64_t lo, hi;
    part_range(c1 - c0, part, nparts, lo, hi);
    const T *A = (const T *)a.host[0];
    const T *v = (MODE == COL_DOT) ? (const T *)a.host[1] : nullptr;
    const T *mean = (MODE == COL_SQDEV) ? (const T *)a.host[1] : nullptr;
    T *out = (T *)a.host[(MODE == COL_SUM) ? 1 : 2];
    for (int64_t j = c0 + lo; j < c0 + hi; ++j) {
        if (aborted(ab)) return false;
        const T mj = (MODE == COL_SQDEV) ? mean[j] : T(0);
        T tot = 0;
        for (int q = 0; q < kColPartitions; ++q) {
            T acc = 0;
            for (int64_t i = q; i < nrows; i += kColPartitions) {
                const T x = A[i * ncols + j];
                if (MODE == COL_DOT) acc = op_fma(x, v[i], acc);
                else if (MODE == COL_SUM) acc = op_add(acc, x);
                else { const T c = op_add(x, -mj); acc = op_fma(c, c, acc); }
            }
            tot = (q == 0) ? acc : op_add(tot, acc);
        }
        if (MODE == COL_DOT) out[j] = tot;
        else if (MODE == COL_SUM) out[j] = (T)((float)tot / (float)nrows);
        else {
            const float s = std::sqrt((float)tot / (float)nrows);
            out[j] = (T)((s <= a.eps) ? 1.0f : s);
        }
    }
    return true;
}

// SYRK / SYR2K: work-item (i, j) runs its k-chain
template <typename T, bool TWO>
bool wg_syrk_wi(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t n = a.n0, m = a.n1;
    Wg2D w = wg2d(g, fgid, n, n);
    if (w.r0 >= w.r1 || w.c0 >= w.c1) return true;
    const int64_t nc = w.c1 - w.c0, nitems = (w.r1 - w.r0) * nc;
    int64_t lo, hi;
    part_range(nitems, part, nparts, lo, hi);
    const T *A = (const T *)a.host[0];
    const T *B = TWO ? (const T *)a.host[1] : nullptr;
    T *C = (T *)a.host[TWO ? 2 : 1];
    const T alpha = a.integer ? (T)(uint32_t)a.ialpha : (T)a.alpha;
    const T beta = a.integer ? (T)(uint32_t)a.ibeta : (T)a.beta;
    for (int64_t it = lo; it < hi; ++it) {
        if ((it & 15) == 0 && aborted(ab)) return false;
        const int64_t i = w.r0 + it / nc, j = w.c0 + it % nc;
        const T *ai = A + i * m, *aj = A + j * m;
        const T *bi = TWO ? B + i * m : nullptr, *bj = TWO ? B + j * m : nullptr;
        T acc = 0;
        for (int64_t k = 0; k < m; ++k) {
            if (TWO && i > j) {                    // below the diagonal: the mirror's order
                acc = op_fma(bi[k], aj[k], acc);   // B[i][k] * A[j][k]
                acc = op_fma(ai[k], bj[k], acc);   // A[i][k] * B[j][k]
            } else if (TWO) {
                acc = op_fma(ai[k], bj[k], acc);   // A[i][k] * B[j][k]
                acc = op_fma(bi[k], aj[k], acc);   // B[i][k] * A[j][k]
            } else {
                acc = op_fma(ai[k], aj[k], acc);
            }
        }
        C[i * n + j] = op_fma(alpha, acc, op_mul(beta, C[i * n + j]));
    }
    return true;
}

// CORR symmat: work-item j1 computes its row, each j2 > j1 down the two columns
bool wg_corr_corr_wi(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *ab) {
    const int64_t n = a.n0, m = a.n1;
    const int64_t lws = g.lws[0];
    const int64_t c0 = fgid * lws, c1 = std::min<int64_t>(c0 + lws, m);
    if (c0 >= c1) return true;
    int64_t lo, hi;
    part_range(c1 - c0, part, nparts, lo, hi);
    const float *d = (const float *)a.host[0];
    float *sym = (float *)a.host[1];
    for (int64_t j1 = c0 + lo; j1 < c0 + hi; ++j1) {
        sym[j1 * m + j1] = 1.0f;
        for (int64_t j2 = j1 + 1; j2 < m; ++j2) {
            if ((j2 & 15) == 0 && aborted(ab)) return false;
            float acc = 0.0f;
            for (int64_t i = 0; i < n; ++i) acc = std::fmaf(d[i * m + j1], d[i * m + j2], acc);
            sym[j1 * m + j2] = acc;
            sym[j2 * m + j1] = acc;
        }
    }
    return true;
}

}  // namespace

int host_num_variants(int kernel) {
    switch (kernel) {
    case K_ATAX_Y: case K_BICG_S: case K_CORR_MEAN: case K_CORR_STD:
    case K_SYRK: case K_SYR2K: case K_CORR_CORR:
        return 2;
    default:
        return 1;   // the work-item order is already the CPU-friendly one
    }
}

const char *host_variant_name(int kernel, int v) {
    if (host_num_variants(kernel) == 1) return "wi";
    return v == 0 ? "cpu" : "wi";
}

bool host_exec_wg(const KArgs &a, const Geom &g, int64_t fgid, int part, int nparts, const AbortFlag *abort_flag) {
    if (a.host_variant == 1 && host_num_variants(a.kernel) > 1) {
        switch (a.kernel) {
        case K_ATAX_Y: case K_BICG_S:
            if (a.integer) return wg_coldot_wi<uint32_t, COL_DOT>(a, g, fgid, part, nparts, abort_flag);
            return wg_coldot_wi<float, COL_DOT>(a, g, fgid, part, nparts, abort_flag);
        case K_CORR_MEAN: return wg_coldot_wi<float, COL_SUM>(a, g, fgid, part, nparts, abort_flag);
        case K_CORR_STD: return wg_coldot_wi<float, COL_SQDEV>(a, g, fgid, part, nparts, abort_flag);
        case K_SYRK:
            if (a.integer) return wg_syrk_wi<uint32_t, false>(a, g, fgid, part, nparts, abort_flag);
            return wg_syrk_wi<float, false>(a, g, fgid, part, nparts, abort_flag);
        case K_SYR2K:
            if (a.integer) return wg_syrk_wi<uint32_t, true>(a, g, fgid, part, nparts, abort_flag);
            return wg_syrk_wi<float, true>(a, g, fgid, part, nparts, abort_flag);
        case K_CORR_CORR: return wg_corr_corr_wi(a, g, fgid, part, nparts, abort_flag);
        default: break;
        }
    }
    switch (a.kernel) {
    case K_ATAX_TMP: case K_BICG_Q: case K_GESUMMV:
        if (a.integer) return wg_rowdot<uint32_t>(a, g, fgid, part, nparts, abort_flag);
        return wg_rowdot<float>(a, g, fgid, part, nparts, abort_flag);
    case K_ATAX_Y: case K_BICG_S:
        if (a.integer) return wg_coldot<uint32_t, COL_DOT>(a, g, fgid, part, nparts, abort_flag);
        return wg_coldot<float, COL_DOT>(a, g, fgid, part, nparts, abort_flag);
    case K_CORR_MEAN: return wg_coldot<float, COL_SUM>(a, g, fgid, part, nparts, abort_flag);
    case K_CORR_STD: return wg_coldot<float, COL_SQDEV>(a, g, fgid, part, nparts, abort_flag);
    case K_CORR_REDUCE: return wg_corr_reduce(a, g, fgid, part, nparts, abort_flag);
    case K_CORR_CORR: return wg_corr_corr(a, g, fgid, part, nparts, abort_flag);
    case K_CONV2D:
        if (a.integer) return wg_conv2d<uint32_t>(a, g, fgid, part, nparts, abort_flag);
        return wg_conv2d<float>(a, g, fgid, part, nparts, abort_flag);
    case K_SYRK:
        if (a.integer) return wg_syrk<uint32_t, false>(a, g, fgid, part, nparts, abort_flag);
        return wg_syrk<float, false>(a, g, fgid, part, nparts, abort_flag);
    case K_SYR2K:
        if (a.integer) return wg_syrk<uint32_t, true>(a, g, fgid, part, nparts, abort_flag);
        return wg_syrk<float, true>(a, g, fgid, part, nparts, abort_flag);
    default: return true;
    }
}

// Work-groups per executor claim: 2-D row-major bodies take runs of work-groups of one
// work-group row as one wide rectangle (2048 columns); the others one work-group at a time.
int64_t host_batch(const KArgs &a, const Geom &g) {
    if ((a.kernel == K_CONV2D || a.kernel == K_CORR_REDUCE) && g.work_dim == 2)
        return std::max<int64_t>(1, 2048 / g.lws[0]);
    return 1;
}

// Work-groups [f_lo, f_hi) (any order is valid: every work-group writes only its own outputs).
// Returns true when every one of them completed (false: the abort flag stopped the run).
bool host_exec_range(const KArgs &a, const Geom &g, int64_t f_lo, int64_t f_hi, const AbortFlag *ab) {
    if ((a.kernel == K_CONV2D || a.kernel == K_CORR_REDUCE) && g.work_dim == 2) {
        const int64_t ngx = g.ng[0];
        for (int64_t f = f_lo; f < f_hi;) {   // one segment per work-group row
            const int64_t gy = f / ngx, gx0 = f % ngx;
            const int64_t gx1 = std::min<int64_t>(ngx, gx0 + (f_hi - f));
            Wg2D w0 = wg2d(g, f, a.n0, a.n1);
            const int64_t c1 = std::min<int64_t>(gx1 * g.lws[0], a.n1);
            bool ok = true;
            if (a.kernel == K_CORR_REDUCE) {
                ok = corr_reduce_rect(a, w0.r0, w0.r1, w0.c0, c1, ab);
            } else {
                const int64_t r0 = std::max<int64_t>(w0.r0, 1), r1 = std::min<int64_t>(w0.r1, a.n0 - 1);
                const int64_t c0 = std::max<int64_t>(w0.c0, 1), cc1 = std::min<int64_t>(c1, a.n1 - 1);
                if (r0 < r1 && c0 < cc1) {
                    if (a.integer) ok = conv2d_rect<uint32_t>(a, r0, r1, c0, cc1, ab);
                    else ok = conv2d_rect<float>(a, r0, r1, c0, cc1, ab);
                }
            }
            if (!ok) return false;
            f = gy * ngx + gx1;
        }
        return true;
    }
    for (int64_t f = f_hi - 1; f >= f_lo; --f) {
        if (aborted(ab)) return false;
        if (!host_exec_wg(a, g, f, 0, 1, ab)) return false;
    }
    return true;
}

// Conservative contiguous output span of work-groups [lo, hi) (see fcl_internal.h).
void out_span(const KArgs &a, const Geom &g, int k, int64_t lo, int64_t hi, size_t *b0, size_t *b1) {
    *b0 = *b1 = 0;
    if (hi <= lo) return;
    const size_t es = 4;
    auto one_d = [&](int64_t n) {
        const int64_t e0 = std::min<int64_t>(lo * g.lws[0], n), e1 = std::min<int64_t>(hi * g.lws[0], n);
        *b0 = (size_t)e0 * es; *b1 = (size_t)e1 * es;
    };
    auto two_d = [&](int64_t nrows, int64_t ncols) {
        const int64_t ngx = g.ng[0];
        const int64_t gy0 = lo / ngx, gy1 = (hi + ngx - 1) / ngx;
        const int64_t r0 = std::min<int64_t>(gy0 * g.lws[1], nrows), r1 = std::min<int64_t>(gy1 * g.lws[1], nrows);
        *b0 = (size_t)(r0 * ncols) * es; *b1 = (size_t)(r1 * ncols) * es;
    };
    switch (a.kernel) {
    case K_ATAX_TMP: case K_BICG_Q: one_d(a.n0); break;
    case K_GESUMMV: one_d(a.n0); break;
    case K_ATAX_Y: case K_BICG_S: case K_CORR_MEAN: case K_CORR_STD: one_d(a.n1); break;
    case K_SYRK: case K_SYR2K: two_d(a.n0, a.n0); break;
    case K_CORR_REDUCE: case K_CONV2D: two_d(a.n0, a.n1); break;
    case K_CORR_CORR: *b0 = 0; *b1 = (size_t)(a.n1 * a.n1) * es; break;   // row + column: whole buffer
    default: break;
    }
    (void)k;
}

void out_span_desc(const KArgs &a, const Geom &g, int k, long long *unit_wgs, long long *unit_bytes,
                   long long *total) {
    (void)k;
    const long long es = 4;
    switch (a.kernel) {
    case K_ATAX_TMP: case K_BICG_Q: case K_GESUMMV:
        *unit_wgs = 1; *unit_bytes = g.lws[0] * es; *total = a.n0 * es; break;
    case K_ATAX_Y: case K_BICG_S: case K_CORR_MEAN: case K_CORR_STD:
        *unit_wgs = 1; *unit_bytes = g.lws[0] * es; *total = a.n1 * es; break;
    case K_SYRK: case K_SYR2K:
        *unit_wgs = g.ng[0]; *unit_bytes = g.lws[1] * a.n0 * es; *total = a.n0 * a.n0 * es; break;
    case K_CORR_REDUCE: case K_CONV2D:
        *unit_wgs = g.ng[0]; *unit_bytes = g.lws[1] * a.n1 * es; *total = a.n0 * a.n1 * es; break;
    case K_CORR_CORR:
    default:
        *unit_wgs = 0; *unit_bytes = 0; *total = a.n1 * a.n1 * es; break;
    }
}

}  // namespace fcl
