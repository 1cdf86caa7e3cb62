/*
 * oracle.c -- plain, slow, serial CPU oracle for the FluidiCL hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (paper_conf_cgo_panditg14_b200/) never links, imports or
 * executes anything under oracle/; the two share no code, headers, tables or
 * constants.  Everything here is written out from the paper
 * (/root/reference/PAPER.md, cited as L<line>.s<sentence>)
 * and, for the benchmark kernels the paper only names, from the standard
 * PolyBench(/GPU) definitions (the paper cites "Polybench [15]", L22.s26; its
 * reference list is on the missing page 10 -- readings R1..R9 in DESIGN.md).
 *
 * Precision: the paper never fixes one, so floating-point kernels run in
 * fp64 on fp64 copies of the fp32 inputs; integer kernels run in uint32
 * two's-complement wraparound (reading R6).  No blocking, fusion or
 * reordering: every work-item is the textbook loop in ascending index order.
 *
 * Parity status of every function is pinned by tests/test_oracle_*.py (the
 * pins are listed in DESIGN.md §3); nothing here is "parity unpinned".
 */
#include <stdint.h>
#include <stddef.h>
#include <string.h>
#include <math.h>

/* ------------------------------------------------------------------------ */
/* Kernel identifiers (the oracle's own numbering).                          */
/* ------------------------------------------------------------------------ */
enum {
    OK_ATAX_TMP = 0,   /* tmp[i] = sum_j A[i][j] x[j]            (PolyBench atax, kernel 1) */
    OK_ATAX_Y = 1,     /* y[j]   = sum_i A[i][j] tmp[i]          (PolyBench atax, kernel 2) */
    OK_BICG_S = 2,     /* s[j]   = sum_i r[i] A[i][j]            (PolyBench bicg, kernel 1) */
    OK_BICG_Q = 3,     /* q[i]   = sum_j A[i][j] p[j]            (PolyBench bicg, kernel 2) */
    OK_GESUMMV = 4,    /* tmp = A x; y = alpha tmp + beta B x    (PolyBench gesummv)        */
    OK_SYRK = 5,       /* C = beta C + alpha A A^T               (PolyBench syrk, full NxN) */
    OK_SYR2K = 6,      /* C = beta C + alpha A B^T + alpha B A^T (PolyBench syr2k)          */
    OK_CORR_MEAN = 7,  /* mean[j] = sum_i d[i][j] / n            (PolyBench correlation)    */
    OK_CORR_STD = 8,   /* std[j]  = sqrt(sum_i (d-mean)^2 / n), 1 if <= eps                 */
    OK_CORR_REDUCE = 9,/* d[i][j] = (d[i][j]-mean[j]) / (sqrt(n) std[j])                    */
    OK_CORR_CORR = 10, /* symmat[j1][j2] = symmat[j2][j1] = sum_i d[i][j1] d[i][j2]         */
    OK_CONV2D = 11,    /* 3x3 stencil, interior only             (PolyBench/GPU 2DCONV)     */
    OK_NUM_KERNELS = 12
};

/*
 * One kernel launch as the oracle sees it.  Buffer order per kernel:
 *   ATAX_TMP : A[n0*n1], x[n1], tmp[n0]            work-items i < n0   (1-D)
 *   ATAX_Y   : A[n0*n1], tmp[n0], y[n1]            work-items j < n1   (1-D)
 *   BICG_S   : A[n0*n1], r[n0], s[n1]              work-items j < n1   (1-D)
 *   BICG_Q   : A[n0*n1], p[n1], q[n0]              work-items i < n0   (1-D)
 *   GESUMMV  : A[n0*n0], B[n0*n0], x[n0], tmp[n0], y[n0]   i < n0      (1-D)
 *   SYRK     : A[n0*n1], C[n0*n0]                  (j, i) < (n0, n0)   (2-D, dim0 = j)
 *   SYR2K    : A[n0*n1], B[n0*n1], C[n0*n0]        (j, i) < (n0, n0)   (2-D, dim0 = j)
 *   CORR_MEAN: data[n0*n1], mean[n1]               j < n1              (1-D)
 *   CORR_STD : data[n0*n1], mean[n1], std[n1]      j < n1              (1-D)
 *   CORR_RED : data[n0*n1], mean[n1], std[n1]      (j, i) < (n1, n0)   (2-D, dim0 = j)
 *   CORR_CORR: data[n0*n1], symmat[n1*n1]          j1 < n1             (1-D)
 *   CONV2D   : A[n0*n1], B[n0*n1]                  (j, i) < (n1, n0)   (2-D, dim0 = j)
 * n0 = rows, n1 = columns of the row-major input matrix (for SYRK/SYR2K:
 * n0 = N, n1 = M).  For dtype 0 buffers are double*, for dtype 1 uint32_t*.
 */
typedef struct {
    int32_t kernel;
    int32_t dtype;          /* 0: fp64 arithmetic, 1: uint32 wraparound */
    int64_t n0, n1;
    int32_t work_dim;
    int64_t gws[3], lws[3];
    double alpha, beta, eps; /* fp scalars (alpha/beta: GESUMMV/SYRK/SYR2K; eps: CORR) */
    uint32_t ialpha, ibeta;  /* integer scalars */
    void *buf[6];
    uint32_t *wcount[6];     /* optional per-element write counters (exactly-once model) */
} oracle_launch;

/* ------------------------------------------------------------------------ */
/* C7 / Fig 5 (L14.s24-31): flattened work-group id.                         */
/* Reading R2: dimension 0 (the column in Fig 5) is fastest:     */
/*   fgid = g0 + ng0 * (g1 + ng1 * g2).                                       */
/* ------------------------------------------------------------------------ */
int64_t oracle_num_groups_dim(int64_t gws, int64_t lws)
{
    /* ng = ceil(gws / lws) (OpenCL 1.x requires gws % lws == 0,
       PolyBench pads gws, so both coincide on every launch we issue). */
    return (gws + lws - 1) / lws;
}

int64_t oracle_num_groups(const oracle_launch *L)
{
    int64_t n = 1;
    for (int d = 0; d < L->work_dim; ++d) n *= oracle_num_groups_dim(L->gws[d], L->lws[d]);
    return n;
}

int64_t oracle_flatten(int32_t work_dim, const int64_t ng[3], const int64_t g[3])
{
    int64_t f = 0;
    for (int d = work_dim - 1; d >= 0; --d) f = f * ng[d] + g[d];
    return f;
}

void oracle_unflatten(int32_t work_dim, const int64_t ng[3], int64_t fgid, int64_t g[3])
{
    g[0] = g[1] = g[2] = 0;
    for (int d = 0; d < work_dim; ++d) { g[d] = fgid % ng[d]; fgid /= ng[d]; }
}

/* ------------------------------------------------------------------------ */
/* Work-item bodies.  Each computes its value into a local and stores it     */
/* once (the write-once reading R5 / SURVEY H4, S13).                         */
/* ------------------------------------------------------------------------ */
#define WC(k, idx) do { if (L->wcount[k]) L->wcount[k][idx] += 1u; } while (0)

static void wi_atax_tmp(const oracle_launch *L, int64_t i)
{
    const int64_t nx = L->n0, ny = L->n1;
    if (i >= nx) return;
    if (L->dtype == 0) {
        const double *A = L->buf[0], *x = L->buf[1]; double *tmp = L->buf[2];
        double s = 0.0;
        for (int64_t j = 0; j < ny; ++j) s += A[i * ny + j] * x[j];
        tmp[i] = s;
    } else {
        const uint32_t *A = L->buf[0], *x = L->buf[1]; uint32_t *tmp = L->buf[2];
        uint32_t s = 0;
        for (int64_t j = 0; j < ny; ++j) s += A[i * ny + j] * x[j];
        tmp[i] = s;
    }
    WC(2, i);
}

static void wi_atax_y(const oracle_launch *L, int64_t j)
{
    const int64_t nx = L->n0, ny = L->n1;
    if (j >= ny) return;
    if (L->dtype == 0) {
        const double *A = L->buf[0], *tmp = L->buf[1]; double *y = L->buf[2];
        double s = 0.0;
        for (int64_t i = 0; i < nx; ++i) s += A[i * ny + j] * tmp[i];
        y[j] = s;
    } else {
        const uint32_t *A = L->buf[0], *tmp = L->buf[1]; uint32_t *y = L->buf[2];
        uint32_t s = 0;
        for (int64_t i = 0; i < nx; ++i) s += A[i * ny + j] * tmp[i];
        y[j] = s;
    }
    WC(2, j);
}

static void wi_bicg_s(const oracle_launch *L, int64_t j)
{
    const int64_t nx = L->n0, ny = L->n1;
    if (j >= ny) return;
    if (L->dtype == 0) {
        const double *A = L->buf[0], *r = L->buf[1]; double *s = L->buf[2];
        double acc = 0.0;
        for (int64_t i = 0; i < nx; ++i) acc += r[i] * A[i * ny + j];
        s[j] = acc;
    } else {
        const uint32_t *A = L->buf[0], *r = L->buf[1]; uint32_t *s = L->buf[2];
        uint32_t acc = 0;
        for (int64_t i = 0; i < nx; ++i) acc += r[i] * A[i * ny + j];
        s[j] = acc;
    }
    WC(2, j);
}

static void wi_bicg_q(const oracle_launch *L, int64_t i)
{
    const int64_t nx = L->n0, ny = L->n1;
    if (i >= nx) return;
    if (L->dtype == 0) {
        const double *A = L->buf[0], *p = L->buf[1]; double *q = L->buf[2];
        double acc = 0.0;
        for (int64_t j = 0; j < ny; ++j) acc += A[i * ny + j] * p[j];
        q[i] = acc;
    } else {
        const uint32_t *A = L->buf[0], *p = L->buf[1]; uint32_t *q = L->buf[2];
        uint32_t acc = 0;
        for (int64_t j = 0; j < ny; ++j) acc += A[i * ny + j] * p[j];
        q[i] = acc;
    }
    WC(2, i);
}

static void wi_gesummv(const oracle_launch *L, int64_t i)
{
    const int64_t n = L->n0;
    if (i >= n) return;
    if (L->dtype == 0) {
        const double *A = L->buf[0], *B = L->buf[1], *x = L->buf[2];
        double *tmp = L->buf[3], *y = L->buf[4];
        double t = 0.0, u = 0.0;
        for (int64_t j = 0; j < n; ++j) { t += A[i * n + j] * x[j]; u += B[i * n + j] * x[j]; }
        tmp[i] = t;
        y[i] = L->alpha * t + L->beta * u;
    } else {
        const uint32_t *A = L->buf[0], *B = L->buf[1], *x = L->buf[2];
        uint32_t *tmp = L->buf[3], *y = L->buf[4];
        uint32_t t = 0, u = 0;
        for (int64_t j = 0; j < n; ++j) { t += A[i * n + j] * x[j]; u += B[i * n + j] * x[j]; }
        tmp[i] = t;
        y[i] = L->ialpha * t + L->ibeta * u;
    }
    WC(3, i); WC(4, i);
}

static void wi_syrk(const oracle_launch *L, int64_t j, int64_t i)
{
    const int64_t n = L->n0, m = L->n1;
    if (i >= n || j >= n) return;
    if (L->dtype == 0) {
        const double *A = L->buf[0]; double *C = L->buf[1];
        double s = 0.0;
        for (int64_t k = 0; k < m; ++k) s += A[i * m + k] * A[j * m + k];
        C[i * n + j] = L->beta * C[i * n + j] + L->alpha * s;
    } else {
        const uint32_t *A = L->buf[0]; uint32_t *C = L->buf[1];
        uint32_t s = 0;
        for (int64_t k = 0; k < m; ++k) s += A[i * m + k] * A[j * m + k];
        C[i * n + j] = L->ibeta * C[i * n + j] + L->ialpha * s;
    }
    WC(1, i * n + j);
}

static void wi_syr2k(const oracle_launch *L, int64_t j, int64_t i)
{
    const int64_t n = L->n0, m = L->n1;
    if (i >= n || j >= n) return;
    if (L->dtype == 0) {
        const double *A = L->buf[0], *B = L->buf[1]; double *C = L->buf[2];
        double s = 0.0;
        for (int64_t k = 0; k < m; ++k)
            s += L->alpha * A[i * m + k] * B[j * m + k] + L->alpha * B[i * m + k] * A[j * m + k];
        C[i * n + j] = L->beta * C[i * n + j] + s;
    } else {
        const uint32_t *A = L->buf[0], *B = L->buf[1]; uint32_t *C = L->buf[2];
        uint32_t s = 0;
        for (int64_t k = 0; k < m; ++k)
            s += L->ialpha * A[i * m + k] * B[j * m + k] + L->ialpha * B[i * m + k] * A[j * m + k];
        C[i * n + j] = L->ibeta * C[i * n + j] + s;
    }
    WC(2, i * n + j);
}

/* CORR: n0 = N data points (rows), n1 = M variables (columns).  Reading R7:
   float_n = N, eps = L->eps (0.1 by default), PolyBench/C convention. */
static void wi_corr_mean(const oracle_launch *L, int64_t j)
{
    const int64_t n = L->n0, m = L->n1;
    if (j >= m) return;
    const double *d = L->buf[0]; double *mean = L->buf[1];
    double s = 0.0;
    for (int64_t i = 0; i < n; ++i) s += d[i * m + j];
    mean[j] = s / (double)n;
    WC(1, j);
}

static void wi_corr_std(const oracle_launch *L, int64_t j)
{
    const int64_t n = L->n0, m = L->n1;
    if (j >= m) return;
    const double *d = L->buf[0], *mean = L->buf[1]; double *sd = L->buf[2];
    double s = 0.0;
    for (int64_t i = 0; i < n; ++i) { double c = d[i * m + j] - mean[j]; s += c * c; }
    double v = sqrt(s / (double)n);
    sd[j] = (v <= L->eps) ? 1.0 : v;
    WC(2, j);
}

static void wi_corr_reduce(const oracle_launch *L, int64_t j, int64_t i)
{
    const int64_t n = L->n0, m = L->n1;
    if (i >= n || j >= m) return;
    double *d = L->buf[0]; const double *mean = L->buf[1], *sd = L->buf[2];
    d[i * m + j] = (d[i * m + j] - mean[j]) / (sqrt((double)n) * sd[j]);
    WC(0, i * m + j);
}

static void wi_corr_corr(const oracle_launch *L, int64_t j1)
{
    const int64_t n = L->n0, m = L->n1;
    if (j1 >= m) return;
    const double *d = L->buf[0]; double *sym = L->buf[1];
    sym[j1 * m + j1] = 1.0;
    WC(1, j1 * m + j1);
    for (int64_t j2 = j1 + 1; j2 < m; ++j2) {
        double s = 0.0;
        for (int64_t i = 0; i < n; ++i) s += d[i * m + j1] * d[i * m + j2];
        sym[j1 * m + j2] = s;
        sym[j2 * m + j1] = s;
        WC(1, j1 * m + j2); WC(1, j2 * m + j1);
    }
}

/* 2DCONV (PolyBench/GPU 2DConvolution; not in the paper -- reading R8).
   c[a][b] multiplies A[i + a - 1][j + b - 1]. */
static const double conv_c_f[3][3] = {
    /* row offset -1 */ { +0.2, +0.5, -0.8 },
    /* row offset  0 */ { -0.3, +0.6, -0.9 },
    /* row offset +1 */ { +0.4, +0.7, +0.10 },
};
static const int32_t conv_c_i[3][3] = {
    { 2, 5, -8 },
    { -3, 6, -9 },
    { 4, 7, 1 },
};

static void wi_conv2d(const oracle_launch *L, int64_t j, int64_t i)
{
    const int64_t ni = L->n0, nj = L->n1;
    if (i < 1 || i >= ni - 1 || j < 1 || j >= nj - 1) return; /* border untouched */
    if (L->dtype == 0) {
        const double *A = L->buf[0]; double *B = L->buf[1];
        double s = 0.0;
        for (int a = 0; a < 3; ++a)
            for (int b = 0; b < 3; ++b)
                s += conv_c_f[a][b] * A[(i + a - 1) * nj + (j + b - 1)];
        B[i * nj + j] = s;
    } else {
        const uint32_t *A = L->buf[0]; uint32_t *B = L->buf[1];
        uint32_t s = 0;
        for (int a = 0; a < 3; ++a)
            for (int b = 0; b < 3; ++b)
                s += (uint32_t)conv_c_i[a][b] * A[(i + a - 1) * nj + (j + b - 1)];
        B[i * nj + j] = s;
    }
    WC(1, i * nj + j);
}

static void exec_work_item(const oracle_launch *L, const int64_t gid[3])
{
    switch (L->kernel) {
    case OK_ATAX_TMP:   wi_atax_tmp(L, gid[0]); break;
    case OK_ATAX_Y:     wi_atax_y(L, gid[0]); break;
    case OK_BICG_S:     wi_bicg_s(L, gid[0]); break;
    case OK_BICG_Q:     wi_bicg_q(L, gid[0]); break;
    case OK_GESUMMV:    wi_gesummv(L, gid[0]); break;
    case OK_SYRK:       wi_syrk(L, gid[0], gid[1]); break;
    case OK_SYR2K:      wi_syr2k(L, gid[0], gid[1]); break;
    case OK_CORR_MEAN:  wi_corr_mean(L, gid[0]); break;
    case OK_CORR_STD:   wi_corr_std(L, gid[0]); break;
    case OK_CORR_REDUCE:wi_corr_reduce(L, gid[0], gid[1]); break;
    case OK_CORR_CORR:  wi_corr_corr(L, gid[0]); break;
    case OK_CONV2D:     wi_conv2d(L, gid[0], gid[1]); break;
    default: break;
    }
}

/* Execute one work-group (Fig 7: a CPU work-group whose fgid is in range
   executes its kernel code; its work-items run as a loop, L20.s35).
   n_items < 0 runs every work-item; otherwise only the first n_items in
   local-id order complete and the rest abort before their store (the abort
   model; legal per L20.s47 under write-once). */
void oracle_exec_wg_partial(const oracle_launch *L, int64_t fgid, int64_t n_items)
{
    int64_t ng[3] = {1, 1, 1}, g[3], lws[3] = {1, 1, 1};
    for (int d = 0; d < L->work_dim; ++d) {
        ng[d] = oracle_num_groups_dim(L->gws[d], L->lws[d]);
        lws[d] = L->lws[d];
    }
    oracle_unflatten(L->work_dim, ng, fgid, g);
    int64_t done = 0;
    for (int64_t l2 = 0; l2 < lws[2]; ++l2)
        for (int64_t l1 = 0; l1 < lws[1]; ++l1)
            for (int64_t l0 = 0; l0 < lws[0]; ++l0) {
                if (n_items >= 0 && done >= n_items) return;
                int64_t gid[3] = { g[0] * lws[0] + l0, g[1] * lws[1] + l1, g[2] * lws[2] + l2 };
                exec_work_item(L, gid);
                ++done;
            }
}

void oracle_exec_wg(const oracle_launch *L, int64_t fgid)
{
    oracle_exec_wg_partial(L, fgid, -1);
}

/* Run work-groups [lo, hi) in ascending or descending fgid order.  The
   single-device result R is oracle_run_range(L, 0, N_wg, 0); the CPU side of
   FluidiCL claims from the top down (L16.s8, L14.s36). */
void oracle_run_range(const oracle_launch *L, int64_t lo, int64_t hi, int32_t descending)
{
    if (!descending) { for (int64_t f = lo; f < hi; ++f) oracle_exec_wg(L, f); }
    else             { for (int64_t f = hi - 1; f >= lo; --f) oracle_exec_wg(L, f); }
}

/* ------------------------------------------------------------------------ */
/* C15/C16, Fig 9 (L18.s1-5; L16.s28-35): diff-merge.                         */
/*   if (index < number_bytes && cpu_buf[index] != orig[index])              */
/*       gpu_buf[index] = cpu_buf[index];                                     */
/* at the granularity of the buffer's base type (L16.s32-33), comparing bit   */
/* patterns (reading R4 / SURVEY S8).  Writes into gpu in place.             */
/* ------------------------------------------------------------------------ */
void oracle_merge(uint8_t *gpu, const uint8_t *cpu, const uint8_t *orig,
                  int64_t number_bytes, int32_t elem_size)
{
    for (int64_t index = 0; index + elem_size <= number_bytes; index += elem_size) {
        if (memcmp(cpu + index, orig + index, (size_t)elem_size) != 0)
            memcpy(gpu + index, cpu + index, (size_t)elem_size);
    }
}

/* ------------------------------------------------------------------------ */
/* C11 (L18.s23-32; L26.s27-28): adaptive chunk size, as a pure function.    */
/* Initial chunk = init_pct % of the work-groups; each subkernel is timed;   */
/* the chunk grows by step_pct % while the average time per work-group       */
/* decreases (reading R3 / SURVEY S5, S7: first growth unconditional, which   */
/* yields the 2%, 4%, 6% sequence of L26.s28; never shrink; hold otherwise).  */
/* A chunk smaller than min_units (the CPU compute units, L18.s31) is raised */
/* to min_units; the last chunk is clamped to what remains.                  */
/* times[k] is the measured time of chunk k (ignored for the last chunk).    */
/* Writes the chunk sizes (descending claims from N_wg down) to sizes[],     */
/* returns the number of chunks.                                             */
/* ------------------------------------------------------------------------ */
static int64_t pct_of(int64_t pct, int64_t n)
{
    return (pct * n + 99) / 100; /* ceil(pct/100 * n) */
}

int64_t oracle_chunk_schedule(int64_t n_wg, int64_t min_units, int64_t init_pct,
                              int64_t step_pct, const double *times, int64_t n_times,
                              int64_t *sizes, int64_t max_chunks)
{
    int64_t remaining = n_wg, k = 0, pct = init_pct;
    double prev_avg = -1.0;
    while (remaining > 0 && k < max_chunks) {
        int64_t size = pct_of(pct, n_wg);
        if (size < min_units) size = min_units;
        if (size < 1) size = 1;
        if (size > remaining) size = remaining;
        sizes[k] = size;
        remaining -= size;
        /* decide the next percentage from this chunk's time per work-group */
        double avg = (k < n_times) ? times[k] / (double)size : prev_avg;
        if (k == 0 || (prev_avg >= 0.0 && avg < prev_avg)) pct += step_pct;
        prev_avg = avg;
        ++k;
    }
    return k;
}
