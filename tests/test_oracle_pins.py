"""Pins for the oracle (oracle/): paper values, closed forms, library routines.

Every oracle function is checked here against something other than itself
(DESIGN.md §3).  CPU only; no GPU needed.
"""
import os

import numpy as np
import pytest

import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden_rows(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


def _drop012(n: int) -> str:
    return "".join(ch for ch in str(n) if ch not in "012")


def to_oracle(o, P: W.Problem):
    """fp32 -> fp64 copies (float kernels) or uint32 views (integer kernels)."""
    if P.integer:
        bufs = [b.view(np.uint32).copy() for b in P.bufs]
    else:
        bufs = [b.astype(np.float64) for b in P.bufs]
    return o.Launch(P.kernel, P.integer, P.n0, P.n1, list(P.gws), list(P.lws), bufs,
                    alpha=P.alpha, beta=P.beta, eps=P.eps, ialpha=P.ialpha, ibeta=P.ibeta)


# ---------------------------------------------------------------- flattening
def test_fig5_flattening_pattern(oracle_mod):
    """Fig 5 (L14.s26-31): column-fastest numbering reproduces the printed '3 4'."""
    ng = (5, 5)  # dim0 = columns, dim1 = rows
    for row, *printed in _golden_rows("fig5_flattening.txt"):
        ids = [oracle_mod.flatten(ng, (col, int(row))) for col in range(5)]
        got = " ".join(s for s in (_drop012(i) for i in ids) if s)
        assert got == " ".join(printed), (row, ids)
    # the transposed (row-fastest) numbering would print differently
    ids_rowfast = [col * 5 + 0 for col in range(5)]
    assert " ".join(s for s in map(_drop012, ids_rowfast) if s) != "3 4"


def test_flatten_bijection(oracle_mod):
    for ng in [(7,), (3, 5), (4, 3, 2)]:
        n = int(np.prod(ng))
        seen = set()
        for f in range(n):
            g = oracle_mod.unflatten(ng, f)
            assert all(0 <= gi < ni for gi, ni in zip(g, ng))
            assert oracle_mod.flatten(ng, g) == f
            seen.add(g)
        assert len(seen) == n


def test_table2_work_group_counts(oracle_mod):
    """Table 2 (L22.s36): the printed work-group counts, after digit loss."""
    for kernel, n0, n1, l1d, expect, printed in _golden_rows("table2_wg_counts.txt"):
        n0, n1, l1d, expect = int(n0), int(n1), int(l1d), int(expect)
        gws, lws = W.geometry(kernel, n0, n1, lws1d=l1d)
        L = oracle_mod.Launch(kernel, False, n0, n1, list(gws), list(lws),
                              [np.zeros(1)] * oracle_mod.KERNELS[kernel][1])
        assert L.num_groups() == expect, kernel
        assert _drop012(expect) == printed


# ---------------------------------------------------------------- merge (Fig 9)
@pytest.mark.parametrize("dtype", [np.uint8, np.uint16, np.uint32, np.uint64])
@pytest.mark.parametrize("frac", [0.0, 0.01, 0.5, 1.0])
def test_merge_vs_numpy_where(oracle_mod, dtype, frac):
    rng = np.random.default_rng(1)
    n = 4099
    info = np.iinfo(dtype)
    twin = rng.integers(0, info.max, n, dtype=dtype, endpoint=True)
    gpu = rng.integers(0, info.max, n, dtype=dtype, endpoint=True)
    cpu = twin.copy()
    idx = rng.random(n) < frac
    cpu[idx] ^= dtype(1)
    out = oracle_mod.merge(gpu, cpu, twin, np.dtype(dtype).itemsize)
    np.testing.assert_array_equal(out, np.where(cpu != twin, cpu, gpu))
    if frac == 0.0:
        np.testing.assert_array_equal(out, gpu)
    if frac == 1.0:
        np.testing.assert_array_equal(out, cpu)
    # idempotence
    np.testing.assert_array_equal(oracle_mod.merge(out, cpu, twin, np.dtype(dtype).itemsize), out)


def test_merge_granularity_is_element_size(oracle_mod):
    """L16.s32-33: a 4-byte element is compared and copied as a whole."""
    twin = np.array([0x11223344, 0x55667788], np.uint32)
    cpu = np.array([0x11223345, 0x55667788], np.uint32)   # one byte differs in word 0
    gpu = np.array([0xAAAAAAAA, 0xBBBBBBBB], np.uint32)
    out4 = oracle_mod.merge(gpu, cpu, twin, 4)
    np.testing.assert_array_equal(out4, [0x11223345, 0xBBBBBBBB])
    out1 = oracle_mod.merge(gpu.view(np.uint8), cpu.view(np.uint8), twin.view(np.uint8), 1)
    # byte granularity (Fig 9's illustration) takes only the changed byte
    assert out1.view(np.uint32)[0] == (0xAAAAAA00 | 0x45)
    assert out1.view(np.uint32)[1] == 0xBBBBBBBB


def test_merge_float_bitwise(oracle_mod):
    """Reading R4: comparison is on bit patterns (+0/-0 and NaN payloads differ)."""
    twin = np.array([0.0, np.nan, 1.0], np.float32)
    cpu = np.array([-0.0, np.float32(np.nan), 1.0], np.float32)
    cpu.view(np.uint32)[1] = twin.view(np.uint32)[1] ^ 1  # other NaN payload
    gpu = np.array([5.0, 6.0, 7.0], np.float32)
    out = oracle_mod.merge(gpu.view(np.uint32), cpu.view(np.uint32), twin.view(np.uint32), 4)
    np.testing.assert_array_equal(out, np.array([cpu.view(np.uint32)[0], cpu.view(np.uint32)[1],
                                                 gpu.view(np.uint32)[2]]))


# ---------------------------------------------------------------- chunk sizer (C11)
def test_chunk_sequence_paper(oracle_mod):
    """L26.s28: 2%, 4%, 6% ... while the time per work-group keeps decreasing."""
    for n, *expect in _golden_rows("chunk_sequence.txt"):
        n = int(n)
        expect = [int(e) for e in expect]
        k = len(expect)
        times = [1.0 / (i + 1) for i in range(k + 5)]   # per-WG time decreasing (t / size)
        sizes = oracle_mod.chunk_schedule(n, 1, 2, 2, times)
        assert sizes[:k] == expect
        assert sum(sizes) == n


def test_chunk_hold_when_not_improving(oracle_mod):
    # per-WG time: chunk0 328 WG in 3.28 (0.01/WG), chunk1 656 in 13.12 (0.02/WG, worse)
    sizes = oracle_mod.chunk_schedule(16384, 1, 2, 2, [3.28, 13.12, 13.12, 13.12])
    assert sizes[:4] == [328, 656, 656, 656]   # grew once unconditionally, then hold
    assert sum(sizes) == 16384


def test_chunk_min_compute_units(oracle_mod):
    """L18.s31: fewer WGs than compute units -> chunk = #compute units."""
    sizes = oracle_mod.chunk_schedule(16, 8, 2, 2, [1.0] * 10)
    assert sizes[0] == 8 and sum(sizes) == 16
    sizes = oracle_mod.chunk_schedule(16, 1, 2, 2, [1.0] * 20)
    assert sizes[0] == 1 and sum(sizes) == 16


# ---------------------------------------------------------------- kernels vs library routines
def _run(o, P):
    L = to_oracle(o, P)
    return o.run(L)


def _f(P, k):
    return P.bufs[k].astype(np.float64)


@pytest.mark.parametrize("n0,n1", [(256, 256), (70, 45)])
def test_atax_bicg_vs_numpy(oracle_mod, n0, n1):
    P = W.make("atax_tmp", n0, n1, seed=3)
    R = _run(oracle_mod, P)
    A = _f(P, 0).reshape(n0, n1)
    np.testing.assert_allclose(R.bufs[2], A @ _f(P, 1), rtol=1e-12)
    P2 = W.make("atax_y", n0, n1, seed=4)
    R2 = _run(oracle_mod, P2)
    A2 = _f(P2, 0).reshape(n0, n1)
    np.testing.assert_allclose(R2.bufs[2], A2.T @ _f(P2, 1), rtol=1e-12)
    P3 = W.make("bicg_s", n0, n1, seed=5)
    R3 = _run(oracle_mod, P3)
    np.testing.assert_allclose(R3.bufs[2], _f(P3, 0).reshape(n0, n1).T @ _f(P3, 1), rtol=1e-12)
    P4 = W.make("bicg_q", n0, n1, seed=6)
    R4 = _run(oracle_mod, P4)
    np.testing.assert_allclose(R4.bufs[2], _f(P4, 0).reshape(n0, n1) @ _f(P4, 1), rtol=1e-12)


def test_gesummv_vs_numpy(oracle_mod):
    n = 300
    P = W.make("gesummv", n, seed=7)
    R = _run(oracle_mod, P)
    A, B, x = _f(P, 0).reshape(n, n), _f(P, 1).reshape(n, n), _f(P, 2)
    np.testing.assert_allclose(R.bufs[3], A @ x, rtol=1e-12)
    np.testing.assert_allclose(R.bufs[4], P.alpha * (A @ x) + P.beta * (B @ x), rtol=1e-12)


@pytest.mark.parametrize("n,m", [(64, 64), (50, 37)])
def test_syrk_syr2k_vs_numpy(oracle_mod, n, m):
    P = W.make("syrk", n, m, seed=8)
    R = _run(oracle_mod, P)
    A, C = _f(P, 0).reshape(n, m), _f(P, 1).reshape(n, n)
    np.testing.assert_allclose(R.bufs[1].reshape(n, n), P.beta * C + P.alpha * A @ A.T, rtol=1e-12)
    P = W.make("syr2k", n, m, seed=9)
    R = _run(oracle_mod, P)
    A, B, C = _f(P, 0).reshape(n, m), _f(P, 1).reshape(n, m), _f(P, 2).reshape(n, n)
    ref = P.beta * C + P.alpha * A @ B.T + P.alpha * B @ A.T
    np.testing.assert_allclose(R.bufs[2].reshape(n, n), ref, rtol=1e-12)


def test_corr_chain_is_pearson(oracle_mod):
    """mean -> std -> reduce -> corr is the Pearson correlation matrix (np.corrcoef)."""
    n, m = 200, 48
    data32 = W.corr_chain_inputs(n, m, seed=10)
    geo = lambda k: W.geometry(k, n, m, lws1d=16)
    data = data32.astype(np.float64)
    mean, std, sym = np.zeros(m), np.zeros(m), np.full(m * m, -5.0)
    mk = lambda k, bufs: oracle_mod.Launch(k, False, n, m, list(geo(k)[0]), list(geo(k)[1]), bufs)
    oracle_mod.run_range(L := mk("corr_mean", [data, mean]), 0, L.num_groups())
    np.testing.assert_allclose(mean, data.reshape(n, m).mean(0), rtol=1e-12)
    oracle_mod.run_range(L := mk("corr_std", [data, mean, std]), 0, L.num_groups())
    np.testing.assert_allclose(std, data.reshape(n, m).std(0), rtol=1e-12)
    oracle_mod.run_range(L := mk("corr_reduce", [data, mean, std]), 0, L.num_groups())
    oracle_mod.run_range(L := mk("corr_corr", [data, sym]), 0, L.num_groups())
    ref = np.corrcoef(data32.astype(np.float64).reshape(n, m), rowvar=False)
    np.testing.assert_allclose(sym.reshape(m, m), ref, rtol=1e-10, atol=1e-12)


def test_corr_std_clamp(oracle_mod):
    """std <= eps is replaced by 1.0 (PolyBench correlation)."""
    n, m = 16, 4
    d = np.tile(np.array([1.0, 2.0, 3.0, 4.0]), n)
    d[1::4] += np.linspace(0, 1, n)      # column 1 varies (std ~0.3 > 0.1)
    mean = d.reshape(n, m).mean(0)
    std = np.zeros(m)
    gws, lws = W.geometry("corr_std", n, m, lws1d=4)
    L = oracle_mod.Launch("corr_std", False, n, m, list(gws), list(lws), [d, mean, std])
    oracle_mod.run_range(L, 0, L.num_groups())
    assert std[0] == 1.0 and std[2] == 1.0 and std[3] == 1.0
    assert abs(std[1] - d.reshape(n, m)[:, 1].std()) < 1e-12


def test_conv2d_vs_scipy(oracle_mod):
    from scipy.signal import correlate2d
    ni, nj = 40, 70
    P = W.make("conv2d", ni, nj, seed=11)
    R = _run(oracle_mod, P)
    A = _f(P, 0).reshape(ni, nj)
    c = np.array([[0.2, 0.5, -0.8], [-0.3, 0.6, -0.9], [0.4, 0.7, 0.10]])
    out = R.bufs[1].reshape(ni, nj)
    np.testing.assert_allclose(out[1:-1, 1:-1], correlate2d(A, c, mode="valid"), rtol=1e-12, atol=1e-14)
    # border untouched (poison preserved)
    B0 = _f(P, 1).reshape(ni, nj)
    for sl in [(0, slice(None)), (-1, slice(None)), (slice(None), 0), (slice(None), -1)]:
        np.testing.assert_array_equal(out[sl], B0[sl])


def test_conv2d_constant_closed_form(oracle_mod):
    """Coefficients sum to 0.5: a constant image gives 0.5*c inside."""
    ni = nj = 20
    P = W.make("conv2d", ni, nj, seed=0)
    P.bufs[0][:] = 3.0
    R = _run(oracle_mod, P)
    np.testing.assert_allclose(R.bufs[1].reshape(ni, nj)[1:-1, 1:-1], 1.5, rtol=1e-14)


def test_identity_closed_forms(oracle_mod):
    n = 64
    eye = np.eye(n, dtype=np.float32).ravel()
    P = W.make("atax_tmp", n, n, seed=1, lws1d=16); P.bufs[0][:] = eye
    tmp = _run(oracle_mod, P).bufs[2]
    np.testing.assert_array_equal(tmp, P.bufs[1].astype(np.float64))
    P = W.make("syrk", n, n, seed=1); P.bufs[0][:] = eye; P.bufs[1][:] = 0
    np.testing.assert_array_equal(_run(oracle_mod, P).bufs[1].reshape(n, n), P.alpha * np.eye(n))
    P = W.make("syr2k", n, n, seed=1); P.bufs[0][:] = eye; P.bufs[1][:] = eye; P.bufs[2][:] = 0
    np.testing.assert_array_equal(_run(oracle_mod, P).bufs[2].reshape(n, n), 2 * P.alpha * np.eye(n))
    P = W.make("gesummv", n, seed=1, lws1d=16); P.bufs[0][:] = eye; P.bufs[1][:] = eye
    np.testing.assert_allclose(_run(oracle_mod, P).bufs[4], (P.alpha + P.beta) * P.bufs[2].astype(np.float64), rtol=1e-15)


def _mod32(x):
    return (np.asarray(x, dtype=np.int64) % (1 << 32)).astype(np.uint32)


def test_integer_kernels_vs_int64_numpy(oracle_mod):
    """Integer instantiations (reading R6) = exact integer math mod 2^32."""
    n = 48
    P = W.make("gesummv", n, integer=True, seed=2, lws1d=16)
    R = _run(oracle_mod, P)
    A, B, x = (P.bufs[k].astype(np.int64) for k in range(3))
    A, B = A.reshape(n, n), B.reshape(n, n)
    np.testing.assert_array_equal(R.bufs[3], _mod32(A @ x))
    np.testing.assert_array_equal(R.bufs[4], _mod32(P.ialpha * (A @ x) + P.ibeta * (B @ x)))
    P = W.make("syr2k", n, 33, integer=True, seed=3)
    R = _run(oracle_mod, P)
    A, B, C = (P.bufs[k].astype(np.int64) for k in range(3))
    A, B, C = A.reshape(n, 33), B.reshape(n, 33), C.reshape(n, n)
    ref = P.ibeta * C + P.ialpha * (A @ B.T) + P.ialpha * (B @ A.T)
    np.testing.assert_array_equal(R.bufs[2].reshape(n, n), _mod32(ref))
    P = W.make("conv2d", 17, 29, integer=True, seed=4)
    R = _run(oracle_mod, P)
    from scipy.signal import correlate2d
    A = P.bufs[0].astype(np.int64).reshape(17, 29)
    ci = np.array([[2, 5, -8], [-3, 6, -9], [4, 7, 1]], np.int64)
    np.testing.assert_array_equal(R.bufs[1].reshape(17, 29)[1:-1, 1:-1], _mod32(correlate2d(A, ci, "valid")))
    for k in ("atax_tmp", "atax_y", "bicg_s", "bicg_q"):
        P = W.make(k, 40, 24, integer=True, seed=5, lws1d=8)
        R = _run(oracle_mod, P)
        A = P.bufs[0].astype(np.int64).reshape(40, 24)
        v = P.bufs[1].astype(np.int64)
        ref = A @ v if k in ("atax_tmp", "bicg_q") else A.T @ v
        np.testing.assert_array_equal(R.bufs[2], _mod32(ref))
    P = W.make("syrk", 30, 20, integer=True, seed=6)
    R = _run(oracle_mod, P)
    A, C = P.bufs[0].astype(np.int64).reshape(30, 20), P.bufs[1].astype(np.int64).reshape(30, 30)
    np.testing.assert_array_equal(R.bufs[1].reshape(30, 30), _mod32(P.ibeta * C + P.ialpha * A @ A.T))
