"""GPU parity: the CUDA path (through the C-ABI) against the oracle, every kernel.

Each case checks, at sizes that span several tiles and a ragged tail:
  * GPU-only (plain grid) and CPU-only (host executor) against the oracle (bit-exact int32,
    1e-5 relative fp32);
  * the bit-identity of the two device bodies;
  * FluidiCL cooperative execution at forced split points and free-running: host copy
    and device copy both equal the single-device result bit for bit.
"""
import numpy as np
import pytest

import fcl_harness as H
import workloads as W
from _util import assert_bits, assert_parity, oracle_outputs

pytestmark = pytest.mark.gpu

CASES = [
    # kernel, n0, n1, integer, lws1d, lws2d
    ("atax_tmp", 300, 200, False, 32, None),
    ("atax_tmp", 300, 200, True, 32, None),
    ("atax_y", 300, 200, False, 32, None),
    ("atax_y", 300, 200, True, 32, None),
    ("bicg_s", 257, 384, False, 64, None),
    ("bicg_s", 257, 384, True, 64, None),
    ("bicg_q", 384, 257, False, 64, None),
    ("bicg_q", 384, 257, True, 64, None),
    ("gesummv", 300, 300, False, 32, None),
    ("gesummv", 300, 300, True, 32, None),
    ("gesummv", 512, 512, False, 256, None),
    ("syrk", 200, 70, False, None, (32, 8)),
    ("syrk", 256, 128, False, None, (32, 8)),
    ("syrk", 200, 70, True, None, (32, 8)),
    ("syr2k", 200, 70, False, None, (32, 8)),
    ("syr2k", 256, 64, True, None, (32, 8)),
    ("conv2d", 150, 300, False, None, (32, 8)),
    ("conv2d", 150, 300, True, None, (32, 8)),
    ("corr_mean", 200, 300, False, 64, None),
    ("corr_std", 200, 300, False, 64, None),
    ("corr_reduce", 200, 300, False, None, (32, 8)),
    ("corr_corr", 200, 300, False, 64, None),
]


def _ids(c):
    return f"{c[0]}-{'i32' if c[3] else 'f32'}-{c[1]}x{c[2]}"


def _problem(c, seed=0):
    kernel, n0, n1, integer, l1, l2 = c
    return W.make(kernel, n0, n1, integer=integer, seed=seed, lws1d=l1 or 256, lws2d=l2 or (32, 8))


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_cgo_panditg14_b200 import _build, fcl
    _build.build()
    c = fcl.Context(0)
    yield c
    c.release()


@pytest.mark.parametrize("case", CASES, ids=_ids)
def test_single_device_modes_vs_oracle(ctx, oracle_mod, case):
    P = _problem(case)
    R = oracle_outputs(oracle_mod, P)
    g_out, g_info = H.run(ctx, P, mode="gpu")
    c_out, c_info = H.run(ctx, P, mode="cpu")
    assert g_info["gpu_launches"] >= 1 and c_info["cpu_did_all"] == 1
    for k in P.out_indices:
        assert_parity(g_out[k], R[k], P.integer, f"{_ids(case)} gpu-only buf{k}")
        assert_parity(c_out[k], R[k], P.integer, f"{_ids(case)} cpu-only buf{k}")
        assert_bits(g_out[k], c_out[k], f"{_ids(case)} gpu vs cpu body buf{k}")


@pytest.mark.parametrize("case", CASES, ids=_ids)
def test_forced_splits_bit_identical(ctx, oracle_mod, case):
    """Every (or a spread of) split point(s): merge(G, C, T) equals the single-device result."""
    P = _problem(case, seed=1)
    ref, _ = H.run(ctx, P, mode="gpu")
    R = oracle_outputs(oracle_mod, P)
    n = P.num_groups
    splits = range(n + 1) if n <= 20 else sorted({0, 1, n // 3, n // 2, n - 1, n})
    for s in splits:
        bufs = H.create_buffers(ctx, P)
        out, info = H.run(ctx, P, mode="coop", bufs=bufs, forced_split=s)
        for k in P.out_indices:
            assert_bits(out[k], ref[k], f"{_ids(case)} split {s} host copy buf{k}")
            dev = H.device_array(bufs[k], np.int32 if P.integer else np.float32)
            assert_bits(dev, ref[k], f"{_ids(case)} split {s} device copy buf{k}")
        if s == n:
            assert info["merged"] == 0
        for b in bufs:
            b.release()
    for k in P.out_indices:
        assert_parity(ref[k], R[k], P.integer, _ids(case))


@pytest.mark.parametrize("case", CASES, ids=_ids)
@pytest.mark.parametrize("status,twin", [("device", "alias"), ("device", "twin"), ("host_mapped", "alias")])
def test_free_running_coop(oracle_mod, case, status, twin, monkeypatch):
    """Free-running race; with the twin aliased to the device copy (exact spans, default) and
    with a captured twin (Fig 9 as printed, FCL_FORCE_TWIN=1)."""
    from paper_conf_cgo_panditg14_b200 import fcl
    monkeypatch.setenv("FCL_FORCE_TWIN", "1" if twin == "twin" else "0")
    ctx = fcl.Context(0, status_location=status)
    try:
        P = _problem(case, seed=2)
        R = oracle_outputs(oracle_mod, P)
        ref, _ = H.run(ctx, P, mode="gpu")
        for trial in range(3):
            bufs = H.create_buffers(ctx, P)
            out, info = H.run(ctx, P, mode="coop", bufs=bufs, host_delay_us=[0, 50, 500][trial])
            for k in P.out_indices:
                assert_bits(out[k], ref[k], f"{_ids(case)} coop host buf{k} trial {trial}")
                dev = H.device_array(bufs[k], np.int32 if P.integer else np.float32)
                assert_bits(dev, ref[k], f"{_ids(case)} coop device buf{k} trial {trial}")
                assert_parity(out[k], R[k], P.integer, _ids(case))
            for b in bufs:
                b.release()
    finally:
        ctx.release()


RACE_CASES = [("conv2d", 600, 1000, False, None, (32, 8)), ("conv2d", 333, 515, True, None, (32, 8)),
              ("syrk", 512, 96, False, None, (32, 8)), ("corr_reduce", 700, 600, False, None, (32, 8)),
              ("gesummv", 2048, 2048, False, 64, None), ("atax_y", 1500, 3000, True, 32, None)]


@pytest.mark.parametrize("case", RACE_CASES, ids=_ids)
def test_return_race(oracle_mod, case, monkeypatch):
    """Return race: the output comes back in small ascending pieces while the
    host keeps computing chunks from the top; INOUT outputs (SYRK, CORR reduce), two outputs
    (GESUMMV) and 2-D spans.  Host and device copies equal the single-device result."""
    from paper_conf_cgo_panditg14_b200 import fcl
    for k, v in dict(FCL_RACE_MIN_BYTES="1", FCL_RACE_PIECE_BYTES="4096", FCL_RACE_CHUNK_MS="0.02",
                     FCL_EAGER_RETURN_BYTES="0").items():
        monkeypatch.setenv(k, v)
    ctx = fcl.Context(0)
    try:
        P = _problem(case, seed=12)
        R = oracle_outputs(oracle_mod, P)
        ref, _ = H.run(ctx, P, mode="gpu")
        for trial, kw in enumerate([{}, dict(host_delay_us=30), dict(init_chunk_pct=1, step_pct=0)]):
            bufs = H.create_buffers(ctx, P)
            out, info = H.run(ctx, P, mode="coop", bufs=bufs, **kw)
            for k in P.out_indices:
                assert_bits(out[k], ref[k], f"{_ids(case)} race host buf{k} {kw}")
                dev = H.device_array(bufs[k], np.int32 if P.integer else np.float32)
                assert_bits(dev, ref[k], f"{_ids(case)} race device buf{k} {kw}")
                assert_parity(out[k], R[k], P.integer, _ids(case))
            for b in bufs:
                b.release()
    finally:
        ctx.release()


@pytest.mark.parametrize("case", [CASES[0], CASES[9], CASES[12], CASES[16]], ids=_ids)
def test_fault_injection(ctx, oracle_mod, case):
    """Dropped publications, slow host, tiny and huge chunks: the result never changes."""
    P = _problem(case, seed=3)
    ref, _ = H.run(ctx, P, mode="gpu")
    for kw in [dict(drop_publish=1), dict(host_delay_us=2000), dict(init_chunk_pct=50, step_pct=0),
               dict(init_chunk_pct=1, step_pct=1), dict(cpu_wg_split=0), dict(n_host_threads=1),
               dict(abort_period=1), dict(abort_period=-1)]:
        out, info = H.run(ctx, P, mode="coop", **kw)
        for k in P.out_indices:
            assert_bits(out[k], ref[k], f"{_ids(case)} {kw}")


def test_cpu_first_returns_host_authoritative(ctx):
    """L16.s21: when the host covers everything first the host copy is final, no D2H."""
    P = W.make("gesummv", 512, integer=True, seed=4, lws1d=256)
    ref, _ = H.run(ctx, P, mode="gpu")
    bufs = H.create_buffers(ctx, P)
    out, info = H.run(ctx, P, mode="coop", bufs=bufs, forced_split=0)
    assert info["cpu_did_all"] == 1 and info["d2h_bytes"] == 0
    for k in P.out_indices:
        assert_bits(out[k], ref[k], "host")
        assert_bits(H.device_array(bufs[k], np.int32), ref[k], "device (merged)")


def test_abandoned_chunk_hazards(ctx):
    """Deferred quiescence: the GPU wins a lite, eagerly returned GESUMMV, whose
    host chunk is abandoned but not waited for.  Overwriting its input right away -- by a launch
    that writes it (WAR) or by fcl_write_buffer -- must not let the abandoned workers write
    anything derived from the new input into the first launch's outputs."""
    n = 2048
    P = W.make("gesummv", n, n, seed=31, lws1d=64, out_init="zero")
    ref, _ = H.run(ctx, P, mode="gpu")
    Q = W.make("atax_tmp", n, n, seed=32, lws1d=64, out_init="zero")   # writes a length-n vector
    for trial in range(6):
        bufs = H.create_buffers(ctx, P)          # A, B, x, tmp, y
        A2, x2 = ctx.buffer_from_array(Q.bufs[0]), ctx.buffer_from_array(Q.bufs[1])
        ctx.enqueue_ndrange("gesummv_f32", P.gws, P.lws, H.make_args(ctx, P, bufs))
        if trial % 2 == 0:   # WAR: x of the first launch is the output of the second
            ctx.enqueue_ndrange("atax_tmp_f32", Q.gws, Q.lws, [A2, x2, bufs[2], n, n])
        else:
            bufs[2].write_array(np.full(n, 7.0, np.float32))
        ctx.finish()
        for k in (3, 4):
            assert_bits(bufs[k].read_array(np.float32), ref[k], f"gesummv buf{k} trial {trial}")
        for b in bufs + [A2, x2]:
            b.release()


def test_slices_cover_only_their_range(ctx):
    """opts.wg_lo/wg_hi: a rank's slice writes exactly its work-groups (multi-GPU building block)."""
    P = W.make("conv2d", 130, 260, integer=True, seed=5)
    ref, _ = H.run(ctx, P, mode="gpu")
    k = ctx.kernel(H.kernel_name(P))
    nwg = P.num_groups
    for nranks in (2, 3):
        acc = P.bufs[1].copy()
        for r in range(nranks):
            lo, hi = ctx.slice_range(k, P.gws, P.lws, r, nranks)
            bufs = H.create_buffers(ctx, P)
            out, info = H.run(ctx, P, mode="coop", bufs=bufs, wg_lo=lo, wg_hi=hi)
            assert info["n_wg"] == hi - lo
            # rows owned by the slice
            ngx = P.gws[0] // P.lws[0]
            r0, r1 = (lo // ngx) * P.lws[1], min((hi // ngx) * P.lws[1], P.n0) if hi < nwg else P.n0
            o2, a2 = out[1].reshape(P.n0, P.n1), acc.reshape(P.n0, P.n1)
            a2[r0:r1] = o2[r0:r1]
            # untouched outside the slice
            np.testing.assert_array_equal(np.delete(o2, np.s_[r0:r1], axis=0),
                                          np.delete(P.bufs[1].reshape(P.n0, P.n1), np.s_[r0:r1], axis=0))
            for b in bufs:
                b.release()
        assert_bits(acc, ref[1], f"{nranks} slices concatenated")


def test_multi_kernel_chain_location_tracking(ctx, oracle_mod):
    """ATAX tmp -> y with the two kernels on different devices (C22 minimal form)."""
    n = 384
    P1 = W.make("atax_tmp", n, n, seed=6, lws1d=64)
    P2 = W.make("atax_y", n, n, seed=7, lws1d=64)
    P2.bufs[0] = P1.bufs[0]
    A, x, tmp = (ctx.buffer_from_array(b) for b in P1.bufs)
    y = ctx.buffer_from_array(P2.bufs[2])
    R1 = oracle_outputs(oracle_mod, P1)[2]
    for m1, m2 in [("cpu", "gpu"), ("gpu", "cpu"), ("coop", "coop"), ("cpu", "coop")]:
        ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode=m1)
        ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode=m2)
        ctx.finish()
        got = y.read_array(np.float32)
        L2 = oracle_mod.Launch("atax_y", False, n, n, list(P2.gws), list(P2.lws),
                               [P1.bufs[0].astype(np.float64), R1.copy(), np.zeros(n)])
        oracle_mod.run_range(L2, 0, L2.num_groups())
        assert_parity(got, L2.bufs[2], False, f"atax chain {m1}->{m2}")
    for b in (A, x, tmp, y):
        b.release()


def test_cpu_only_then_coop_refreshes_device_copy(ctx, oracle_mod):
    """A CPU-only launch leaves the device copy of its output stale; a following cooperative
    launch reading that buffer must see the host's values (lazy H2D), not the old device ones."""
    n = 384
    P1 = W.make("atax_tmp", n, n, seed=16, lws1d=64)
    P2 = W.make("atax_y", n, n, seed=17, lws1d=64)
    A, x, tmp = (ctx.buffer_from_array(b) for b in P1.bufs)
    y = ctx.buffer_from_array(P2.bufs[2])
    # device copy of tmp <- A x (GPU); then x changes and tmp is recomputed on the host only
    ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="gpu")
    ctx.finish()
    x2 = (P1.bufs[1] * 2.0 + 1.0).astype(np.float32)
    x.write_array(x2)
    ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="cpu")
    ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode="coop", forced_split=0)
    ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode="coop")
    ctx.finish()
    L1 = oracle_mod.Launch("atax_tmp", False, n, n, list(P1.gws), list(P1.lws),
                           [P1.bufs[0].astype(np.float64), x2.astype(np.float64), np.zeros(n)])
    oracle_mod.run_range(L1, 0, L1.num_groups())
    L2 = oracle_mod.Launch("atax_y", False, n, n, list(P2.gws), list(P2.lws),
                           [P1.bufs[0].astype(np.float64), L1.bufs[2].copy(), np.zeros(n)])
    oracle_mod.run_range(L2, 0, L2.num_groups())
    assert_parity(y.read_array(np.float32), L2.bufs[2], False, "cpu -> coop chain with a stale device copy")
    assert_parity(H.device_array(y, np.float32), L2.bufs[2], False, "device copy of y")
    for b in (A, x, tmp, y):
        b.release()


def test_corr_chain_coop_vs_oracle(ctx, oracle_mod):
    n, m = 300, 200
    data = W.corr_chain_inputs(n, m, seed=8)
    gws1, lws1 = W.geometry("corr_mean", n, m, lws1d=64)
    gws2, lws2 = W.geometry("corr_reduce", n, m)
    d = ctx.buffer_from_array(data)
    mean = ctx.buffer_from_array(np.zeros(m, np.float32))
    std = ctx.buffer_from_array(np.zeros(m, np.float32))
    sym = ctx.buffer_from_array(np.full(m * m, -3.0, np.float32))
    ctx.enqueue_ndrange("corr_mean_f32", gws1, lws1, [d, mean, n, m])
    ctx.enqueue_ndrange("corr_std_f32", gws1, lws1, [d, mean, std, n, m, 0.1])
    ctx.enqueue_ndrange("corr_reduce_f32", gws2, lws2, [d, mean, std, n, m])
    ctx.enqueue_ndrange("corr_corr_f32", gws1, lws1, [d, sym, n, m])
    ctx.finish()
    got = sym.read_array(np.float32)
    # the oracle's chain on the same inputs
    d64, mean64, std64, sym64 = data.astype(np.float64), np.zeros(m), np.zeros(m), np.full(m * m, -3.0)
    for kname, bl, g in [("corr_mean", [d64, mean64], (gws1, lws1)), ("corr_std", [d64, mean64, std64], (gws1, lws1)),
                         ("corr_reduce", [d64, mean64, std64], (gws2, lws2)), ("corr_corr", [d64, sym64], (gws1, lws1))]:
        L = oracle_mod.Launch(kname, False, n, m, list(g[0]), list(g[1]), bl)
        oracle_mod.run_range(L, 0, L.num_groups())
    assert_parity(got, sym64, False, "corr chain")
    assert_parity(mean.read_array(np.float32), mean64, False, "corr mean")
    assert_parity(d.read_array(np.float32), d64, False, "corr reduced data")
    for b in (d, mean, std, sym):
        b.release()


def test_async_independent_launches(ctx):
    """Non-blocking enqueue: independent launches queue their GPU work back to back while the
    coordinator runs their host sides in order; results match the single-device ones."""
    cases = [CASES[8], CASES[9], CASES[4], CASES[6], CASES[11], CASES[16], CASES[19], CASES[1]]
    probs = [_problem(c, seed=9 + k) for k, c in enumerate(cases)]
    refs = [H.run(ctx, P, mode="gpu")[0] for P in probs]
    bufs = [H.create_buffers(ctx, P) for P in probs]
    for rep in range(3):
        for P, b in zip(probs, bufs):
            ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="coop",
                                host_delay_us=[0, 30, 300][rep])
        ctx.finish()
        for P, b, ref in zip(probs, bufs, refs):
            if P.inout_indices:      # INOUT kernels accumulate across repetitions: reset input
                continue
            dt = np.int32 if P.integer else np.float32
            for k in P.out_indices:
                assert_bits(b[k].read_array(dt), ref[k], f"{P.kernel} rep {rep} host")
                assert_bits(H.device_array(b[k], dt), ref[k], f"{P.kernel} rep {rep} device")
    for bl in bufs:
        for b in bl:
            b.release()


def test_blocking_launch_reports_complete_info(ctx):
    P = W.make("gesummv", 1024, seed=5, lws1d=256)
    bufs = H.create_buffers(ctx, P)
    info = ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bufs), mode="coop", blocking=1)
    assert info["n_wg"] == 4 and info["gpu_launches"] >= 1
    ctx.finish()
    for b in bufs:
        b.release()


def _atax_chain(ctx, n, seed):
    P1 = W.make("atax_tmp", n, n, seed=seed, lws1d=64)
    P2 = W.make("atax_y", n, n, seed=seed + 1, lws1d=64)
    A, x, tmp = (ctx.buffer_from_array(b) for b in P1.bufs)
    y = ctx.buffer_from_array(P2.bufs[2])
    x2 = ctx.buffer_from_array((P1.bufs[1] * -0.5 + 0.25).astype(np.float32))
    Pg = W.make("gesummv", 256, seed=seed + 2, lws1d=64)
    g = [ctx.buffer_from_array(b) for b in Pg.bufs]
    return (P1, P2, Pg), (A, x, tmp, y, x2), g


def _run_sequence(ctx, P, B, g, modes, sync_each):
    (P1, P2, Pg), (A, x, tmp, y, x2) = P, B
    n = P1.n0
    seq = [
        ("atax_tmp_f32", P1, [A, x, tmp, n, n]),      # tmp = A x
        ("gesummv_f32", Pg, H.make_args(ctx, Pg, g)),  # independent
        ("atax_y_f32", P2, [A, tmp, y, n, n]),        # RAW on tmp
        ("atax_tmp_f32", P1, [A, x2, tmp, n, n]),     # WAR on tmp (read just above), WAW on tmp
        ("gesummv_f32", Pg, H.make_args(ctx, Pg, g)),  # WAW on its own outputs
        ("atax_y_f32", P2, [A, tmp, y, n, n]),        # RAW on the new tmp, WAW on y
    ]
    for k, (name, Pk, args) in enumerate(seq):
        ctx.enqueue_ndrange(name, Pk.gws, Pk.lws, args, mode=modes[k % len(modes)])
        if sync_each:
            ctx.finish()
    ctx.finish()
    return [b.read_array(np.float32) for b in (tmp, y, g[3], g[4])], \
           [H.device_array(b, np.float32) for b in (tmp, y, g[3], g[4])]


@pytest.mark.parametrize("modes", [("gpu",), ("coop",), ("gpu", "coop"), ("coop", "gpu", "gpu")], ids=lambda m: "-".join(m))
def test_dependent_launch_chains_without_sync(ctx, modes):
    """Back-to-back launches with RAW / WAR / WAW dependencies and independent ones, no finish
    in between (programmatic dependent launch decides per grid whether to wait in-kernel, and
    small outputs return lazily): host and device copies equal the fully synchronised run."""
    P, B, g = _atax_chain(ctx, 320, seed=30)
    want_h, want_d = _run_sequence(ctx, P, B, g, ("gpu",), sync_each=True)
    for rep in range(3):
        got_h, got_d = _run_sequence(ctx, P, B, g, modes, sync_each=False)
        for k in range(4):
            assert_bits(got_h[k], want_h[k], f"host output {k}, rep {rep}")
            assert_bits(got_d[k], want_d[k], f"device output {k}, rep {rep}")
    for b in list(B) + g:
        b.release()


def test_many_independent_plain_grids_then_dependent(ctx):
    """More independent plain grids in a row than one PDL chain may hold (8), then a grid that
    reads all their outputs' producers' inputs: every result equals the single-launch one."""
    probs = [W.make("bicg_q", 384, 257, seed=40 + k, lws1d=64) for k in range(11)]
    refs = [H.run(ctx, P, mode="gpu")[0][2] for P in probs]
    bufs = [H.create_buffers(ctx, P) for P in probs]
    for P, b in zip(probs, bufs):
        ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="gpu")
    # WAW on the first launch's output, then RAW through the host (CPU-only reads nothing of it,
    # but must see coherent host copies of everything)
    P0 = probs[0]
    ctx.enqueue_ndrange(H.kernel_name(P0), P0.gws, P0.lws, H.make_args(ctx, P0, bufs[0]), mode="coop")
    for P, b, r in zip(probs, bufs, refs):
        assert_bits(b[2].read_array(np.float32), r, f"{P.kernel} read before finish")
    ctx.finish()
    for P, b, r in zip(probs, bufs, refs):
        assert_bits(H.device_array(b[2], np.float32), r, f"{P.kernel} device")
    for bl in bufs:
        for b in bl:
            b.release()


def test_lazy_return_consumers(ctx, oracle_mod):
    """A GPU-only launch's small output returns lazily: a read before fcl_finish, a CPU-only
    launch reading it on the host, and a cooperative launch whose host chunks read it must all
    see the GPU's values."""
    n = 320
    P1 = W.make("atax_tmp", n, n, seed=50, lws1d=64)
    P2 = W.make("atax_y", n, n, seed=51, lws1d=64)
    A, x, tmp = (ctx.buffer_from_array(b) for b in P1.bufs)
    y = ctx.buffer_from_array(P2.bufs[2])
    R1 = oracle_outputs(oracle_mod, P1)[2]
    L2 = oracle_mod.Launch("atax_y", False, n, n, list(P2.gws), list(P2.lws),
                           [P1.bufs[0].astype(np.float64), R1.copy(), np.zeros(n)])
    oracle_mod.run_range(L2, 0, L2.num_groups())
    # read before finish
    ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="gpu")
    assert_parity(tmp.read_array(np.float32), R1, False, "lazy tmp read before finish")
    # host-side consumers of a lazily returned output
    for m2, opts in [("cpu", {}), ("coop", {"forced_split": 0}), ("coop", {"host_delay_us": 0})]:
        tmp.write_array(np.full(n, 7.0, np.float32))
        ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="gpu")
        ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode=m2, **opts)
        ctx.finish()
        assert_parity(y.read_array(np.float32), L2.bufs[2], False, f"gpu -> {m2} {opts}")
    for b in (A, x, tmp, y):
        b.release()


VARIANT_CASES = [c for c in CASES if c[0] in ("atax_y", "bicg_s", "corr_mean", "corr_std", "syrk", "syr2k", "corr_corr")]


@pytest.mark.parametrize("case", VARIANT_CASES, ids=_ids)
def test_host_variants_bit_identical(ctx, case):
    """Every alternate host body (C26: "cpu" loop-interchanged, "wi" work-item order as written
    for the GPU) gives the GPU-only result bit for bit, alone and in a cooperative split."""
    P = _problem(case, seed=21)
    k = ctx.kernel(H.kernel_name(P))
    assert k.host_variants == ["cpu", "wi"]
    ref, _ = H.run(ctx, P, mode="gpu")
    for v in (0, 1):
        for mode, opts in [("cpu", {}), ("coop", {"forced_split": P.num_groups // 3})]:
            out, info = H.run(ctx, P, mode=mode, host_variant=v, **opts)
            assert info["host_variant"] == v and info["n_host_variants"] == 2
            for i in P.out_indices:
                assert_bits(out[i], ref[i], f"{P.kernel} variant {v} {mode}")


@pytest.mark.parametrize("kernel,n0,n1,lws,must_win", [("bicg_s", 2048, 2048, 64, None),
                                                       ("corr_corr", 1024, 1024, 64, 0)])
def test_online_profiling_picks_the_faster_body(kernel, n0, n1, lws, must_win):
    """CPU-only launches with profiling on (the default): the first launch of a shape times each
    host body on one small allocation and keeps the fastest per work-group; later launches of
    the shape reuse the choice without profiling (L22.s4-11).  CORR's symmat is the paper's
    case (L26.s5-7): the work-item order walks two columns per output and loses clearly."""
    from paper_conf_cgo_panditg14_b200 import fcl
    c = fcl.Context(0)
    try:
        P = W.make(kernel, n0, n1, seed=22, lws1d=lws)
        o = P.out_indices[0]
        ref, _ = H.run(c, P, mode="gpu")
        out, info = H.run(c, P, mode="cpu")
        assert info["n_host_variants"] == 2
        t = info["profile_ms_per_wg"]
        assert t[0] > 0 and t[1] > 0, info
        assert info["host_variant"] == (0 if t[0] <= t[1] else 1)
        if must_win is not None:
            assert info["host_variant"] == must_win, f"per-work-group times {t}"
        assert_bits(out[o], ref[o], "profiled CPU-only")
        out, info2 = H.run(c, P, mode="cpu")
        assert info2["host_variant"] == info["host_variant"] and info2["profile_ms_per_wg"] == [0.0, 0.0]
        assert_bits(out[o], ref[o], "cached choice")
        # a forced variant bypasses the profiler
        _, info3 = H.run(c, P, mode="cpu", host_variant=1)
        assert info3["host_variant"] == 1 and info3["profile_ms_per_wg"] == [0.0, 0.0]
    finally:
        c.release()


def test_executor_back_to_back_jobs_in_place(ctx):
    """Regression: a worker that woke for an empty job could claim an 'item' of it while the next
    job's fields were being written and run that job's work-group a second time -- an in-place
    (INOUT) kernel then applied twice.  CPU-only launches of new shapes (each profiles its host
    bodies behind an empty wake-up job, then runs more jobs back to back) must equal GPU-only."""
    for k, n in enumerate(range(160, 320, 8)):
        P = W.make("syrk", n, 70, seed=40 + k)
        ref, _ = H.run(ctx, P, mode="gpu")
        out, info = H.run(ctx, P, mode="cpu")
        assert info["cpu_did_all"] == 1
        for i in P.out_indices:
            assert_bits(out[i], ref[i], f"syrk {n}x70 cpu-only")


@pytest.mark.parametrize("kernel", ["syrk", "syr2k"])
def test_syrk_slices_same_buffer(ctx, kernel):
    """SYRK / SYR2K (C in place) run as consecutive slices on the SAME buffers, each slice
    cooperative: every element of C is updated exactly once (a slice must not touch C's device
    copy outside its rows -- the upper-triangle grid's mirror blocks would), and the result is the
    GPU-only one (a slice runs every tile of its rows: SYR2K tiles below the diagonal take the
    mirror's per-k order, diagonal tiles store their upper half and its mirror)."""
    P = W.make(kernel, 384, 96, seed=61)
    ref, _ = H.run(ctx, P, mode="gpu")
    k = ctx.kernel(H.kernel_name(P))
    for nranks in (2, 3):
        bufs = H.create_buffers(ctx, P)
        for r in range(nranks):
            lo, hi = ctx.slice_range(k, P.gws, P.lws, r, nranks)
            ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bufs), mode="coop",
                                wg_lo=lo, wg_hi=hi)
            ctx.finish()
        o = P.out_indices[0]
        out = bufs[o].read_array(np.float32)
        assert_bits(out, ref[o], f"{kernel} {nranks} slices on one buffer")
        dev = H.device_array(bufs[o], np.float32)
        assert_bits(dev, ref[o], f"{kernel} {nranks} slices, device copy")
        for b in bufs:
            b.release()


@pytest.mark.parametrize("integer", [False, True])
@pytest.mark.parametrize("kernel,n,m", [("syrk", 300, 77), ("syr2k", 300, 77), ("syr2k", 256, 64)])
def test_symmetric_accumulators(ctx, kernel, n, m, integer):
    """SYRK and SYR2K's canonical per-k order is symmetric: with a symmetric C
    the result is symmetric bit for bit -- on the GPU (upper-triangle grid with mirrors, and the
    full grid of a forced split), and on the host."""
    P = W.make(kernel, n, m, integer=integer, seed=62)
    o = P.out_indices[0]
    C = P.bufs[o].reshape(n, n)
    P.bufs[o] = np.ascontiguousarray(np.triu(C) + np.triu(C, 1).T).reshape(-1)
    dt = np.int32 if integer else np.float32
    for mode, opts in [("gpu", {}), ("cpu", {}), ("coop", {"forced_split": P.num_groups // 3})]:
        out, _ = H.run(ctx, P, mode=mode, **opts)
        r = out[o].reshape(n, n).view(np.uint32)
        assert np.array_equal(r, r.T), f"{kernel} {mode} {opts}: not symmetric at {np.argwhere(r != r.T)[:3]}"


def test_context_allocator_vtable(oracle_mod):
    """fcl_context_desc's allocator: buffers and the twin/stage pool come from the
    torch caching allocator; cooperative launches (free-running with a captured twin, forced
    splits) give the GPU-only bits and every allocation is returned."""
    import os
    from paper_conf_cgo_panditg14_b200 import fcl
    alloc, free = fcl.torch_allocator(0)
    live, made = {}, [0]

    def a(n):
        p = alloc(n)
        live[p] = n
        made[0] += 1
        return p

    def f(p):
        live.pop(p)
        free(p)

    os.environ["FCL_FORCE_TWIN"] = "1"
    try:
        ctx = fcl.Context(0, allocator=(a, f))
    finally:
        del os.environ["FCL_FORCE_TWIN"]
    try:
        P = W.make("conv2d", 150, 300, seed=63)
        ref, _ = H.run(ctx, P, mode="gpu")
        assert made[0] >= 2, "no buffer came from the allocator"
        for opts in (dict(), dict(forced_split=P.num_groups // 2), dict(gpu_delay_us=100)):
            out, info = H.run(ctx, P, mode="coop", **opts)
            assert_bits(out[1], ref[1], f"allocator vtable {opts}")
        assert len(live) >= 2   # the pool's twin and stage are still held
    finally:
        ctx.release()
    assert not live, f"{len(live)} allocations not returned"
