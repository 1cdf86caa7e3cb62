"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py / the config
benchmarks time (COOP mode, free-running): sampled work-groups against the oracle, plus the
bit-identity of the cooperative result with the GPU-only one over the whole output.
"""
import numpy as np
import pytest

import fcl_harness as H
import workloads as W
from _util import assert_bits, assert_parity, to_oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_cgo_panditg14_b200 import _build, fcl
    _build.build()
    c = fcl.Context(0)
    yield c
    c.release()


def _check_sampled(oracle_mod, P, out, wgs, partial=None):
    """Run the oracle on just work-groups `wgs` (or the first `partial` work-items of each) and
    compare the words those work-groups write."""
    L = to_oracle(oracle_mod, P).copy(with_wcount=True)
    for f in wgs:
        if partial is None:
            oracle_mod.exec_wg_partial(L, f, -1)
        else:
            oracle_mod.exec_wg_partial(L, f, partial)
    checked = 0
    for k in P.out_indices:
        mask = L.wcount[k] > 0
        checked += int(mask.sum())
        assert_parity(out[k], L.bufs[k], P.integer, f"{P.kernel} sampled WGs {wgs}", mask=mask)
    assert checked > 0
    return checked


@pytest.mark.parametrize("kernel", ["gesummv", "bicg_s", "bicg_q"])
def test_config2_n4096(ctx, oracle_mod, kernel):
    P = W.make(kernel, 4096, 4096, seed=21, lws1d=256)
    ref, _ = H.run(ctx, P, mode="gpu")
    out, info = H.run(ctx, P, mode="coop")
    for k in P.out_indices:
        assert_bits(out[k], ref[k], f"{kernel} coop vs gpu-only")
    _check_sampled(oracle_mod, P, out, [0, 7, 15])


@pytest.mark.parametrize("kernel", ["syrk", "syr2k"])
def test_config3_n2048(ctx, oracle_mod, kernel):
    P = W.make(kernel, 2048, 2048, seed=22)
    ref, _ = H.run(ctx, P, mode="gpu")
    out, info = H.run(ctx, P, mode="coop")
    assert_bits(out[P.out_indices[0]], ref[P.out_indices[0]], f"{kernel} coop vs gpu-only")
    n = P.num_groups
    _check_sampled(oracle_mod, P, out, [0, 63, n // 2 + 17, n - 1])


def test_config4_conv2d_16384(ctx, oracle_mod):
    P = W.make("conv2d", 16384, 16384, seed=23, out_init="zero")
    ref, _ = H.run(ctx, P, mode="gpu")
    out, info = H.run(ctx, P, mode="coop")
    assert_bits(out[1], ref[1], "conv2d coop vs gpu-only")
    n = P.num_groups
    ngx = P.gws[0] // P.lws[0]
    _check_sampled(oracle_mod, P, out, [0, ngx - 1, n // 2 + 3, n - ngx, n - 1])


def test_config4_corr_4096_chain(ctx, oracle_mod):
    n = m = 4096
    data = W.corr_chain_inputs(n, m, seed=24)
    gws1, lws1 = W.geometry("corr_mean", n, m, lws1d=256)
    gws2, lws2 = W.geometry("corr_reduce", n, m)
    d = ctx.buffer_from_array(data)
    mean = ctx.buffer_from_array(np.zeros(m, np.float32))
    std = ctx.buffer_from_array(np.zeros(m, np.float32))
    sym = ctx.buffer_from_array(np.zeros(m * m, np.float32))
    ctx.enqueue_ndrange("corr_mean_f32", gws1, lws1, [d, mean, n, m])
    ctx.enqueue_ndrange("corr_std_f32", gws1, lws1, [d, mean, std, n, m, 0.1])
    ctx.enqueue_ndrange("corr_reduce_f32", gws2, lws2, [d, mean, std, n, m])
    ctx.enqueue_ndrange("corr_corr_f32", gws1, lws1, [d, sym, n, m])
    ctx.finish()
    got_sym = sym.read_array(np.float32)
    # oracle: mean, std and the reduction in full (fp64), symmat on sampled work-items
    d64, mean64, std64 = data.astype(np.float64), np.zeros(m), np.zeros(m)
    for kname, bl, g in [("corr_mean", [d64, mean64], (gws1, lws1)), ("corr_std", [d64, mean64, std64], (gws1, lws1)),
                         ("corr_reduce", [d64, mean64, std64], (gws2, lws2))]:
        L = oracle_mod.Launch(kname, False, n, m, list(g[0]), list(g[1]), bl)
        oracle_mod.run_range(L, 0, L.num_groups())
    assert_parity(mean.read_array(np.float32), mean64, False, "corr mean 4096")
    assert_parity(std.read_array(np.float32), std64, False, "corr std 4096")
    assert_parity(d.read_array(np.float32), d64, False, "corr reduced data 4096")
    sym64 = np.zeros(m * m)
    L = oracle_mod.Launch("corr_corr", False, n, m, list(gws1), list(lws1), [d64, sym64]).copy(with_wcount=True)
    oracle_mod.exec_wg_partial(L, 15, -1)          # the last work-group: j1 in [3840, 4096)
    oracle_mod.exec_wg_partial(L, 0, 2)            # first two rows of the heaviest work-group
    oracle_mod.exec_wg_partial(L, 8, 1)            # one row in the middle
    mask = L.wcount[1] > 0
    assert mask.sum() > 2 * 4000
    # tolerance floor relative to the largest |symmat| entry (1 on the diagonal)
    assert_parity(np.where(mask, got_sym, 0.0), np.where(mask, L.bufs[1], 0.0), False, "corr symmat sampled")
    for b in (d, mean, std, sym):
        b.release()


@pytest.mark.parametrize("kernel,n0,n1", [("gesummv", 4096, 4096), ("bicg_s", 4096, 4096), ("syrk", 2048, 2048)])
def test_device_selection_full_size(ctx, oracle_mod, kernel, n0, n1):
    """The bench's launch configuration: COOP with device selection on.  The
    probe runs cooperatively, the next launches of the shape on the GPU alone; every result is
    the GPU-only result bit for bit and matches the oracle on sampled work-groups."""
    P = W.make(kernel, n0, n1, seed=23, lws1d=256)
    ref, _ = H.run(ctx, P, mode="gpu")
    n = P.num_groups
    seen = []
    for i in range(3):
        out, info = H.run(ctx, P, mode="coop", select=1)
        seen.append((info["probe"], info["selected"]))
        for k in P.out_indices:
            assert_bits(out[k], ref[k], f"{kernel} launch {i} {seen[-1]}")
    assert seen[0] == (1, 0) and seen[1][0] == 0, seen
    _check_sampled(oracle_mod, P, out, [0, n // 2, n - 1])


@pytest.mark.parametrize("kernel", ["gesummv", "bicg_q"])
def test_streamed_inputs_full_size(ctx, oracle_mod, kernel):
    """The bench's e2e configuration at full size: inputs written non-blocking (device copies
    stale), the row-dot matrices streamed to the GPU in row pieces while the host computes from
    the top.  Bits equal GPU-only; sampled work-groups match the oracle."""
    P = W.make(kernel, 4096, 4096, seed=24, lws1d=256)
    ref, _ = H.run(ctx, P, mode="gpu")
    bufs = H.create_buffers(ctx, P)
    for k in range(len(P.bufs)):
        if k not in P.out_indices:
            bufs[k].write(bufs[k].host_ptr, blocking=False)
    out, info = H.run(ctx, P, mode="coop", bufs=bufs, select=-1)
    assert info["streamed_wgs"] > 0 or info["cpu_did_all"] == 1, info
    for k in P.out_indices:
        assert_bits(out[k], ref[k], f"{kernel} streamed")
    n = P.num_groups
    _check_sampled(oracle_mod, P, out, [0, n // 2, n - 1])
    for b in bufs:
        b.release()
