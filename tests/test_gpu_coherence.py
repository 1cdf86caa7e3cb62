"""Multi-kernel coherence (§5.3 buffer version tracking L20.s1-9, §5.6
the D2H thread L20.s13-19, §6.2 data location tracking L20.s31-33): chains whose kernels land on
different devices run back to back -- no fcl_finish in between and no launch waiting for the
pending host sides (FCL_COUNT_LAUNCH_DRAINS stays 0) -- and every host and device copy ends
bit-identical to the all-GPU chain.  A CPU-only launch runs in queue order on the coordinator;
a GPU launch that reads its output waits on the device for the transfer of that output.  With
that wait switched off (FCL_NO_VERSION_WAIT=1) the GPU reads the stale device copy and the test
that checks it fails -- which is what the last test asserts.
"""
import itertools
import os

import numpy as np
import pytest

import fcl_harness as H
import workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_cgo_panditg14_b200 import _build, fcl
    _build.build()
    c = fcl.Context(0)
    yield c
    c.release()


def _atax(ctx, n, seed):
    P1 = W.make("atax_tmp", n, n, seed=seed, lws1d=64)
    P2 = W.make("atax_y", n, n, seed=seed + 1, lws1d=64)
    return P1, P2


def _atax_run(ctx, P1, P2, m1, m2, **o2):
    n = P1.n0
    A, x, tmp = (ctx.buffer_from_array(b) for b in P1.bufs)
    y = ctx.buffer_from_array(P2.bufs[2])
    ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode=m1)
    ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode=m2, **o2)
    ctx.finish()
    out = {"tmp_h": tmp.read_array(np.float32), "y_h": y.read_array(np.float32),
           "tmp_d": H.device_array(tmp, np.float32), "y_d": H.device_array(y, np.float32),
           "ver": (tmp.versions(), y.versions())}
    for b in (A, x, tmp, y):
        b.release()
    return out


def _same(a, b, what):
    ua, ub = np.ascontiguousarray(a).view(np.uint32), np.ascontiguousarray(b).view(np.uint32)
    assert np.array_equal(ua, ub), f"{what}: {np.count_nonzero(ua != ub)} words differ"


@pytest.mark.parametrize("m1,m2", list(itertools.product(["cpu", "gpu", "coop"], repeat=2)))
def test_atax_chain_across_devices_without_drains(ctx, m1, m2):
    P1, P2 = _atax(ctx, 640, seed=90)
    want = _atax_run(ctx, P1, P2, "gpu", "gpu")
    c0 = ctx.counters()
    got = _atax_run(ctx, P1, P2, m1, m2)
    c1 = ctx.counters()
    assert c1["launch_drains"] == c0["launch_drains"], (m1, m2, c0, c1)
    for k in ("tmp_h", "y_h", "tmp_d", "y_d"):
        if (k == "y_d" and m2 == "cpu") or (k == "tmp_d" and m1 == "cpu" and m2 == "cpu"):
            continue   # (a CPU-only output's device copy is stale by design until a GPU use)
        _same(got[k], want[k], f"{m1}->{m2} {k}")
    (te, th, td), (ye, yh, yd) = got["ver"]
    assert th == te and ye == yh and ye > te, got["ver"]       # host copies hold the expected versions
    assert td == (0 if m1 == "cpu" and m2 == "cpu" else te)    # tmp reached the device iff a GPU read it


CORR_MODES = [("coop", "coop", "coop", "coop"), ("cpu", "gpu", "coop", "gpu"), ("gpu", "cpu", "coop", "cpu"),
              ("cpu", "cpu", "coop", "gpu"), ("gpu", "gpu", "coop", "coop")]


@pytest.mark.parametrize("modes", CORR_MODES, ids=lambda m: "-".join(m))
def test_corr_chain_across_devices_without_drains(ctx, modes):
    n, m = 300, 260
    data = W.corr_chain_inputs(n, m, seed=91)
    gws1, lws1 = W.geometry("corr_mean", n, m, lws1d=32)
    gws2, lws2 = W.geometry("corr_reduce", n, m)

    def chain(ms):
        bl = [ctx.buffer_from_array(x) for x in (data, np.zeros(m, np.float32), np.zeros(m, np.float32),
                                                 np.full(m * m, -3.0, np.float32))]
        d, mean, std, sym = bl
        ctx.enqueue_ndrange("corr_mean_f32", gws1, lws1, [d, mean, n, m], mode=ms[0])
        ctx.enqueue_ndrange("corr_std_f32", gws1, lws1, [d, mean, std, n, m, 0.1], mode=ms[1])
        ctx.enqueue_ndrange("corr_reduce_f32", gws2, lws2, [d, mean, std, n, m], mode=ms[2])
        ctx.enqueue_ndrange("corr_corr_f32", gws1, lws1, [d, sym, n, m], mode=ms[3])
        ctx.finish()
        out = [b.read_array(np.float32) for b in bl]
        dev = [H.device_array(b, np.float32) if b.versions()[2] else None for b in bl]
        for b in bl:
            b.release()
        return out, dev

    want, want_d = chain(("gpu",) * 4)
    c0 = ctx.counters()
    got, got_d = chain(modes)
    c1 = ctx.counters()
    assert c1["launch_drains"] == c0["launch_drains"], (modes, c0, c1)
    for k, name in enumerate(["data", "mean", "std", "symmat"]):
        _same(got[k], want[k], f"{modes} host {name}")
        if got_d[k] is not None:
            _same(got_d[k], want_d[k], f"{modes} device {name}")


def test_gpu_reader_waits_for_cpu_only_writer(ctx):
    """A slow CPU-only producer (20 ms before its chunk) and a GPU-only consumer enqueued right
    behind it: the consumer's grid waits on the device for the producer's transfer."""
    P1, P2 = _atax(ctx, 512, seed=92)
    want = _atax_run(ctx, P1, P2, "gpu", "gpu")
    c0 = ctx.counters()
    n = P1.n0
    A, x, tmp = (ctx.buffer_from_array(b) for b in P1.bufs)
    y = ctx.buffer_from_array(P2.bufs[2])
    ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="cpu", host_delay_us=20000)
    ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode="gpu")
    ctx.finish()
    c1 = ctx.counters()
    assert c1["launch_drains"] == c0["launch_drains"]
    _same(y.read_array(np.float32), want["y_h"], "y after a slow CPU producer")
    for b in (A, x, tmp, y):
        b.release()


def test_without_the_version_wait_the_gpu_reads_stale_data(monkeypatch):
    """The same chain with the device-side wait switched off (a test hook): the GPU consumer runs
    before the CPU producer's result reaches the device and computes from the stale device copy
    (the poison the output buffer started with) -- the check above would fail."""
    from paper_conf_cgo_panditg14_b200 import fcl
    monkeypatch.setenv("FCL_NO_VERSION_WAIT", "1")
    c = fcl.Context(0)
    try:
        P1, P2 = _atax(c, 512, seed=92)
        want = _atax_run(c, P1, P2, "gpu", "gpu")
        n = P1.n0
        A, x, tmp = (c.buffer_from_array(b) for b in P1.bufs)
        y = c.buffer_from_array(P2.bufs[2])
        c.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="cpu", host_delay_us=20000)
        c.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode="gpu")
        c.finish()
        got = y.read_array(np.float32)
        assert not np.array_equal(got.view(np.uint32), want["y_h"].view(np.uint32)), \
            "the GPU read the producer's data although it did not wait for it"
        for b in (A, x, tmp, y):
            b.release()
    finally:
        c.release()


@pytest.mark.parametrize("seed", range(12))
def test_random_chains_across_devices(ctx, seed):
    """Random chains of dependent launches (RAW / WAR / WAW through four shared vectors) with every
    launch on a random device (cooperative with random host / GPU delays, GPU-only, CPU-only,
    device selection), no fcl_finish in between and the occasional read in the middle: every host
    and device copy ends bit-identical to the same chain run one launch at a time on the GPU.
    Integer kernels (exact wraparound), so values never overflow into inf."""
    rng = np.random.default_rng(1000 + seed)
    n = 384
    A = rng.integers(-8, 9, size=n * n, dtype=np.int32)
    vecs0 = [rng.integers(-8, 9, size=n, dtype=np.int32) for _ in range(4)]
    gws, lws = (n,), (64,)
    kernels = ["atax_tmp_i32", "atax_y_i32", "bicg_s_i32", "bicg_q_i32"]
    ops = []
    for _ in range(14):
        i, j = rng.choice(4, size=2, replace=False)
        ops.append((kernels[rng.integers(4)], int(i), int(j)))

    def run(modes):
        bA = ctx.buffer_from_array(A)
        bv = [ctx.buffer_from_array(v) for v in vecs0]
        for k, (name, i, j) in enumerate(ops):
            m = modes[k]
            opts = dict(m[1])
            ctx.enqueue_ndrange(name, gws, lws, [bA, bv[i], bv[j], n, n], mode=m[0], **opts)
            if modes is REF:
                ctx.finish()
            elif m[2]:   # a read in the middle of the chain
                bv[j].read_array(np.int32)
        ctx.finish()
        out = [b.read_array(np.int32) for b in bv] + [H.device_array(b, np.int32) if b.versions()[2] else None for b in bv]
        for b in [bA] + bv:
            b.release()
        return out

    REF = [("gpu", {}, False)] * len(ops)
    choices = [("coop", {}), ("coop", {"host_delay_us": 100}), ("coop", {"gpu_delay_us": 200}), ("gpu", {}),
               ("cpu", {}), ("cpu", {"host_delay_us": 300}), ("coop", {"select": 1}), ("coop", {"forced_split": 3})]
    modes = [choices[rng.integers(len(choices))] + (bool(rng.random() < 0.15),) for _ in ops]
    want = run(REF)
    got = run(modes)
    for q in range(4):
        _same(got[q], want[q], f"seed {seed} vector {q} host ({modes})")
        if got[4 + q] is not None:
            _same(got[4 + q], want[q], f"seed {seed} vector {q} device")
