"""Device selection from online profiles (opts.select): a COOP launch of a shape
whose last cooperative probe showed that one device cannot contribute runs on the other alone,
with every FCL_SELECT_PERIOD-th launch (16) of the shape probing cooperatively again.  Whatever
runs, the result is the single-device result bit for bit."""
import numpy as np
import pytest

import fcl_harness as H
import workloads as W
from _util import assert_bits

pytestmark = pytest.mark.gpu

SEL_COOP, SEL_GPU, SEL_CPU = 0, 1, 2
PATH_NONE, PATH_PLAIN = 0, 3


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_cgo_panditg14_b200 import _build, fcl
    _build.build()
    c = fcl.Context(0)
    yield c
    c.release()


def test_gpu_favoured_shape_runs_on_the_gpu_alone(ctx):
    """SYRK 512: the GPU finishes long before the host's first 2 % chunk (21 work-groups), so the
    probe records "host finished nothing": the host is far slower on this shape and the next
    probe comes 256 launches later; all launches in between are GPU-only plain grids."""
    P = W.make("syrk", 512, 512, seed=5)
    ref, _ = H.run(ctx, P, mode="gpu")
    c0 = ctx.counters()
    seen = []
    for i in range(50):
        out, info = H.run(ctx, P, mode="coop", select=1)
        seen.append((info["probe"], info["selected"]))
        for k in P.out_indices:
            assert_bits(out[k], ref[k], f"launch {i}")
        if info["probe"]:
            assert info["selected"] == SEL_COOP and info["gpu_path"] in (1, 2)
        else:
            assert info["selected"] == SEL_GPU, seen
            assert info["gpu_path"] == PATH_PLAIN and info["cpu_wgs"] == 0
    assert seen[0] == (1, SEL_COOP), seen
    assert all(s == (0, SEL_GPU) for s in seen[1:]), seen
    c1 = ctx.counters()
    assert c1["sel_gpu"] - c0["sel_gpu"] == 49 and c1["probe"] - c0["probe"] == 1, (c0, c1)
    assert c1["coop"] - c0["coop"] == 1 and c1["gpu_only"] - c0["gpu_only"] == 0, (c0, c1)


def test_probe_backoff_doubles_while_confirmed(ctx):
    """A probe in which the host did complete work but not enough (below 10 % of the range) keeps
    the shape on the GPU; each confirming probe doubles the distance to the next (16, 32, ...)."""
    P = W.make("conv2d", 2048, 2048, seed=6, out_init="zero")
    c0 = ctx.counters()
    probes = []
    for i in range(60):
        out, info = H.run(ctx, P, mode="coop", select=1, gpu_delay_us=0)
        if info["probe"]:
            probes.append((i, info["cpu_wgs"], info["selected"]))
    c1 = ctx.counters()
    assert probes and probes[0][0] == 0, probes
    gaps = [b[0] - a[0] for a, b in zip(probes, probes[1:])]
    # a cooperative outcome probes every launch (gap 1); a GPU one waits the base period, double
    # the previous gap when confirmed, or the long one after a probe without host progress
    assert all(g in (1, 16, 32, 64, 128, 256) for g in gaps), (probes, gaps)
    assert c1["probe"] - c0["probe"] == len(probes), (c0, c1, probes)


def test_host_favoured_shape_runs_on_the_host_alone(ctx, monkeypatch):
    """The host covers a small ATAX range before the GPU exits (L16.s21) in a probe started on an
    idle GPU -- made slow here by a fault-injection sleep in front of the grid -- so the next
    launch of the shape runs on the host alone and leaves the device copy stale (refreshed on
    the next GPU use).  A probe whose grid waits behind earlier GPU work proves nothing: a GPU
    busy with a long SYRK does not make the host the faster device."""
    from paper_conf_cgo_panditg14_b200 import fcl
    P = W.make("atax_tmp", 64, 64, seed=7, lws1d=16)
    ref, _ = H.run(ctx, P, mode="gpu")
    # a GPU busy with earlier work: the probe proves nothing, the shape stays cooperative
    big = W.make("syrk", 2048, 2048, seed=6)
    bb = H.create_buffers(ctx, big)
    ctx.enqueue_ndrange(H.kernel_name(big), big.gws, big.lws, H.make_args(ctx, big, bb), mode="gpu")
    out, info = H.run(ctx, P, mode="coop", select=1)
    assert info["probe"] == 1
    _, info = H.run(ctx, P, mode="coop", select=1)
    assert info["selected"] != SEL_CPU, info   # cooperative, or the GPU alone if it won anyway
    for b in bb:
        b.release()
    # an idle but slow GPU (its grid idles 20 ms first): the host covers the range, the shape
    # moves to the host
    monkeypatch.setenv("FCL_TEST_GPU_DELAY_US", "20000")
    c2 = fcl.Context(0)
    try:
        out, info = H.run(c2, P, mode="coop", select=1)
        assert info["probe"] == 1 and info["cpu_did_all"] == 1, info
        for k in P.out_indices:
            assert_bits(out[k], ref[k], "probe")
        bufs = H.create_buffers(c2, P)
        out, info = H.run(c2, P, mode="coop", select=1, bufs=bufs)
        assert info["selected"] == SEL_CPU and info["gpu_path"] == PATH_NONE and info["d2h_bytes"] == 0, info
        for k in P.out_indices:
            assert_bits(out[k], ref[k], "host alone")
    # the stale device copy is refreshed before a GPU launch reads it
        Q = W.make("atax_y", 64, 64, seed=7, lws1d=16)
        Q.bufs[0] = P.bufs[0]
        Q.bufs[1] = out[2].copy()
        refq, _ = H.run(c2, Q, mode="cpu")
        yb = c2.buffer_from_array(Q.bufs[2])
        outq, _ = H.run(c2, Q, mode="gpu", bufs=[bufs[0], bufs[2], yb])
        for k in Q.out_indices:
            assert_bits(outq[k], refq[k], "GPU after a host-alone launch")
        for b in bufs + [yb]:
            b.release()
    finally:
        c2.release()


def test_selection_off_always_cooperative(ctx):
    P = W.make("syrk", 256, 256, seed=8)
    for _ in range(4):
        _, info = H.run(ctx, P, mode="coop", select=-1)
        assert info["selected"] == SEL_COOP and info["probe"] == 0 and info["gpu_path"] in (1, 2)


def test_test_hooks_are_never_redirected(ctx):
    P = W.make("syrk", 256, 256, seed=9)
    ref, _ = H.run(ctx, P, mode="gpu")
    for _ in range(3):
        H.run(ctx, P, mode="coop", select=1)
    out, info = H.run(ctx, P, mode="coop", select=1, forced_split=P.num_groups // 2)
    assert info["selected"] == SEL_COOP and info["cpu_wgs"] == P.num_groups - P.num_groups // 2
    for k in P.out_indices:
        assert_bits(out[k], ref[k], "forced split")


def test_lazy_write_refresh_and_host_alone(ctx):
    """A non-blocking write of a whole buffer leaves the device copy stale (include/fcl.h): a
    GPU launch refreshes it first (the bytes show in fcl_get_counters), a CPU-only launch moves
    nothing, and both give the reference result."""
    P = W.make("gesummv", 512, seed=31, lws1d=64)
    ref, _ = H.run(ctx, P, mode="gpu")
    bufs = H.create_buffers(ctx, P)
    ins = [bufs[k] for k in range(len(P.bufs)) if k not in P.out_indices]
    for mode, moves in (("gpu", True), ("cpu", False)):
        for b in ins:
            b.write(b.host_ptr, blocking=False)
        c0 = ctx.counters()
        out, _ = H.run(ctx, P, mode=mode, bufs=bufs)
        c1 = ctx.counters()
        moved = c1["h2d_bytes"] - c0["h2d_bytes"]
        if moves:
            assert moved >= sum(b.nbytes for b in ins), (moved, mode)
        else:
            assert moved == 0, (moved, mode)
        for k in P.out_indices:
            assert_bits(out[k], ref[k], f"after lazy write, {mode}")
    for b in bufs:
        b.release()


@pytest.mark.parametrize("kernel,integer,lws,n1", [("gesummv", False, 64, 2048), ("gesummv", True, 64, 2048),
                                                   ("atax_tmp", False, 32, 2048), ("bicg_q", False, 128, 2048),
                                                   ("atax_tmp", False, 32, 2045), ("bicg_q", True, 64, 2047)])
def test_streamed_inputs(ctx, kernel, integer, lws, n1):
    """Stale input matrices (a non-blocking whole-buffer write) of a row-dot kernel stream to the
    GPU in row pieces while the host computes from the top; GPU work-groups
    wait for their rows or for the host to cover them.  The result is the GPU-only one bit for
    bit, with the host slowed down (the GPU then takes most pieces) and at full speed.  Rows that
    are not a multiple of 16 bytes (n1 % 4 != 0, the scalar path) put piece boundaries inside
    cache lines: the streamed rows are read through L2 only, never from a stale L1 line."""
    P = W.make(kernel, 2048, n1, integer=integer, seed=33, lws1d=lws)
    ref, _ = H.run(ctx, P, mode="gpu")
    for kw in (dict(host_delay_us=300), dict()):
        bufs = H.create_buffers(ctx, P)
        for k in range(len(P.bufs)):
            if k not in P.out_indices:
                bufs[k].write(bufs[k].host_ptr, blocking=False)
        out, info = H.run(ctx, P, mode="coop", bufs=bufs, select=-1, **kw)
        assert info["streamed_wgs"] > 0 or info["cpu_did_all"] == 1, info
        if kw:
            assert info["streamed_wgs"] > 0, info
        for k in P.out_indices:
            assert_bits(out[k], ref[k], f"{kernel} streamed {kw}")
        for b in bufs:
            b.release()


def test_streamed_probe_with_host_majority_moves_to_the_host(monkeypatch):
    """A streamed probe (stale inputs crossing PCIe while the launch runs) of which the host covered
    at least FCL_SELECT_STREAM_SHARE of the range sends the next launches of that shape to the
    host alone: no bytes cross PCIe for them.  The share is set to 0 here (any streamed probe the
    GPU finished qualifies, FCL_SELECT_MIN_SHARE 0 so that the GPU-alone rule cannot take it
    first); the same shape with resident inputs is not streamed and stays cooperative.  Every
    result is the GPU-only one bit for bit."""
    from paper_conf_cgo_panditg14_b200 import fcl
    monkeypatch.setenv("FCL_SELECT_STREAM_SHARE", "0")
    monkeypatch.setenv("FCL_SELECT_MIN_SHARE", "0")
    c2 = fcl.Context(0)
    try:
        # the bench's size: the link delivers a third of the rows while the host computes the rest
        P = W.make("gesummv", 4096, seed=34, lws1d=64)
        ref, _ = H.run(c2, P, mode="gpu")
        bufs = H.create_buffers(c2, P)
        ins = [bufs[k] for k in range(len(P.bufs)) if k not in P.out_indices]
        seen = []
        for i in range(4):
            for b in ins:
                b.write(b.host_ptr, blocking=False)
            c0 = c2.counters()
            out, info = H.run(c2, P, mode="coop", bufs=bufs, select=1)
            moved = c2.counters()["h2d_bytes"] - c0["h2d_bytes"]
            seen.append((info["probe"], info["selected"], info["streamed_wgs"] > 0, moved))
            for k in P.out_indices:
                assert_bits(out[k], ref[k], f"launch {i}")
        assert seen[0][0] == 1 and seen[0][2], seen
        assert all(s[:2] == (0, SEL_CPU) and s[3] == 0 for s in seen[1:]), seen
        # resident inputs (blocking writes refresh the device copies): another key, nothing to
        # stream, so the probe's outcome is the ordinary one -- not the host alone (a lite grid
        # computes everything: the GPU alone)
        for b in ins:
            b.write(b.host_ptr)
        infos = []
        for i in range(2):
            out, info = H.run(c2, P, mode="coop", bufs=bufs, select=1)
            infos.append(info)
            for k in P.out_indices:
                assert_bits(out[k], ref[k], f"resident launch {i}")
        assert infos[0]["probe"] == 1 and infos[0]["streamed_wgs"] == 0, infos[0]
        assert infos[1]["selected"] != SEL_CPU and infos[1]["gpu_path"] != PATH_NONE, infos[1]
        for b in bufs:
            b.release()
    finally:
        c2.release()


def test_e2e_loop_selection_and_streaming(ctx):
    """The bench's e2e loop at a reduced size: every step writes the inputs (non-blocking, device
    copies stale), runs GESUMMV + BICG s/q as COOP launches with device selection, reads the
    outputs.  Probes, streamed launches, host-alone and GPU-alone launches interleave over 20
    steps; every step's results equal the GPU-only ones bit for bit."""
    Ps = [W.make("gesummv", 1024, seed=41, lws1d=64),
          W.make("bicg_s", 1024, 1024, seed=42, lws1d=64),
          W.make("bicg_q", 1024, 1024, seed=43, lws1d=64)]
    refs = [H.run(ctx, P, mode="gpu")[0] for P in Ps]
    bufs = [H.create_buffers(ctx, P) for P in Ps]
    c0 = ctx.counters()
    for step in range(20):
        for P, bl in zip(Ps, bufs):
            for k in range(len(P.bufs)):
                if k not in P.out_indices:
                    bl[k].write(bl[k].host_ptr, blocking=False)
        for P, bl in zip(Ps, bufs):
            ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bl), mode="coop", select=1)
        ctx.finish()
        for P, bl, ref in zip(Ps, bufs, refs):
            for k in P.out_indices:
                assert_bits(bl[k].read_array(np.float32), ref[k], f"{P.kernel} step {step}")
    c1 = ctx.counters()
    assert c1["probe"] > c0["probe"]
    for bl in bufs:
        for b in bl:
            b.release()


_FIRST_LAUNCH_SCRIPT = r'''
import sys
sys.path.insert(0, sys.argv[1])
import numpy as np
import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl
ctx = fcl.Context(0)
P = W.make("gesummv", 2048, seed=51, lws1d=64)
Q = W.make("conv2d", 512, 512, seed=52)
bp, bq = H.create_buffers(ctx, P), H.create_buffers(ctx, Q)
for k in range(len(P.bufs)):
    if k not in P.out_indices:
        bp[k].write(bp[k].host_ptr, blocking=False)
# a streamed launch (its grid waits for host-driven copies), then kernels this process has never
# launched, queued behind it without a drain
ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bp), mode="coop", select=-1, host_delay_us=200)
ctx.enqueue_ndrange(H.kernel_name(Q), Q.gws, Q.lws, H.make_args(ctx, Q, bq), mode="coop", select=-1)
ctx.finish()
print("ok")
'''


def test_first_launch_of_a_kernel_behind_a_streamed_grid(tmp_path):
    """Regression: with CUDA's lazy module loading a kernel was loaded at its first launch, which
    could wait for a cooperative grid that itself waited for host-driven copies of streamed inputs
    (a deadlock, caught by the 5 s guard as a launch failure).  The context now loads every
    kernel at creation; a fresh process launching a new kernel behind a streamed one must finish."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = tmp_path / "first_launch.py"
    script.write_text(_FIRST_LAUNCH_SCRIPT)
    env = dict(os.environ, FCL_SELECT="0")
    r = subprocess.run([sys.executable, str(script), root], capture_output=True, text=True, timeout=120, env=env)
    assert r.returncode == 0 and "ok" in r.stdout, (r.stdout[-2000:], r.stderr[-2000:])


def _atax_chain(ctx, seed=0):
    """BASELINE configs[0]: ATAX N=256, 16 work-groups per kernel; kernel 2 reads kernel 1's tmp."""
    P1 = W.make("atax_tmp", 256, 256, seed=seed, lws1d=16, out_init="zero")
    P2 = W.make("atax_y", 256, 256, seed=seed + 1, lws1d=16, out_init="zero")
    b1, b2 = H.create_buffers(ctx, P1), H.create_buffers(ctx, P2)
    b2[0].release(); b2[0] = b1[0]   # A
    b2[1].release(); b2[1] = b1[2]   # tmp
    return (P1, b1), (P2, b2)


def test_sequence_selection_atax_chain(ctx):
    """Sequence selection (last item): the two ATAX launches between fcl_finish
    calls are timed as one sequence; the probes' host rates put the host alone within 2x, so a
    trial of two sequences runs every launch on the host alone (info.seq_host) and the faster
    median wins.  Whatever each sequence ran, y and tmp equal the GPU-only chain bit for bit."""
    (P1, b1), (P2, b2) = _atax_chain(ctx, seed=61)
    launches = [(P1, b1), (P2, b2)]

    def step(mode, select):
        for P, b in launches:
            ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=mode, select=select)
        ctx.finish()
        return (b1[2].read_array(np.float32).copy(), b2[2].read_array(np.float32).copy())

    ref = step("gpu", 0)
    c0 = ctx.counters()
    for i in range(80):
        got = step("coop", 1)
        assert_bits(got[0], ref[0], f"tmp, sequence {i}")
        assert_bits(got[1], ref[1], f"y, sequence {i}")
    c1 = ctx.counters()
    d = {k: c1[k] - c0[k] for k in c1}
    assert d["seq_trials"] >= 1, d
    assert d["seq_host"] >= 4 and d["seq_host"] % 2 == 0, d   # whole sequences: both launches
    assert d["seq_host"] <= d["sel_cpu"], d
    for bl in (b1, b2):
        for k, b in enumerate(bl):
            if not (bl is b2 and k in (0, 1)):
                b.release()


def test_sequence_selection_never_tries_a_hopeless_host(ctx):
    """GESUMMV 4096: the GPU finishes before the host's first chunk, so the host rate is unknown
    and no trial ever runs the host alone (it would cost ~40x the GPU's time)."""
    P = W.make("gesummv", 4096, seed=62, lws1d=256)
    b = H.create_buffers(ctx, P)
    c0 = ctx.counters()
    for i in range(40):
        ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="coop", select=1)
        ctx.finish()
    c1 = ctx.counters()
    assert c1["seq_host"] == c0["seq_host"] and c1["seq_trials"] == c0["seq_trials"], (c0, c1)
    for x in b:
        x.release()


def test_sequence_plan_broken_midway(ctx):
    """A sequence that starts like a signature whose plan is "host alone" but then launches a
    different kernel: the first launch runs on the host by the plan, the plan stops at the
    mismatch, the rest runs by per-launch selection -- and every result is still the GPU-only
    one bit for bit (sequences alternate between the two shapes, 60 times)."""
    (P1, b1), (P2, b2) = _atax_chain(ctx, seed=71)
    Q = W.make("gesummv", 256, seed=72, lws1d=16, out_init="zero")
    bq = H.create_buffers(ctx, Q)

    def launch(P, b, mode, select):
        ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=mode, select=select)

    def seq(kind, mode, select):
        launch(P1, b1, mode, select)
        if kind == "a":
            launch(P2, b2, mode, select)
        else:
            launch(Q, bq, mode, select)
        ctx.finish()
        out = [b1[2].read_array(np.float32).copy()]
        out.append(b2[2].read_array(np.float32).copy() if kind == "a" else bq[4].read_array(np.float32).copy())
        return out

    ref = {k: seq(k, "gpu", 0) for k in ("a", "b")}
    c0 = ctx.counters()
    for i in range(60):
        k = "a" if i % 3 else "b"
        got = seq(k, "coop", 1)
        for g, r in zip(got, ref[k]):
            assert_bits(g, r, f"sequence {i} ({k})")
    c1 = ctx.counters()
    # host plans ran (this test's trial, or the standing choice of the ATAX signature an earlier
    # test of the module established: sequence keys are shapes, not buffers)
    assert c1["seq_host"] > c0["seq_host"] or c1["seq_trials"] > c0["seq_trials"], (c0, c1)
    for bl in (b1, b2, bq):
        for k, b in enumerate(bl):
            if not (bl is b2 and k in (0, 1)):
                b.release()
