"""The cooperative race itself, observed on the GPU.

* Exactly-once (north_star; PAPER.md L16.s9 "the CPU and GPU ... non-overlapping parts"): with
  ``record_exec_counts`` the runtime counts, per work-group, completed GPU task fragments and
  completed host executions.  At EVERY forced split s (the GPU is told s before it starts, its
  first task included) each work-group below s ran completely on the GPU and never on the host,
  each one at or above s ran once on the host and never on the GPU -- tile tasks that straddle s
  store only their work-groups below it.
* Free-running races at the configs' sizes with a slow GPU (``gpu_delay_us``, every dispatcher
  task starts late): the host covers a suffix, the GPU's dispatcher skips or aborts covered tasks
  (``gpu_watermark < n_wg``), the merge runs (``merged``), every work-group completed on at least
  one device, and host and device copies equal the GPU-only result bit for bit.
* Config 1 (BASELINE.json configs[0]): ATAX N=256, lws 16 -> 16 work-groups per kernel; all 17
  splits per kernel with exactly-once counts, all 17^2 joint splits, 100 free-running runs with
  random host and GPU delays, against the oracle (PAPER.md L12.s22, s.33-35).
* The runtime's C11 chunk sizer (PAPER.md L18.s23-32) against ``oracle.chunk_schedule`` fed the
  chunk times the runtime measured.
"""
import numpy as np
import pytest

import fcl_harness as H
import workloads as W
from _util import assert_bits, assert_parity, oracle_outputs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_cgo_panditg14_b200 import _build, fcl
    _build.build()
    c = fcl.Context(0)
    yield c
    c.release()


def _dt(P):
    return np.int32 if P.integer else np.float32


def check_exactly_once(cnt, s, n, what):
    """Forced split s: [0, s) completely and only on the GPU, [s, n) once and only on the host."""
    gd, gf, cd = cnt["gpu_done"][:n], cnt["gpu_frags"][:n], cnt["cpu_done"][:n]
    assert np.all(gf > 0), f"{what}: a work-group no GPU task covers"
    lo, hi = np.arange(n) < s, np.arange(n) >= s
    bad = np.nonzero(lo & ((gd != gf) | (cd != 0)))[0]
    assert bad.size == 0, f"{what}: GPU part wrong at {bad[:5]}: gpu {gd[bad[:5]]}/{gf[bad[:5]]} cpu {cd[bad[:5]]}"
    bad = np.nonzero(hi & ((gd != 0) | (cd != 1)))[0]
    assert bad.size == 0, f"{what}: host part wrong at {bad[:5]}: gpu {gd[bad[:5]]}/{gf[bad[:5]]} cpu {cd[bad[:5]]}"


def check_race_counts(cnt, n, published, what):
    """Free-running: every work-group completed on some device; the host ran each at most once,
    and every published chunk completely -- the published work-groups are the suffix
    [published, n) (descending chunks, L14.s36; status follows data, L16.s15).  Below it only an
    abandoned chunk's work-groups may have host completions, and the GPU completed all of them."""
    gd, gf, cd = cnt["gpu_done"][:n], cnt["gpu_frags"][:n], cnt["cpu_done"][:n]
    full_gpu = gd == gf
    assert np.all(full_gpu | (cd >= 1)), f"{what}: work-groups nobody completed: {np.nonzero(~(full_gpu | (cd >= 1)))[0][:5]}"
    assert np.all(cd <= 1), f"{what}: host ran a work-group twice"
    assert np.all(cd[published:] == 1), f"{what}: a published work-group the host did not complete"
    assert np.all(full_gpu[:published]), f"{what}: an unpublished work-group the GPU did not complete"
    return int(np.count_nonzero(cd)), int(np.count_nonzero(gd == 0))


FORCED_CASES = [
    # kernel, n0, n1, integer, lws1d, lws2d -- tiles that span several work-groups (masking)
    ("atax_tmp", 256, 256, False, 16, None),
    ("atax_y", 256, 256, True, 16, None),
    ("gesummv", 300, 300, False, 32, None),
    ("syrk", 200, 70, False, None, (32, 8)),        # upper-triangle tiles + mirrors
    ("syrk", 256, 64, True, None, (16, 4)),
    ("syr2k", 200, 70, False, None, (32, 8)),
    ("conv2d", 150, 300, False, None, (32, 8)),
    ("conv2d", 70, 130, True, None, (16, 4)),
    ("corr_reduce", 120, 300, False, None, (32, 8)),
    ("corr_corr", 100, 300, False, 32, None),       # 4 work-groups per 128-row tile block
    ("corr_mean", 200, 300, False, 64, None),
]


def _ids(c):
    return f"{c[0]}-{'i32' if c[3] else 'f32'}-{c[1]}x{c[2]}-" + (f"l{c[4]}" if c[4] else f"l{c[5][0]}x{c[5][1]}")


def _problem(c, seed=0):
    kernel, n0, n1, integer, l1, l2 = c
    return W.make(kernel, n0, n1, integer=integer, seed=seed, lws1d=l1 or 256, lws2d=l2 or (32, 8))


@pytest.mark.parametrize("case", FORCED_CASES, ids=_ids)
def test_exactly_once_every_forced_split(ctx, case):
    P = _problem(case, seed=3)
    n = P.num_groups
    ref, ginfo = H.run(ctx, P, mode="gpu", record_exec_counts=1)
    cnt = ctx.exec_counts(n)
    check_exactly_once(cnt, n, n, f"{_ids(case)} gpu-only")
    _, cinfo = H.run(ctx, P, mode="cpu", record_exec_counts=1)
    check_exactly_once(ctx.exec_counts(n), 0, n, f"{_ids(case)} cpu-only")
    splits = range(n + 1) if n <= 40 else sorted({0, 1, 2, n // 7, n // 3, n // 2, n - 2, n - 1, n} |
                                                set(range(3 * n // 5, 3 * n // 5 + 9)))
    for s in splits:
        bufs = H.create_buffers(ctx, P)
        out, info = H.run(ctx, P, mode="coop", bufs=bufs, forced_split=s, record_exec_counts=1)
        check_exactly_once(ctx.exec_counts(n), s, n, f"{_ids(case)} split {s}")
        for k in P.out_indices:
            assert_bits(out[k], ref[k], f"{_ids(case)} split {s} host buf{k}")
            assert_bits(H.device_array(bufs[k], _dt(P)), ref[k], f"{_ids(case)} split {s} device buf{k}")
        for b in bufs:
            b.release()


def test_exec_counts_api_errors(ctx):
    from paper_conf_cgo_panditg14_b200 import fcl
    P = W.make("atax_tmp", 64, 64, seed=1, lws1d=16)
    H.run(ctx, P, mode="gpu", record_exec_counts=1)
    with pytest.raises(fcl.FclError):
        ctx.exec_counts(P.num_groups - 1)
    cnt = ctx.exec_counts(P.num_groups + 3)   # longer arrays: the tail stays 0
    assert np.all(cnt["gpu_frags"][P.num_groups:] == 0)


# ---------------------------------------------------------------- free-running at config sizes
RACE_FULL = [
    # kernel, n0, n1, lws1d, gpu_delay_us: a slow GPU lets the host cover part of the range
    ("conv2d", 16384, 16384, None, 30),
    ("syrk", 2048, 2048, None, 40000),
    ("syr2k", 2048, 2048, None, 80000),
    ("corr_reduce", 4096, 4096, None, 1000),
    ("gesummv", 4096, 4096, 64, 3000),
]


@pytest.mark.parametrize("case", RACE_FULL, ids=lambda c: f"{c[0]}-{c[1]}")
def test_free_running_race_is_observable(ctx, case):
    kernel, n0, n1, l1, delay = case
    P = W.make(kernel, n0, n1, seed=5, lws1d=l1 or 256, out_init="zero")
    n = P.num_groups
    ref, _ = H.run(ctx, P, mode="gpu")
    bufs = H.create_buffers(ctx, P)
    out, info = H.run(ctx, P, mode="coop", bufs=bufs, gpu_delay_us=delay, record_exec_counts=1)
    what = f"{kernel} {n0}x{n1} free-running, GPU delay {delay} us"
    assert info["gpu_path"] == 1, f"{what}: not the dispatcher: {info['gpu_path']}"
    assert info["cpu_wgs"] > 0, f"{what}: host finished no chunk: {info}"
    assert info["gpu_watermark"] < n, f"{what}: the GPU never acted on a watermark: {info}"
    assert info["merged"] == 1, f"{what}: no merge: {info}"
    host_wgs, gpu_skipped = check_race_counts(ctx.exec_counts(n), n, info["published_watermark"], what)
    print(f"{what}: host {host_wgs}/{n} work-groups in {info['n_chunks']} chunks, GPU skipped {gpu_skipped}, "
          f"gpu_watermark {info['gpu_watermark']}, published {info['published_watermark']}, race {info['race']}")
    assert host_wgs > 0 and gpu_skipped > 0, (what, host_wgs, gpu_skipped)
    for k in P.out_indices:
        assert_bits(out[k], ref[k], f"{what} host buf{k}")
        assert_bits(H.device_array(bufs[k], _dt(P)), ref[k], f"{what} device buf{k}")
    for b in bufs:
        b.release()


# ---------------------------------------------------------------- config 1: ATAX N = 256
def _atax256(ctx, seed):
    n = 256
    P1 = W.make("atax_tmp", n, n, seed=seed, lws1d=16)
    P2 = W.make("atax_y", n, n, seed=seed + 1, lws1d=16)
    P2.bufs[0] = P1.bufs[0]
    A, x, tmp = (ctx.buffer_from_array(b) for b in P1.bufs)
    y = ctx.buffer_from_array(P2.bufs[2])
    return P1, P2, (A, x, tmp, y)


def _atax_ref(oracle_mod, P1, P2):
    R1 = oracle_outputs(oracle_mod, P1)[2]
    n = P1.n0
    L2 = oracle_mod.Launch("atax_y", False, n, n, list(P2.gws), list(P2.lws),
                           [P1.bufs[0].astype(np.float64), R1.copy(), np.zeros(n)])
    oracle_mod.run_range(L2, 0, L2.num_groups())
    return R1, L2.bufs[2]


def _atax_step(ctx, P1, P2, B, o1, o2):
    A, x, tmp, y = B
    n = P1.n0
    ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="coop", **o1)
    ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode="coop", **o2)
    ctx.finish()
    return tmp.read_array(np.float32), y.read_array(np.float32)


def test_config1_atax256_every_split_per_kernel(ctx, oracle_mod):
    P1, P2, B = _atax256(ctx, seed=70)
    A, x, tmp, y = B
    assert P1.num_groups == 16 and P2.num_groups == 16
    R1, R2 = _atax_ref(oracle_mod, P1, P2)
    ref_t, ref_y = _atax_step(ctx, P1, P2, B, dict(forced_split=16), dict(forced_split=16))   # GPU alone
    assert_parity(ref_t, R1, False, "atax256 tmp")
    assert_parity(ref_y, R2, False, "atax256 y")
    n = P1.n0
    for s in range(17):
        ctx.enqueue_ndrange("atax_tmp_f32", P1.gws, P1.lws, [A, x, tmp, n, n], mode="coop",
                            forced_split=s, record_exec_counts=1)
        check_exactly_once(ctx.exec_counts(16), s, 16, f"atax_tmp split {s}")
        ctx.enqueue_ndrange("atax_y_f32", P2.gws, P2.lws, [A, tmp, y, n, n], mode="coop",
                            forced_split=s, record_exec_counts=1)
        check_exactly_once(ctx.exec_counts(16), s, 16, f"atax_y split {s}")
        ctx.finish()
        assert_bits(tmp.read_array(np.float32), ref_t, f"tmp split {s}")
        assert_bits(y.read_array(np.float32), ref_y, f"y split {s}")
        assert_bits(H.device_array(y, np.float32), ref_y, f"y device copy split {s}")
    for b in B:
        b.release()


def test_config1_atax256_all_joint_splits(ctx, oracle_mod):
    P1, P2, B = _atax256(ctx, seed=72)
    R1, R2 = _atax_ref(oracle_mod, P1, P2)
    ref_t, ref_y = _atax_step(ctx, P1, P2, B, dict(forced_split=16), dict(forced_split=16))
    assert_parity(ref_y, R2, False, "atax256 y")
    for s1 in range(17):
        for s2 in range(17):
            t, yy = _atax_step(ctx, P1, P2, B, dict(forced_split=s1), dict(forced_split=s2))
            assert_bits(t, ref_t, f"tmp joint split ({s1}, {s2})")
            assert_bits(yy, ref_y, f"y joint split ({s1}, {s2})")
    for b in B:
        b.release()


def test_config1_atax256_free_running_random_delays(ctx, oracle_mod):
    P1, P2, B = _atax256(ctx, seed=74)
    R1, R2 = _atax_ref(oracle_mod, P1, P2)
    ref_t, ref_y = _atax_step(ctx, P1, P2, B, dict(forced_split=16), dict(forced_split=16))
    assert_parity(ref_y, R2, False, "atax256 y")
    rng = np.random.default_rng(75)
    host_shares = []
    for r in range(100):
        o1 = dict(host_delay_us=int(rng.integers(0, 200)), gpu_delay_us=int(rng.choice([0, 0, 20, 200])))
        o2 = dict(host_delay_us=int(rng.integers(0, 200)), gpu_delay_us=int(rng.choice([0, 0, 20, 200])))
        t, yy = _atax_step(ctx, P1, P2, B, o1, o2)
        host_shares.append(ctx.launch_info()["cpu_wgs"])
        assert_bits(t, ref_t, f"tmp free run {r} {o1}")
        assert_bits(yy, ref_y, f"y free run {r} {o2}")
    # the race went both ways over the 100 runs
    assert max(host_shares) > 0, host_shares


# ---------------------------------------------------------------- C11 in the runtime vs the oracle
@pytest.mark.parametrize("init,step", [(2, 2), (1, 3), (5, 0)])
def test_runtime_chunk_sizes_follow_c11(ctx, oracle_mod, init, step):
    """The runtime's host chunk sizes are the C11 heuristic (L18.s23-32) applied to the chunk
    times the runtime itself measured (info.chunk_ms), as the oracle's pure function computes it."""
    P = W.make("gesummv", 4096, seed=9, lws1d=16, out_init="zero")   # 256 work-groups
    n = P.num_groups
    ref, _ = H.run(ctx, P, mode="gpu")
    bufs = H.create_buffers(ctx, P)
    out, info = H.run(ctx, P, mode="coop", bufs=bufs, gpu_delay_us=20000, init_chunk_pct=init,
                      step_pct=step)
    k = info["n_c11_chunks"]
    assert k >= 3, f"too few C11 chunks to pin the heuristic: {info}"
    sizes, times = info["chunk_sizes"][:k], info["chunk_ms"][:k]
    want = oracle_mod.chunk_schedule(n, min_units=1, init_pct=init, step_pct=step, times=times[:k - 1])
    assert sizes == want[:k], (sizes, want[:k], times)
    for q in P.out_indices:
        assert_bits(out[q], ref[q], f"gesummv C11 run buf{q}")
    for b in bufs:
        b.release()


@pytest.mark.parametrize("kernel,lws2d", [("conv2d", (32, 8)), ("syrk", (32, 8)), ("corr_reduce", (16, 4))])
def test_exactly_once_inside_a_slice(ctx, kernel, lws2d):
    """A multi-GPU slice [lo, hi) split at s (forced): [lo, s) on the GPU only, [s, hi) once on the
    host only, and nothing outside the slice on either device."""
    P = W.make(kernel, 300 if kernel != "syrk" else 512, 200 if kernel != "syrk" else 64, seed=7, lws2d=lws2d)
    n = P.num_groups
    k = ctx.kernel(H.kernel_name(P))
    lo, hi = ctx.slice_range(k, P.gws, P.lws, 1, 3)
    assert 0 < lo < hi < n
    for s in sorted({lo, lo + 1, (lo + hi) // 2, hi - 1, hi}):
        bufs = H.create_buffers(ctx, P)
        H.run(ctx, P, mode="coop", bufs=bufs, wg_lo=lo, wg_hi=hi, forced_split=s, record_exec_counts=1)
        c = ctx.exec_counts(n)
        f = np.arange(n)
        inside = (f >= lo) & (f < hi)
        assert np.all(c["gpu_done"][~inside] == 0) and np.all(c["cpu_done"][~inside] == 0), (kernel, s)
        g, h = inside & (f < s), inside & (f >= s)
        assert np.all(c["gpu_done"][g] == c["gpu_frags"][g]) and np.all(c["gpu_frags"][g] > 0), (kernel, s)
        assert np.all(c["cpu_done"][g] == 0) and np.all(c["gpu_done"][h] == 0) and np.all(c["cpu_done"][h] == 1), (kernel, s)
        for b in bufs:
            b.release()
