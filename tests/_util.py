"""Shared test helpers: oracle marshalling and the parity criteria."""
import numpy as np

import workloads as W

# fp32 tolerance (north_star: 1e-5 relative; SURVEY S19 adds an absolute floor of 1e-6 of
# the largest reference magnitude for results produced by cancellation).
RTOL, ATOL_REL = 1e-5, 1e-6


def to_oracle(o, P: W.Problem):
    """fp32 -> fp64 copies (float kernels) or uint32 views (integer kernels)."""
    if P.integer:
        bufs = [b.view(np.uint32).copy() for b in P.bufs]
    else:
        bufs = [b.astype(np.float64) for b in P.bufs]
    return o.Launch(P.kernel, P.integer, P.n0, P.n1, list(P.gws), list(P.lws), bufs,
                    alpha=P.alpha, beta=P.beta, eps=P.eps, ialpha=P.ialpha, ibeta=P.ibeta)


def assert_parity(got: np.ndarray, ref: np.ndarray, integer: bool, what: str = "", mask=None):
    """Bit-exact for integer data; |x - r| <= 1e-5 |r| + 1e-6 max|r| for fp32 vs fp64."""
    g = np.asarray(got)
    r = np.asarray(ref)
    if mask is not None:
        g, r = g[mask], r[mask]
    if integer:
        gu, ru = g.view(np.uint32), r.astype(np.uint32)
        bad = np.nonzero(gu != ru)[0]
        assert bad.size == 0, f"{what}: {bad.size} integer mismatches, first at {bad[:5]}: {gu[bad[:5]]} vs {ru[bad[:5]]}"
        return 0.0
    g64 = g.astype(np.float64)
    scale = float(np.max(np.abs(r))) if r.size else 0.0
    err = np.abs(g64 - r)
    lim = RTOL * np.abs(r) + ATOL_REL * scale
    bad = np.nonzero(~(err <= lim))[0]
    assert bad.size == 0, (f"{what}: {bad.size}/{r.size} outside tolerance; worst {bad[:5]}: "
                           f"{g64[bad[:5]]} vs {r[bad[:5]]}")
    with np.errstate(divide="ignore", invalid="ignore"):
        rel = np.where(np.abs(r) > ATOL_REL * scale, err / np.abs(r), 0.0)
    return float(rel.max()) if rel.size else 0.0


def assert_bits(a: np.ndarray, b: np.ndarray, what: str = ""):
    ua, ub = np.ascontiguousarray(a).view(np.uint32), np.ascontiguousarray(b).view(np.uint32)
    bad = np.nonzero(ua != ub)[0]
    assert bad.size == 0, f"{what}: {bad.size} words differ bitwise, first {bad[:5]}"


def oracle_outputs(o, P: W.Problem, lo=None, hi=None):
    """Oracle result R (all work-groups, or [lo, hi) on a copy) -> {out index: array}."""
    L = to_oracle(o, P)
    n = L.num_groups()
    R = L.copy()
    o.run_range(R, 0 if lo is None else lo, n if hi is None else hi)
    return {k: R.bufs[k] for k in P.out_indices}
