"""Brute-force pins of the cooperative-execution model.

For tiny NDRanges and EVERY split point s in [0, N_wg]: the GPU runs [0, s)
ascending, the CPU runs [s, N_wg) descending, and the Fig 9 merge of the two
against the twin equals the single-device result R bit for bit; every output
word is written by exactly one device (the "non-overlapping parts" of L16.s9).
The overlap model (both run [b, a), the race of L16.s18) and the abort model
(L20.s44-47) must give R as well.  CPU only.
"""
import numpy as np
import pytest

import workloads as W
from test_oracle_pins import to_oracle

# (kernel, n0, n1, integer, lws1d, lws2d) -- tiny launches with ragged tails
CASES = [
    ("atax_tmp", 256, 256, False, 16, None),   # config 1: 16 work-groups
    ("atax_y", 256, 256, False, 16, None),
    ("atax_tmp", 256, 256, True, 16, None),
    ("bicg_s", 37, 50, False, 8, None),
    ("bicg_q", 50, 37, True, 8, None),
    ("gesummv", 45, 45, False, 8, None),
    ("gesummv", 45, 45, True, 8, None),
    ("syrk", 32, 24, False, None, (8, 8)),
    ("syrk", 19, 7, True, None, (8, 4)),
    ("syr2k", 21, 9, False, None, (8, 8)),
    ("conv2d", 33, 40, False, None, (16, 8)),
    ("conv2d", 33, 40, True, None, (16, 8)),
    ("corr_mean", 30, 40, False, 8, None),
    ("corr_std", 30, 40, False, 8, None),
    ("corr_reduce", 30, 40, False, None, (16, 8)),
    ("corr_corr", 30, 40, False, 8, None),
]


def _launch(o, kernel, n0, n1, integer, l1, l2, seed=0):
    P = W.make(kernel, n0, n1, integer=integer, seed=seed,
               lws1d=l1 or 256, lws2d=l2 or (32, 8))
    return to_oracle(o, P)


def _eq(a, b):
    return np.array_equal(a.view(np.uint8), b.view(np.uint8))


@pytest.mark.parametrize("case", CASES, ids=lambda c: f"{c[0]}-{'i32' if c[3] else 'f'}-{c[1]}x{c[2]}")
def test_every_split_point(oracle_mod, case):
    L = _launch(oracle_mod, *case)
    n = L.num_groups()
    R = oracle_mod.run(L)
    Rd = oracle_mod.run(L, descending=True)   # WG independence (L14.s23): order-free
    for k in L.out_indices:
        assert _eq(R.bufs[k], Rd.bufs[k])
    # R writes every output word it writes exactly once
    Rw = L.copy(with_wcount=True)
    oracle_mod.run_range(Rw, 0, n)
    for s in range(n + 1):
        M, G, C = oracle_mod.split_model(L, s, track_writes=True)
        for k in L.out_indices:
            assert _eq(M.bufs[k], R.bufs[k]), (case, s, k)
            # exactly-once: each word R writes is written by exactly one device
            tot = G.wcount[k] + C.wcount[k]
            np.testing.assert_array_equal(tot, Rw.wcount[k])
            assert tot.max() <= 1


@pytest.mark.parametrize("case", [CASES[0], CASES[2], CASES[7], CASES[10], CASES[15]],
                         ids=lambda c: f"{c[0]}-{'i32' if c[3] else 'f'}")
def test_overlap_pairs(oracle_mod, case):
    """The race: both devices execute [b, a); merge still gives R (L16.s18)."""
    L = _launch(oracle_mod, *case, seed=1)
    n = L.num_groups()
    R = oracle_mod.run(L)
    step = max(1, n // 8)
    for a in range(0, n + 1, step):
        for b in range(0, a + 1, step):
            M = oracle_mod.overlap_model(L, a, b)
            for k in L.out_indices:
                assert _eq(M.bufs[k], R.bufs[k]), (case, a, b)


@pytest.mark.parametrize("case", [CASES[0], CASES[6], CASES[8], CASES[14]],
                         ids=lambda c: f"{c[0]}-{'i32' if c[3] else 'f'}")
def test_abort_model(oracle_mod, case):
    """GPU aborts WG s part-way; under write-once every stored word is final."""
    L = _launch(oracle_mod, *case, seed=2)
    n = L.num_groups()
    R = oracle_mod.run(L)
    wg_items = int(np.prod(L.lws))
    for s in range(n):
        for items in (0, 1, wg_items // 2, wg_items - 1):
            M = oracle_mod.abort_model(L, s, items)
            for k in L.out_indices:
                assert _eq(M.bufs[k], R.bufs[k]), (case, s, items)


def test_adversarial_final_equals_original(oracle_mod):
    """S13: where the CPU's final value equals the original, the merge keeps
    the GPU word.  Write-once makes that safe; an accumulate-in-place body that
    aborts leaves a partial sum and the merge would return a wrong word."""
    n = 64
    P = W.make("bicg_q", n, n, integer=True, seed=3, lws1d=8)
    A = P.bufs[0].reshape(n, n)
    A[::2, :] = 0                          # even rows: q[i] = 0 ...
    P.bufs[2][:] = 0                       # ... and the original q is 0 as well
    L = to_oracle(oracle_mod, P)
    R = oracle_mod.run(L)
    for s in range(L.num_groups() + 1):
        M, _, _ = oracle_mod.split_model(L, s)
        assert _eq(M.bufs[2], R.bufs[2])
    # a non-write-once GPU body: a partial sum stored into q before aborting
    G = L.copy()
    G.bufs[2][0] = np.uint32(12345)        # partial (non-final) value for row 0 (final = 0)
    C = oracle_mod.run(L)                   # CPU computes row 0: final 0 == original 0
    M = oracle_mod.merge(G.bufs[2], C.bufs[2], L.bufs[2], 4)
    assert M[0] != R.bufs[2][0]             # the hazard the write-once contract removes


def test_chunked_descending_schedule_covers_once(oracle_mod):
    """CPU subkernels from the top down with C11 sizes cover [s, N) once (L18.s34-36)."""
    L = _launch(oracle_mod, "syrk", 64, 16, True, None, (8, 4))
    n = L.num_groups()
    R = oracle_mod.run(L)
    sizes = oracle_mod.chunk_schedule(n, 1, 2, 2, [1.0 / (k + 1) for k in range(n)])
    C = L.copy(with_wcount=True)
    hi = n
    for sz in sizes:
        oracle_mod.run_range(C, hi - sz, hi)
        hi -= sz
    assert hi == 0
    assert _eq(C.bufs[1], R.bufs[1])
    assert C.wcount[1].max() == 1
