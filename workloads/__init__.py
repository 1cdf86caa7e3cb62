"""Seeded synthetic inputs and launch geometry for the FluidiCL workloads.

This module is shared by the tests, ``bench.py``, the oracle side and the CUDA
side; it holds NONE of the method's arithmetic -- only random number
generation (numpy PCG64 via ``default_rng``), shapes and the NDRange geometry
of each benchmark kernel (PolyBench/GPU launch shapes, reconstructed in
SURVEY.md §0 from the paper's Table 2, PAPER.md L22.s36).

Recipe: float inputs are U[0,1) fp32 (ATAX's x is U[-1,1));
integer instantiations draw from the integers in [-8, 8]; OUT/INOUT buffers
start either zero or as a random "poison" pattern, so a merge bug that keeps
a stale word is visible.  Scalars: alpha = 1.5, beta = 1.2 (fp32) or
alpha = 3, beta = 2 (int32); CORR eps = 0.1 (reading R7).
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Sequence, Tuple

import numpy as np

ALPHA_F, BETA_F = np.float32(1.5), np.float32(1.2)
ALPHA_I, BETA_I = 3, 2
CORR_EPS = np.float32(0.1)

# kernel -> (buffer names, indices of OUT/INOUT buffers, indices of INOUT buffers)
SIGNATURES: Dict[str, Tuple[Tuple[str, ...], Tuple[int, ...], Tuple[int, ...]]] = {
    "atax_tmp": (("A", "x", "tmp"), (2,), ()),
    "atax_y": (("A", "tmp", "y"), (2,), ()),
    "bicg_s": (("A", "r", "s"), (2,), ()),
    "bicg_q": (("A", "p", "q"), (2,), ()),
    "gesummv": (("A", "B", "x", "tmp", "y"), (3, 4), ()),
    "syrk": (("A", "C"), (1,), (1,)),
    "syr2k": (("A", "B", "C"), (2,), (2,)),
    "corr_mean": (("data", "mean"), (1,), ()),
    "corr_std": (("data", "mean", "std"), (2,), ()),
    "corr_reduce": (("data", "mean", "std"), (0,), (0,)),
    "corr_corr": (("data", "symmat"), (1,), ()),
    "conv2d": (("A", "B"), (1,), ()),
}
FLOAT_ONLY = frozenset({"corr_mean", "corr_std", "corr_reduce", "corr_corr"})


def pad(n: int, l: int) -> int:
    return -(-int(n) // int(l)) * int(l)


@dataclass
class Problem:
    """One kernel launch's inputs and geometry (no arithmetic)."""
    kernel: str
    integer: bool
    n0: int                 # rows of the row-major input matrix (SYRK: N)
    n1: int                 # columns (SYRK: M)
    gws: Tuple[int, ...]
    lws: Tuple[int, ...]
    bufs: List[np.ndarray]  # fp32 or int32 host arrays in signature order
    alpha: float = float(ALPHA_F)
    beta: float = float(BETA_F)
    ialpha: int = ALPHA_I
    ibeta: int = BETA_I
    eps: float = float(CORR_EPS)
    meta: dict = field(default_factory=dict)

    @property
    def names(self):
        return SIGNATURES[self.kernel][0]

    @property
    def out_indices(self):
        return SIGNATURES[self.kernel][1]

    @property
    def inout_indices(self):
        return SIGNATURES[self.kernel][2]

    @property
    def num_groups(self) -> int:
        n = 1
        for g, l in zip(self.gws, self.lws):
            n *= -(-g // l)
        return n

    def copy(self) -> "Problem":
        return Problem(self.kernel, self.integer, self.n0, self.n1, tuple(self.gws), tuple(self.lws),
                       [b.copy() for b in self.bufs], self.alpha, self.beta, self.ialpha, self.ibeta,
                       self.eps, dict(self.meta))


def geometry(kernel: str, n0: int, n1: int, lws1d: int = 256, lws2d=(32, 8)):
    """PolyBench/GPU NDRange of ``kernel`` (gws padded to a multiple of lws)."""
    l0, l1 = lws2d
    if kernel in ("atax_tmp", "bicg_q", "gesummv"):
        return (pad(n0, lws1d),), (lws1d,)
    if kernel in ("atax_y", "bicg_s", "corr_mean", "corr_std", "corr_corr"):
        return (pad(n1, lws1d),), (lws1d,)
    if kernel in ("syrk", "syr2k"):
        return (pad(n0, l0), pad(n0, l1)), (l0, l1)
    if kernel in ("corr_reduce", "conv2d"):
        return (pad(n1, l0), pad(n0, l1)), (l0, l1)
    raise KeyError(kernel)


def _shapes(kernel: str, n0: int, n1: int):
    """Element counts of each buffer, in signature order."""
    return {
        "atax_tmp": [n0 * n1, n1, n0],
        "atax_y": [n0 * n1, n0, n1],
        "bicg_s": [n0 * n1, n0, n1],
        "bicg_q": [n0 * n1, n1, n0],
        "gesummv": [n0 * n0, n0 * n0, n0, n0, n0],
        "syrk": [n0 * n1, n0 * n0],
        "syr2k": [n0 * n1, n0 * n1, n0 * n0],
        "corr_mean": [n0 * n1, n1],
        "corr_std": [n0 * n1, n1, n1],
        "corr_reduce": [n0 * n1, n1, n1],
        "corr_corr": [n0 * n1, n1 * n1],
        "conv2d": [n0 * n1, n0 * n1],
    }[kernel]


def make(kernel: str, n0: int, n1: int = None, *, integer: bool = False, seed: int = 0,
         out_init: str = "poison", lws1d: int = 256, lws2d=(32, 8)) -> Problem:
    """Seeded inputs for one launch.  ``out_init`` in {"poison", "zero"} sets
    the initial contents of pure-OUT buffers (INOUT buffers are always inputs)."""
    if n1 is None:
        n1 = n0
    if integer and kernel in FLOAT_ONLY:
        raise ValueError(f"{kernel} is float-only")
    rng = np.random.default_rng(seed)
    names, outs, inouts = SIGNATURES[kernel]
    bufs = []
    for k, count in enumerate(_shapes(kernel, n0, n1)):
        pure_out = k in outs and k not in inouts
        if pure_out and out_init == "zero":
            b = np.zeros(count, np.int32 if integer else np.float32)
        elif integer:
            b = rng.integers(-8, 9, size=count, dtype=np.int32)
        else:
            b = rng.random(count, dtype=np.float32)
            if kernel == "atax_tmp" and names[k] == "x":
                b = (2.0 * b - 1.0).astype(np.float32)
            if pure_out:  # poison: distinct, recognisable non-result values
                b = (b * -1e3 - 7.0).astype(np.float32)
        bufs.append(np.ascontiguousarray(b))
    gws, lws = geometry(kernel, n0, n1, lws1d, lws2d)
    return Problem(kernel, integer, n0, n1, gws, lws, bufs)


def corr_chain_inputs(n: int, m: int, seed: int = 0) -> np.ndarray:
    """CORR data matrix (n data points x m variables), U[0,1) fp32."""
    rng = np.random.default_rng(seed)
    return rng.random(n * m, dtype=np.float32)


# The BASELINE.json configurations, as concrete launch lists.
CONFIGS = {
    "atax256": dict(desc="ATAX N=256 fp32, 16 work-groups, split-point sweep vs serial CPU oracle",
                    kernels=[("atax_tmp", 256, 256, 16), ("atax_y", 256, 256, 16)]),
    "gesummv_bicg4096": dict(desc="GESUMMV / BICG N=4096 fp32 on 1 B200 + host cores",
                             kernels=[("gesummv", 4096, 4096, 256), ("bicg_s", 4096, 4096, 256),
                                      ("bicg_q", 4096, 4096, 256)]),
    "syrk_syr2k2048": dict(desc="SYRK / SYR2K N=2048 fp32 (compute-heavy, GPU-favoured split)",
                           kernels=[("syrk", 2048, 2048, None), ("syr2k", 2048, 2048, None)]),
    "conv2d_corr": dict(desc="2DCONV 16384^2 / CORR 4096^2, per-GPU slices + NCCL all-gather",
                        kernels=[("conv2d", 16384, 16384, None), ("corr_mean", 4096, 4096, 256),
                                 ("corr_std", 4096, 4096, 256), ("corr_reduce", 4096, 4096, None),
                                 ("corr_corr", 4096, 4096, 256)]),
}


def merge_inputs(n_words: int, frac: float, structure: str = "suffix", seed: int = 0,
                 dtype=np.uint32):
    """Diff-merge microbench streams: twin ~ random,
    gpu ~ random, cpu = twin with a fraction ``frac`` of words changed
    (bit-flipped, so guaranteed != twin).  ``structure``: suffix | scatter | runs."""
    rng = np.random.default_rng(seed)
    info = np.iinfo(dtype)
    twin = rng.integers(0, info.max, size=n_words, dtype=dtype, endpoint=True)
    gpu = rng.integers(0, info.max, size=n_words, dtype=dtype, endpoint=True)
    cpu = twin.copy()
    k = int(round(frac * n_words))
    if k > 0:
        if structure == "suffix":
            idx = np.arange(n_words - k, n_words)
        elif structure == "scatter":
            idx = rng.choice(n_words, size=k, replace=False)
        elif structure == "runs":
            nruns = max(1, k // 128)
            starts = rng.choice(max(1, n_words // 128), size=min(nruns, max(1, n_words // 128)),
                                replace=False) * 128
            idx = np.unique(np.concatenate([np.arange(s, min(n_words, s + 128)) for s in starts]))
        else:
            raise ValueError(structure)
        cpu[idx] = ~cpu[idx]
    return gpu, cpu, twin
