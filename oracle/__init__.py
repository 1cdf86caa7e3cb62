"""Serial CPU oracle for the FluidiCL hot path (Pandit & Govindarajan, CGO 2014).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package ``paper_conf_cgo_panditg14_b200`` never imports
it, and this package never imports the product: the two share no code.

The arithmetic lives in ``oracle.c`` (plain C, fp64 / uint32, ascending loops,
one function per definition, each citing PAPER.md).  This module only
marshals numpy arrays into it and writes out the paper's *models* of the
method on top of it, step by step in the paper's order:

* ``run``             -- single-device result R (all work-groups, L14.s22-23)
* ``split_model``     -- GPU runs [0, s), CPU runs [s, N), merge  (L14.s36-38,
                         L16.s5-9, L16.s28-31)
* ``overlap_model``   -- GPU runs [0, a), CPU runs [b, N), b <= a  (L16.s18)
* ``abort_model``     -- split + GPU aborts WG s part-way          (L20.s44-47)
* ``merge``           -- Fig 9 diff-merge at element granularity    (L18.s1-5)
* ``chunk_schedule``  -- the adaptive chunk-size heuristic         (L18.s23-32)
* ``flatten``/``unflatten`` -- Fig 5 flattened work-group ids      (L14.s24-31)

Parity status: every function here is pinned by ``tests/test_oracle_*.py``
against values the paper prints, closed forms, library routines or brute
force.  Nothing is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

# kernel name -> (id, n_buffers, indices of OUT/INOUT buffers, work_dim)
KERNELS: Dict[str, tuple] = {
    "atax_tmp": (0, 3, (2,), 1),
    "atax_y": (1, 3, (2,), 1),
    "bicg_s": (2, 3, (2,), 1),
    "bicg_q": (3, 3, (2,), 1),
    "gesummv": (4, 5, (3, 4), 1),
    "syrk": (5, 2, (1,), 2),
    "syr2k": (6, 3, (2,), 2),
    "corr_mean": (7, 2, (1,), 1),
    "corr_std": (8, 3, (2,), 1),
    "corr_reduce": (9, 3, (0,), 2),
    "corr_corr": (10, 2, (1,), 1),
    "conv2d": (11, 2, (1,), 2),
}
FLOAT_ONLY = {"corr_mean", "corr_std", "corr_reduce", "corr_corr"}


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (no fast-math, no contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-ffp-contract=off",
               "-fno-fast-math", "-o", _LIB, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_exec_wg_partial.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64]
        lib.oracle_run_range.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int32]
        lib.oracle_num_groups.argtypes = [ctypes.c_void_p]
        lib.oracle_num_groups.restype = ctypes.c_int64
        lib.oracle_merge.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                     ctypes.c_int64, ctypes.c_int32]
        lib.oracle_chunk_schedule.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                                              ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64,
                                              ctypes.c_void_p, ctypes.c_int64]
        lib.oracle_chunk_schedule.restype = ctypes.c_int64
        lib.oracle_flatten.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p]
        lib.oracle_flatten.restype = ctypes.c_int64
        lib.oracle_unflatten.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]
        _lib = lib
    return _lib


class _CLaunch(ctypes.Structure):
    _fields_ = [
        ("kernel", ctypes.c_int32), ("dtype", ctypes.c_int32),
        ("n0", ctypes.c_int64), ("n1", ctypes.c_int64),
        ("work_dim", ctypes.c_int32),
        ("gws", ctypes.c_int64 * 3), ("lws", ctypes.c_int64 * 3),
        ("alpha", ctypes.c_double), ("beta", ctypes.c_double), ("eps", ctypes.c_double),
        ("ialpha", ctypes.c_uint32), ("ibeta", ctypes.c_uint32),
        ("buf", ctypes.c_void_p * 6), ("wcount", ctypes.c_void_p * 6),
    ]


@dataclass
class Launch:
    """One kernel launch: geometry, scalars and the oracle's buffers.

    ``bufs`` are numpy arrays in the kernel's buffer order (see oracle.c);
    float kernels take float64 arrays (fp64 copies of the fp32 inputs), integer
    kernels uint32 arrays.  Use :meth:`copy` before mutating runs.
    """
    kernel: str
    integer: bool
    n0: int
    n1: int
    gws: Sequence[int]
    lws: Sequence[int]
    bufs: List[np.ndarray]
    alpha: float = 1.5
    beta: float = 1.2
    eps: float = 0.1
    ialpha: int = 3
    ibeta: int = 2
    wcount: Optional[List[Optional[np.ndarray]]] = None
    _keep: list = field(default_factory=list, repr=False)

    @property
    def work_dim(self) -> int:
        return len(self.gws)

    @property
    def out_indices(self):
        return KERNELS[self.kernel][2]

    def copy(self, with_wcount: bool = False) -> "Launch":
        wc = None
        if with_wcount:
            wc = [np.zeros(b.size, np.uint32) if k in self.out_indices else None
                  for k, b in enumerate(self.bufs)]
        return Launch(self.kernel, self.integer, self.n0, self.n1, list(self.gws), list(self.lws),
                      [b.copy() for b in self.bufs], self.alpha, self.beta, self.eps,
                      self.ialpha, self.ibeta, wc)

    def _c(self) -> _CLaunch:
        kid, nbuf, _, wd = KERNELS[self.kernel]
        assert len(self.bufs) == nbuf, (self.kernel, len(self.bufs))
        assert self.work_dim == wd, (self.kernel, self.gws)
        if self.integer and self.kernel in FLOAT_ONLY:
            raise ValueError(f"{self.kernel} has no integer instantiation")
        want = np.uint32 if self.integer else np.float64
        c = _CLaunch()
        c.kernel, c.dtype, c.n0, c.n1, c.work_dim = kid, int(self.integer), self.n0, self.n1, wd
        for d in range(3):
            c.gws[d] = int(self.gws[d]) if d < wd else 1
            c.lws[d] = int(self.lws[d]) if d < wd else 1
        c.alpha, c.beta, c.eps = float(self.alpha), float(self.beta), float(self.eps)
        c.ialpha, c.ibeta = int(self.ialpha) & 0xFFFFFFFF, int(self.ibeta) & 0xFFFFFFFF
        for k, b in enumerate(self.bufs):
            if b.dtype != want or not b.flags.c_contiguous:
                raise TypeError(f"buffer {k} of {self.kernel} must be contiguous {want}")
            c.buf[k] = b.ctypes.data
            if self.wcount is not None and self.wcount[k] is not None:
                c.wcount[k] = self.wcount[k].ctypes.data
        return c

    def num_groups(self) -> int:
        return int(_load().oracle_num_groups(ctypes.byref(self._c())))


def num_groups_dim(gws: int, lws: int) -> int:
    return -(-int(gws) // int(lws))


def flatten(ng: Sequence[int], g: Sequence[int]) -> int:
    """Fig 5 flattened id; dimension 0 (the column) fastest (reading R2)."""
    wd = len(ng)
    a = (ctypes.c_int64 * 3)(*(list(ng) + [1] * (3 - wd)))
    b = (ctypes.c_int64 * 3)(*(list(g) + [0] * (3 - wd)))
    return int(_load().oracle_flatten(wd, a, b))


def unflatten(ng: Sequence[int], fgid: int) -> tuple:
    wd = len(ng)
    a = (ctypes.c_int64 * 3)(*(list(ng) + [1] * (3 - wd)))
    out = (ctypes.c_int64 * 3)()
    _load().oracle_unflatten(wd, a, int(fgid), out)
    return tuple(out[:wd])


def run_range(L: Launch, lo: int, hi: int, descending: bool = False) -> Launch:
    """Execute work-groups [lo, hi) of ``L`` in place (ascending or descending)."""
    c = L._c()
    _load().oracle_run_range(ctypes.byref(c), int(lo), int(hi), int(bool(descending)))
    return L


def exec_wg_partial(L: Launch, fgid: int, n_items: int) -> Launch:
    c = L._c()
    _load().oracle_exec_wg_partial(ctypes.byref(c), int(fgid), int(n_items))
    return L


def run(L: Launch, descending: bool = False) -> Launch:
    """Single-device result R: every work-group once, on a copy of L."""
    R = L.copy()
    return run_range(R, 0, R.num_groups(), descending)


def merge(gpu: np.ndarray, cpu: np.ndarray, orig: np.ndarray, elem_size: int) -> np.ndarray:
    """Fig 9 diff-merge (L18.s1-5) at ``elem_size`` granularity; returns a new array."""
    g = np.ascontiguousarray(gpu).copy()
    c = np.ascontiguousarray(cpu)
    o = np.ascontiguousarray(orig)
    assert g.nbytes == c.nbytes == o.nbytes
    _load().oracle_merge(g.ctypes.data, c.ctypes.data, o.ctypes.data, g.nbytes, int(elem_size))
    return g


def chunk_schedule(n_wg: int, min_units: int = 1, init_pct: int = 2, step_pct: int = 2,
                   times: Optional[Sequence[float]] = None, max_chunks: int = 1 << 20) -> List[int]:
    """C11 adaptive chunk sizes (L18.s23-32, L26.s27-28) for a given timing sequence."""
    t = np.ascontiguousarray(np.asarray(times if times is not None else [], np.float64))
    out = np.zeros(max(1, min(max_chunks, n_wg + 1)), np.int64)
    k = _load().oracle_chunk_schedule(int(n_wg), int(min_units), int(init_pct), int(step_pct),
                                      t.ctypes.data if t.size else None, int(t.size),
                                      out.ctypes.data, int(out.size))
    return [int(v) for v in out[:k]]


def _merge_outputs(G: Launch, C: Launch, T: Launch) -> Launch:
    M = G.copy()
    for k in G.out_indices:
        es = G.bufs[k].itemsize
        M.bufs[k] = merge(G.bufs[k], C.bufs[k], T.bufs[k], es).view(G.bufs[k].dtype)
    return M


def split_model(L: Launch, s: int, track_writes: bool = False):
    """T = orig; G runs [0, s); C runs [s, N); M = merge(G, C, T).

    Returns (M, G, C).  With ``track_writes`` the write counters of G and C are
    populated so the caller can assert exactly-once writes.
    """
    n = L.num_groups()
    assert 0 <= s <= n
    T = L.copy()
    G = L.copy(with_wcount=track_writes)
    C = L.copy(with_wcount=track_writes)
    run_range(G, 0, s)                       # GPU: ascending from the bottom (L14.s38)
    run_range(C, s, n, descending=True)      # CPU: descending from the top  (L14.s36)
    return _merge_outputs(G, C, T), G, C


def overlap_model(L: Launch, a: int, b: int) -> Launch:
    """Both devices run the overlap [b, a) (the race of L16.s18); b <= a."""
    n = L.num_groups()
    assert 0 <= b <= a <= n
    T = L.copy()
    G = run_range(L.copy(), 0, a)
    C = run_range(L.copy(), b, n, descending=True)
    return _merge_outputs(G, C, T)


def abort_model(L: Launch, s: int, n_items: int) -> Launch:
    """Split at s, and the GPU additionally starts WG s and aborts it after
    ``n_items`` work-items have stored (L20.s44-47; write-once makes every
    stored word final)."""
    n = L.num_groups()
    T = L.copy()
    G = run_range(L.copy(), 0, s)
    if s < n:
        exec_wg_partial(G, s, n_items)
    C = run_range(L.copy(), s, n, descending=True)
    return _merge_outputs(G, C, T)
