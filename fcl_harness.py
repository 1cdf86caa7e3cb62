"""Glue between ``workloads.Problem`` (seeded inputs) and the fcl C-ABI binding.

Used by tests/, bench.py and __graft_entry__.smoke(); never by the oracle.  It only
creates buffers, forwards arguments in the kernel's signature order and reads results
back -- every step of the method runs inside libfcl.so.
"""
from __future__ import annotations

from typing import Dict, List, Optional, Tuple

import numpy as np

from paper_conf_cgo_panditg14_b200 import fcl
import workloads as W


def pin_caller() -> list:
    """Pin the calling (launching) thread to the core the runtime leaves for it.

    The context pins its coordinator to the first core of the process affinity and its workers
    from the third on (csrc/runtime.cpp, Executor::start); the second is the caller's.  Left
    floating, the caller can be placed on a core where a worker spins and lose a scheduler
    quantum (~1 ms) in the middle of a launch or fcl_finish.  Returns the cores left over after
    the workers (for helper processes), possibly empty."""
    import os
    global _CALLER_CORES
    if _CALLER_CORES is None:
        _CALLER_CORES = sorted(os.sched_getaffinity(0))
    cores = _CALLER_CORES
    if len(cores) < 3:
        return []
    os.sched_setaffinity(0, {cores[1]})
    return cores


def unpin_caller() -> None:
    """Restore the affinity pin_caller() narrowed (before creating another context: the runtime
    lays its threads out over the creating thread's affinity)."""
    import os
    if _CALLER_CORES is not None:
        os.sched_setaffinity(0, set(_CALLER_CORES))


_CALLER_CORES = None


def kernel_name(P: W.Problem) -> str:
    return f"{P.kernel}_{'i32' if P.integer else 'f32'}"


def make_args(ctx: fcl.Context, P: W.Problem, bufs: List[fcl.Buffer]) -> list:
    k = ctx.kernel(kernel_name(P))
    args, nb, ni = [], 0, 0
    for pname, pkind in k.params:
        if pkind in ("in", "out", "inout"):
            args.append(bufs[nb]); nb += 1
        elif pname == "alpha":
            args.append(P.ialpha if P.integer else P.alpha)
        elif pname == "beta":
            args.append(P.ibeta if P.integer else P.beta)
        elif pname == "eps":
            args.append(P.eps)
        else:
            args.append(P.n0 if ni == 0 else P.n1); ni += 1
    return args


def create_buffers(ctx: fcl.Context, P: W.Problem) -> List[fcl.Buffer]:
    return [ctx.buffer_from_array(b) for b in P.bufs]


def run(ctx: fcl.Context, P: W.Problem, mode: str = "coop", bufs: Optional[List[fcl.Buffer]] = None,
        read_all: bool = False, **opts) -> Tuple[Dict[int, np.ndarray], dict]:
    """Launch P through the C-ABI, wait, and return ({buffer index: host array}, launch info)."""
    own = bufs is None
    if own:
        bufs = create_buffers(ctx, P)
    info = ctx.enqueue_ndrange(kernel_name(P), P.gws, P.lws, make_args(ctx, P, bufs), mode=mode, **opts)
    ctx.finish()
    info = ctx.launch_info()
    dt = np.int32 if P.integer else np.float32
    idx = range(len(P.bufs)) if read_all else P.out_indices
    outs = {k: bufs[k].read_array(dt) for k in idx}
    if own:
        for b in bufs:
            b.release()
    return outs, info


class _CudaView:
    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def device_array(buf: fcl.Buffer, dtype) -> np.ndarray:
    """Copy a buffer's DEVICE copy to a numpy array (bypassing the host mirror), via torch."""
    import torch
    dt = np.dtype(dtype)
    n = buf.nbytes // dt.itemsize
    torch.cuda.synchronize()
    t = torch.as_tensor(_CudaView(buf.device_ptr, n, dt.str), device="cuda")
    return t.clone().cpu().numpy().view(dtype)
