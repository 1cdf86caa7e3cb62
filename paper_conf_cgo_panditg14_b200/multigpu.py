"""Multi-GPU slicing and all-gather glue (north_star; not in the paper, L22.s17).

Each rank owns a contiguous, task-aligned flattened work-group range (``fcl_slice_range``),
runs the cooperative FluidiCL path on it with its own host-thread pool
(``opts.wg_lo / wg_hi``), and the output slices are concatenated with
``torch.distributed.all_gather_into_tensor`` (NCCL over NVLink on B200s; gloo on CPU in the
tests) when the consumer needs the whole output.  Slices can be uneven: they are padded to the
largest slice for the collective and unpadded afterwards.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

from . import fcl


def slice_ranges(kernel: str, gws: Sequence[int], lws: Sequence[int], nranks: int) -> List[Tuple[int, int]]:
    """Work-group ranges of every rank (host-only C-ABI call; no device needed)."""
    import ctypes
    lib = fcl.load()
    h = ctypes.c_void_p()
    st = lib.fcl_get_kernel(None, kernel.encode(), ctypes.byref(h))
    if st != 0:
        raise fcl.FclError(st, f"fcl_get_kernel({kernel})")
    out = []
    for r in range(nranks):
        lo, hi = ctypes.c_int64(), ctypes.c_int64()
        st = lib.fcl_slice_range(h, len(gws), fcl._sizes3(gws), fcl._sizes3(lws), r, nranks,
                                 ctypes.byref(lo), ctypes.byref(hi))
        if st != 0:
            raise fcl.FclError(st, "fcl_slice_range")
        out.append((lo.value, hi.value))
    return out


def row_span(wg_lo: int, wg_hi: int, gws: Sequence[int], lws: Sequence[int], nrows: int) -> Tuple[int, int]:
    """Output rows owned by the work-groups [wg_lo, wg_hi) of a row-major kernel (1-D: elements)."""
    if len(gws) == 1:
        return min(wg_lo * lws[0], nrows), min(wg_hi * lws[0], nrows)
    ngx = gws[0] // lws[0]
    return min((wg_lo // ngx) * lws[1], nrows), min(-(-wg_hi // ngx) * lws[1], nrows)


def gather_slices(local, counts: Sequence[int], group=None):
    """All-gather uneven leading-dimension slices of a tensor; returns the concatenation.

    ``local`` holds this rank's ``counts[rank]`` rows (any trailing shape).  The collective is
    ``all_gather_into_tensor`` on slices padded to ``max(counts)`` rows.
    """
    import torch
    import torch.distributed as dist
    # unsigned types are not supported by every backend: move the bits as the signed type
    alias = {torch.uint32: torch.int32, torch.uint16: torch.int16, torch.uint64: torch.int64}.get(local.dtype)
    if alias is not None:
        return gather_slices(local.view(alias), counts, group).view(local.dtype)
    world = dist.get_world_size(group)
    assert len(counts) == world
    mx = max(counts)
    tail = tuple(local.shape[1:])
    pad = torch.zeros((mx,) + tail, dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    out = torch.empty((world * mx,) + tail, dtype=local.dtype, device=local.device)
    dist.all_gather_into_tensor(out, pad, group=group)
    return torch.cat([out[r * mx: r * mx + counts[r]] for r in range(world)], dim=0)
