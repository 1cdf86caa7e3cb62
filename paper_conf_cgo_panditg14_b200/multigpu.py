"""Multi-GPU slicing, exchange and the sharded runner (north_star; not in the paper,
L22.s17).

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


# ------------------------------------------------------------------------------------------
# The sharded runner (BASELINE.json configs[3]): every rank runs the cooperative
# path on its own task-aligned work-group slice with its own host pool, then the output slices
# are exchanged so that every rank holds the whole output on its device.  The exchange is the
# path's one collective: all_gather_into_tensor over NCCL (NVLink) straight into the fcl
# buffers' device copies -- in place when the slices are even -- or, on the gloo backend (the
# CPU-side tests, several ranks sharing one GPU), the same gather staged through host tensors.
# ------------------------------------------------------------------------------------------
class _DevView:
    def __init__(self, ptr: int, nbytes: int, typestr: str, itemsize: int):
        self.__cuda_array_interface__ = {"shape": (nbytes // itemsize,), "typestr": typestr,
                                         "data": (int(ptr), False), "version": 3, "strides": None}


def device_tensor(buf, dtype=None):
    """A torch tensor over an fcl buffer's device copy (no copy; the buffer must outlive it)."""
    import torch
    dtype = dtype or torch.float32
    itemsize = torch.empty((), dtype=dtype).element_size()
    typestr = {torch.float32: "<f4", torch.int32: "<i4", torch.float64: "<f8", torch.int64: "<i8"}[dtype]
    return torch.as_tensor(_DevView(buf.device_ptr, buf.nbytes, typestr, itemsize), device="cuda")


def rank_world(group=None) -> Tuple[int, int]:
    """(rank, world size) of the process group, (0, 1) without one (a single GPU)."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        return dist.get_rank(group), dist.get_world_size(group)
    return 0, 1


def exchange_rows(buf, nrows: int, ncols: int, spans: Sequence[Tuple[int, int]], group=None,
                  dtype=None, mirror: bool = False):
    """All-gather the row slabs spans[r] = [r0, r1) of the row-major nrows x ncols matrix held by
    `buf` (rank r computed rows spans[r]); afterwards every rank's device copy holds all of them.
    mirror: the matrix is CORR's symmat, whose slices are L-shaped (a work-group writes its row
    right of the diagonal and its column below it): only the upper triangle of the gathered row
    slabs is trusted, and fcl_mirror_upper rebuilds the lower one on the device."""
    import torch
    import torch.distributed as dist
    rank, world = rank_world(group)
    t = device_tensor(buf, dtype)[: nrows * ncols].view(nrows, ncols)
    counts = [b - a for a, b in spans]
    stream = torch.cuda.current_stream()
    # (with a process group the collective runs even for one rank: the same NCCL path)
    if world > 1 or (dist.is_available() and dist.is_initialized()):
        r0, r1 = spans[rank]
        contiguous = spans[0][0] == 0 and all(spans[k][1] == spans[k + 1][0] for k in range(world - 1))
        if dist.get_backend(group) == "nccl":
            if contiguous and len(set(counts)) == 1:
                # in place: rank r's slab already sits at offset r * count of the output
                dist.all_gather_into_tensor(t[: spans[-1][1]], t[r0:r1], group=group)
            else:
                full = gather_slices(t[r0:r1], counts, group)
                t[spans[0][0]: spans[0][0] + full.shape[0]].copy_(full)
        else:
            full = gather_slices(t[r0:r1].cpu(), counts, group)
            t[spans[0][0]: spans[0][0] + full.shape[0]].copy_(full.to(t.device, non_blocking=False))
    if mirror:
        fcl.mirror_upper(t.data_ptr(), nrows, t.element_size(), stream.cuda_stream)
    # (the legacy default stream has handle 0, which the C-ABI reads as "the context's main
    # stream": pass cudaStreamLegacy, 0x1, so that main is ordered after the writes)
    buf.device_written(0, nrows * ncols * t.element_size(), stream.cuda_stream or 1)


def run_slice(ctx, kernel: str, gws, lws, args, rank: int, world: int, **opts) -> Tuple[int, int]:
    """Launch this rank's work-group slice of `kernel` (cooperative by default) and wait for it."""
    lo, hi = ctx.slice_range(kernel, gws, lws, rank, world)
    ctx.enqueue_ndrange(kernel, gws, lws, args, wg_lo=lo, wg_hi=hi, **opts)
    ctx.finish()
    return lo, hi


def _spans(kernel: str, gws, lws, nrows: int, world: int):
    return [row_span(lo, hi, gws, lws, nrows) for lo, hi in slice_ranges(kernel, gws, lws, world)]


def conv2d_sharded(ctx, A, B, ni: int, nj: int, gws, lws, group=None, integer: bool = False, **opts):
    """2DCONV (PolyBench/GPU) over ranks: row slabs of B, then the all-gather of B."""
    rank, world = rank_world(group)
    name = f"conv2d_{'i32' if integer else 'f32'}"
    run_slice(ctx, name, gws, lws, [A, B, ni, nj], rank, world, **opts)
    import torch
    exchange_rows(B, ni, nj, _spans(name, gws, lws, ni, world), group, torch.int32 if integer else torch.float32)


def corr_sharded(ctx, data, mean, std, symmat, n: int, m: int, gws1, lws1, gws2, lws2, group=None,
                 eps: float = 0.1, **opts):
    """CORR's four kernels (Table 2) over ranks, each followed by the exchange of its output:
    mean and std (column slices, 16 KiB at m = 4096), the reduced data (row slabs), symmat (row
    slabs of the upper triangle + the device-side mirror)."""
    rank, world = rank_world(group)
    run_slice(ctx, "corr_mean_f32", gws1, lws1, [data, mean, n, m], rank, world, **opts)
    exchange_rows(mean, m, 1, _spans("corr_mean_f32", gws1, lws1, m, world), group)
    run_slice(ctx, "corr_std_f32", gws1, lws1, [data, mean, std, n, m, eps], rank, world, **opts)
    exchange_rows(std, m, 1, _spans("corr_std_f32", gws1, lws1, m, world), group)
    run_slice(ctx, "corr_reduce_f32", gws2, lws2, [data, mean, std, n, m], rank, world, **opts)
    exchange_rows(data, n, m, _spans("corr_reduce_f32", gws2, lws2, n, world), group)
    run_slice(ctx, "corr_corr_f32", gws1, lws1, [data, symmat, n, m], rank, world, **opts)
    exchange_rows(symmat, m, m, _spans("corr_corr_f32", gws1, lws1, m, world), group, mirror=True)
