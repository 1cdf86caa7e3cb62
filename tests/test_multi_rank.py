"""Multi-rank slice + all-gather glue on CPU (gloo, world size 2 and 3).

Each rank takes its task-aligned work-group slice from fcl_slice_range (host-only C-ABI),
computes that slice (here with the oracle, standing in for the per-rank FluidiCL run, which
needs a GPU), and the slices are all-gathered; the concatenation must equal the single-device
result bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import workloads as W


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, kernel, n0, n1, integer, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    sys.path.insert(0, os.path.join(root, "tests"))
    import torch
    import torch.distributed as dist
    import oracle
    from _util import to_oracle
    from paper_conf_cgo_panditg14_b200 import multigpu
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        P = W.make(kernel, n0, n1, integer=integer, seed=7, out_init="zero")
        name = f"{kernel}_{'i32' if integer else 'f32'}"
        ranges = multigpu.slice_ranges(name, P.gws, P.lws, world)
        lo, hi = ranges[rank]
        L = to_oracle(oracle, P)
        oracle.run_range(L, lo, hi)
        out = L.bufs[P.out_indices[0]].reshape(P.n0, -1) if len(P.gws) == 2 else L.bufs[P.out_indices[0]].reshape(-1, 1)
        nrows = out.shape[0]
        spans = [multigpu.row_span(a, b, P.gws, P.lws, nrows) for a, b in ranges]
        r0, r1 = spans[rank]
        local = torch.from_numpy(np.ascontiguousarray(out[r0:r1]))
        full = multigpu.gather_slices(local, [b - a for a, b in spans])
        if rank == 0:
            R = oracle.run(to_oracle(oracle, P)).bufs[P.out_indices[0]].reshape(full.shape)
            q.put(bool(np.array_equal(full.numpy().view(np.uint8), R.view(np.uint8))) and
                  spans[0][0] == 0 and spans[-1][1] == nrows)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("kernel,n0,n1,integer", [("conv2d", 70, 130, False), ("gesummv", 600, 600, True),
                                                   ("syrk", 300, 40, True)])
def test_slices_allgather_gloo(world, kernel, n0, n1, integer):
    from paper_conf_cgo_panditg14_b200 import _build
    _build.build()
    import oracle
    oracle.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kernel, n0, n1, integer, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    assert q.get(timeout=5) is True
