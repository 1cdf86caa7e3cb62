"""The sharded multi-rank path (BASELINE configs[3]) through the product: two ranks on
the one GPU of the test box (each its own process, fcl context and host pool), gloo for the
exchange (NCCL needs one GPU per rank; the runner stages the same all-gather through host
tensors on gloo).  Every rank runs the cooperative path on its slice, the outputs are exchanged,
and each rank's host and device copies must equal the single-rank GPU-only result bit for bit:
2DCONV (row slabs) and the whole CORR chain (mean / std column slices, reduced-data row slabs,
symmat's L-shaped slices combined by the upper-triangle gather + device mirror).
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, mode, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    sys.path.insert(0, os.path.join(root, "tests"))
    os.environ.setdefault("FCL_SELECT", "0")
    import torch
    import torch.distributed as dist
    import fcl_harness as H
    import workloads as W
    from paper_conf_cgo_panditg14_b200 import fcl, multigpu
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    msgs = []
    try:
        torch.cuda.set_device(0)
        cores = sorted(os.sched_getaffinity(0))
        per = max(3, len(cores) // world)
        os.sched_setaffinity(0, cores[rank * per:(rank + 1) * per] or cores)
        ctx = fcl.Context(0, n_host_threads=max(1, per - 2))
        # ---- 2DCONV
        P = W.make("conv2d", 700, 1000, seed=80, out_init="zero")
        ref, _ = H.run(ctx, P, mode="gpu")
        A, B = H.create_buffers(ctx, P)
        multigpu.conv2d_sharded(ctx, A, B, P.n0, P.n1, P.gws, P.lws, mode=mode)
        got_h = B.read_array(np.float32)
        got_d = H.device_array(B, np.float32)
        msgs.append(("conv2d host", bool(np.array_equal(got_h.view(np.uint32), ref[1].view(np.uint32)))))
        msgs.append(("conv2d device", bool(np.array_equal(got_d.view(np.uint32), ref[1].view(np.uint32)))))
        # ---- CORR chain: 4 kernels, 3 kinds of exchange
        n, m = 300, 420
        data = W.corr_chain_inputs(n, m, seed=81)
        gws1, lws1 = W.geometry("corr_mean", n, m, lws1d=32)
        gws2, lws2 = W.geometry("corr_reduce", n, m)
        init_sym = np.full(m * m, -3.0, np.float32)

        def chain(sharded, md):
            bl = [ctx.buffer_from_array(x) for x in (data, np.zeros(m, np.float32), np.zeros(m, np.float32), init_sym)]
            d, mean, std, sym = bl
            if sharded:
                multigpu.corr_sharded(ctx, d, mean, std, sym, n, m, gws1, lws1, gws2, lws2, mode=md)
            else:
                ctx.enqueue_ndrange("corr_mean_f32", gws1, lws1, [d, mean, n, m], mode=md)
                ctx.enqueue_ndrange("corr_std_f32", gws1, lws1, [d, mean, std, n, m, 0.1], mode=md)
                ctx.enqueue_ndrange("corr_reduce_f32", gws2, lws2, [d, mean, std, n, m], mode=md)
                ctx.enqueue_ndrange("corr_corr_f32", gws1, lws1, [d, sym, n, m], mode=md)
                ctx.finish()
            out = [b.read_array(np.float32) for b in bl] + [H.device_array(b, np.float32) for b in bl]
            for b in bl:
                b.release()
            return out

        want = chain(False, "gpu")
        got = chain(True, mode)
        for k, name in enumerate(["data", "mean", "std", "symmat"] * 2):
            where = "host" if k < 4 else "device"
            msgs.append((f"corr {name} {where}", bool(np.array_equal(got[k].view(np.uint32), want[k].view(np.uint32)))))
        ctx.release()
    except Exception as e:   # reported through the queue
        msgs.append((f"exception {type(e).__name__}: {e}", False))
    finally:
        q.put((rank, msgs))
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["coop", "gpu"])
def test_sharded_conv2d_and_corr_two_ranks(mode):
    from paper_conf_cgo_panditg14_b200 import _build
    _build.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    world = 2
    procs = [ctx.Process(target=_worker, args=(r, world, port, mode, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(60)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    bad = [(r, m) for r, msgs in results for m, ok in msgs if not ok]
    assert not bad, bad
    assert all(len(msgs) == 10 for _, msgs in results), results


def test_mirror_upper_and_device_written():
    """The exchange's building blocks: fcl_mirror_upper copies the upper triangle onto the lower
    one (ragged n, both element sizes), leaving the diagonal and the upper triangle untouched;
    fcl_buffer_device_written makes a device-side update the authoritative copy -- a read and a
    cooperative launch whose host side reads the buffer both see it."""
    import torch
    import fcl_harness as H
    import workloads as W
    from paper_conf_cgo_panditg14_b200 import _build, fcl, multigpu
    _build.build()
    for n, dt in ((300, torch.float32), (129, torch.float64), (1, torch.float32), (64, torch.float32)):
        a = torch.randn(n, n, dtype=dt, device="cuda")
        want = torch.triu(a) + torch.triu(a, 1).T
        fcl.mirror_upper(a.data_ptr(), n, a.element_size())
        torch.cuda.synchronize()
        assert torch.equal(a, want), (n, dt)
    ctx = fcl.Context(0, n_host_threads=4)
    try:
        P = W.make("atax_tmp", 512, 512, seed=83, lws1d=64)
        A, x, tmp = H.create_buffers(ctx, P)
        x2 = (P.bufs[1] * 3.0 - 1.0).astype(np.float32)
        dev = multigpu.device_tensor(x)
        dev.copy_(torch.from_numpy(x2).cuda())
        x.device_written(0, x.nbytes, torch.cuda.current_stream().cuda_stream or 1)
        assert x.versions()[1] == 0 and x.versions()[2] > 0          # host copy stale, device current
        assert np.array_equal(x.read_array(np.float32), x2)
        x.device_written(0, x.nbytes, torch.cuda.current_stream().cuda_stream or 1)
        ref = x2.copy()
        ctx.enqueue_ndrange("atax_tmp_f32", P.gws, P.lws, [A, x, tmp, 512, 512], mode="coop", forced_split=3)
        ctx.finish()
        got = tmp.read_array(np.float32)
        A2 = P.bufs[0].reshape(512, 512).astype(np.float64)
        assert np.allclose(got, A2 @ ref.astype(np.float64), rtol=1e-5, atol=1e-4)
        for b in (A, x, tmp):
            b.release()
    finally:
        ctx.release()
