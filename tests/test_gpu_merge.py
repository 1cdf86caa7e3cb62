"""The Fig 9 diff-merge kernel (fcl_merge_raw) against the oracle merge, bit for bit."""
import numpy as np
import pytest

import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


def _dev(a: np.ndarray):
    return torch.from_numpy(a.view(np.uint8).copy()).cuda()


def _merge_gpu(gpu, cpu, twin, es, off=0, n=None):
    g, c, t = _dev(gpu), _dev(cpu), _dev(twin)
    nbytes = g.numel() - off if n is None else n
    fcl.merge_raw(g.data_ptr() + off, c.data_ptr() + off, t.data_ptr() + off, nbytes, es,
                  torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    return g.cpu().numpy()


@pytest.mark.parametrize("dtype", [np.uint8, np.uint16, np.uint32, np.uint64])
@pytest.mark.parametrize("frac", [0.0, 1e-3, 0.1, 0.5, 1.0])
@pytest.mark.parametrize("structure", ["suffix", "scatter", "runs"])
def test_merge_vs_oracle(oracle_mod, dtype, frac, structure):
    n = 100_003
    gpu, cpu, twin = W.merge_inputs(n, frac, structure, seed=11, dtype=dtype)
    es = np.dtype(dtype).itemsize
    got = _merge_gpu(gpu, cpu, twin, es)
    ref = oracle_mod.merge(gpu, cpu, twin, es)
    np.testing.assert_array_equal(got, ref.view(np.uint8))


@pytest.mark.parametrize("es", [1, 2, 4, 8])
@pytest.mark.parametrize("off_elems", [0, 1, 3])
def test_merge_unaligned_head_and_tail(oracle_mod, es, off_elems):
    dtype = {1: np.uint8, 2: np.uint16, 4: np.uint32, 8: np.uint64}[es]
    n = 4133
    gpu, cpu, twin = W.merge_inputs(n, 0.3, "scatter", seed=12, dtype=dtype)
    off = off_elems * es
    count = (n - 2 * off_elems) * es
    got = _merge_gpu(gpu, cpu, twin, es, off=off, n=count)
    ref = gpu.copy()
    sl = slice(off_elems, n - off_elems)
    ref[sl] = oracle_mod.merge(gpu[sl], cpu[sl], twin[sl], es)
    np.testing.assert_array_equal(got, ref.view(np.uint8))


def test_merge_large_sampled(oracle_mod):
    """1 GiB per stream (beyond L2): checked on sampled windows and by counts."""
    n = (1 << 30) // 4
    g = torch.randint(0, 2**31 - 1, (n,), dtype=torch.int32, device="cuda")
    t = torch.randint(0, 2**31 - 1, (n,), dtype=torch.int32, device="cuda")
    c = t.clone()
    idx = torch.randperm(n, device="cuda")[: n // 10]
    c[idx] = c[idx] ^ 1
    g0 = g.clone()
    fcl.merge_raw(g.data_ptr(), c.data_ptr(), t.data_ptr(), n * 4, 4, torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    rng = np.random.default_rng(0)
    for start in rng.integers(0, n - 65536, 8):
        sl = slice(int(start), int(start) + 65536)
        ref = oracle_mod.merge(g0[sl].cpu().numpy().view(np.uint32), c[sl].cpu().numpy().view(np.uint32),
                               t[sl].cpu().numpy().view(np.uint32), 4)
        np.testing.assert_array_equal(g[sl].cpu().numpy().view(np.uint32), ref)
    # property at full size: changed words equal cpu, others keep gpu
    changed = c != t
    assert bool(torch.equal(g[changed], c[changed]))
    assert bool(torch.equal(g[~changed], g0[~changed]))
