"""The C-ABI library builds, loads and exports every symbol include/fcl.h declares (CPU only).

No compute calls: on a machine without a GPU only the host-side entry points that need no
device are exercised (status strings, defaults, signatures, slicing, argument validation).
"""
import ctypes
import os
import re

import pytest

from paper_conf_cgo_panditg14_b200 import _build, fcl

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    _build.build()
    return fcl.load()


def _declared():
    with open(os.path.join(ROOT, "include", "fcl.h")) as f:
        text = f.read()
    return sorted(set(re.findall(r"^(?:fcl_status|const char \*)\s*(fcl_[a-z_0-9]+)\s*\(", text, re.M)))


def test_every_declared_symbol_is_exported(lib):
    names = _declared()
    assert len(names) >= 20
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(fcl.EXPORTED) == names


def test_status_strings_and_version(lib):
    assert lib.fcl_status_string(0) == b"FCL_SUCCESS"
    assert lib.fcl_status_string(-52) == b"FCL_INVALID_KERNEL_ARGS"
    assert lib.fcl_status_string(-1000) == b"FCL_CONTEXT_LOST"
    assert b"sm_100a" in lib.fcl_version()


def test_default_opts(lib):
    o = fcl.LaunchOpts()
    assert lib.fcl_default_launch_opts(ctypes.byref(o)) == 0
    assert (o.mode, o.forced_split, o.init_chunk_pct, o.step_pct, o.cpu_wg_split) == (0, -1, 2, 2, 1)
    assert lib.fcl_default_launch_opts(None) == -30


def test_struct_layouts_match_header(tmp_path):
    """Every field offset and struct size of the ctypes mirrors equals what the C compiler
    gives for include/fcl.h (a probe program compiled with gcc prints them)."""
    import subprocess
    structs = {"fcl_context_desc": fcl.ContextDesc, "fcl_arg": fcl.Arg,
               "fcl_launch_opts": fcl.LaunchOpts, "fcl_launch_info": fcl.LaunchInfo}
    src = ['#include <stdio.h>', '#include <stddef.h>', '#include "fcl.h"', "int main(void) {"]
    for cname, py in structs.items():
        src.append(f'printf("{cname} sizeof %zu\\n", sizeof({cname}));')
        for fname, _ in py._fields_:
            src.append(f'printf("{cname} {fname} %zu\\n", offsetof({cname}, {fname}));')
    src.append("return 0; }")
    c = tmp_path / "probe.c"
    c.write_text("\n".join(src))
    exe = tmp_path / "probe"
    inc = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include")
    subprocess.run(["gcc", "-I", inc, str(c), "-o", str(exe)], check=True)
    out = subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split("\n")
    got = {}
    for line in out:
        if line:
            cname, field, v = line.split()
            got[(cname, field)] = int(v)
    for cname, py in structs.items():
        assert got[(cname, "sizeof")] == ctypes.sizeof(py), cname
        for fname, _ in py._fields_:
            assert got[(cname, fname)] == getattr(py, fname).offset, (cname, fname)


def test_counter_names_match_header():
    """fcl.Context.counters() names the FCL_COUNT_* entries in the header's order, all of them."""
    inc = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include", "fcl.h")
    text = open(inc).read()
    idx = {m.group(1): int(m.group(2)) for m in re.finditer(r"#define FCL_COUNT_([A-Z_0-9]+)\s+(\d+)", text)}
    n = idx.pop("N")
    assert sorted(idx.values()) == list(range(n))
    names = [k.lower() for k, _ in sorted(idx.items(), key=lambda kv: kv[1])]
    assert list(fcl.Context.COUNTERS) == names


def test_kernel_table_and_signatures(lib):
    names = ["atax_tmp", "atax_y", "bicg_s", "bicg_q", "gesummv", "syrk", "syr2k", "conv2d"]
    for n in names:
        for t in ("f32", "i32"):
            h = ctypes.c_void_p()
            assert lib.fcl_get_kernel(None, f"{n}_{t}".encode(), ctypes.byref(h)) == 0
            buf = ctypes.create_string_buffer(256)
            assert lib.fcl_kernel_signature(h, buf, 256) == 0
            assert buf.value.count(b":") >= 4
    for n in ["corr_mean", "corr_std", "corr_reduce", "corr_corr"]:
        h = ctypes.c_void_p()
        assert lib.fcl_get_kernel(None, f"{n}_f32".encode(), ctypes.byref(h)) == 0
        assert lib.fcl_get_kernel(None, f"{n}_i32".encode(), ctypes.byref(h)) == -46
    h = ctypes.c_void_p()
    lib.fcl_get_kernel(None, b"gesummv_f32", ctypes.byref(h))
    buf = ctypes.create_string_buffer(256)
    lib.fcl_kernel_signature(h, buf, 256)
    assert buf.value == b"A:in B:in x:in tmp:out y:out n:i alpha:f beta:f"


def _slice(lib, name, gws, lws, r, n):
    h = ctypes.c_void_p()
    assert lib.fcl_get_kernel(None, name.encode(), ctypes.byref(h)) == 0
    lo, hi = ctypes.c_int64(), ctypes.c_int64()
    st = lib.fcl_slice_range(h, len(gws), fcl._sizes3(gws), fcl._sizes3(lws), r, n,
                             ctypes.byref(lo), ctypes.byref(hi))
    assert st == 0
    return lo.value, hi.value


@pytest.mark.parametrize("nranks", [1, 2, 3, 4, 8])
def test_slice_ranges_partition_and_align(lib, nranks):
    # 2DCONV 16384^2, lws 32x8: 512 x 2048 work-groups, tiles of 4 x 1 work-groups (128 x 8 outputs)
    gws, lws = (16384, 16384), (32, 8)
    n_wg = 512 * 2048
    prev = 0
    for r in range(nranks):
        lo, hi = _slice(lib, "conv2d_f32", gws, lws, r, nranks)
        assert lo == prev and hi >= lo
        assert lo % 512 == 0   # whole tile rows
        prev = hi
    assert prev == n_wg
    # 1-D kernels slice at any work-group
    total = 0
    for r in range(nranks):
        lo, hi = _slice(lib, "gesummv_f32", (4096 * 8,), (256,), r, nranks)
        total += hi - lo
    assert total == 128


def test_no_device_is_reported_not_crashed(lib):
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("a GPU is present")
    except Exception:
        pass
    h = ctypes.c_void_p()
    st = lib.fcl_create_context(None, ctypes.byref(h))
    assert st == -2 and not h.value   # FCL_DEVICE_NOT_AVAILABLE
    assert lib.fcl_merge_raw(None, None, None, 16, 3, None) == -30   # elem_size 3 invalid
    assert lib.fcl_merge_raw(None, None, None, 10, 4, None) == -30   # bytes % elem_size


def test_product_has_no_oracle_dependency():
    """The product package and harness never import or link the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_cgo_panditg14_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                text = open(os.path.join(dirpath, fn)).read()
                assert "import oracle" not in text and "from oracle" not in text and "liboracle" not in text, fn
    for fn in ("fcl_harness.py",):
        text = open(os.path.join(ROOT, fn)).read()
        assert "import oracle" not in text and "from oracle" not in text
