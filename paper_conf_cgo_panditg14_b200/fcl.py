"""Thin Python binding of the FluidiCL C-ABI (include/fcl.h) -- argument marshalling only.

Every step of the hot path runs in libfcl.so (sm_100a kernels + the native host runtime);
this module only converts Python values to the C structs and back.  PyTorch is used, when
given, purely as plumbing: device memory, pinned host memory and streams.

The library must exist in-tree (``paper_conf_cgo_panditg14_b200/libfcl.so``, built by
``__graft_entry__.build()``); there is deliberately no fallback of any kind -- a missing or
unloadable library raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import Dict, Iterable, List, Optional, Sequence

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libfcl.so")

# ---- constants (mirror include/fcl.h) ----
SUCCESS = 0
MEM_READ_WRITE, MEM_WRITE_ONLY, MEM_READ_ONLY = 1, 2, 4
MEM_USE_HOST_PTR, MEM_USE_DEVICE_PTR = 8, 16
ARG_BUFFER, ARG_INT, ARG_FLOAT = 0, 1, 2
ACCESS_IN, ACCESS_OUT, ACCESS_INOUT = 1, 2, 3
MODE_COOP, MODE_GPU_ONLY, MODE_CPU_ONLY = 0, 1, 2
STATUS_DEVICE, STATUS_HOST_MAPPED = 0, 1
LAUNCH_TIMING = 1
MODES = {"coop": MODE_COOP, "gpu": MODE_GPU_ONLY, "gpu_only": MODE_GPU_ONLY,
         "cpu": MODE_CPU_ONLY, "cpu_only": MODE_CPU_ONLY}

# Every entry point include/fcl.h declares (checked by tests/test_abi.py).
EXPORTED = [
    "fcl_create_context", "fcl_release_context", "fcl_create_buffer", "fcl_create_buffer_ext",
    "fcl_release_buffer", "fcl_write_buffer", "fcl_read_buffer", "fcl_buffer_info",
    "fcl_get_kernel", "fcl_kernel_signature", "fcl_kernel_host_variants", "fcl_default_launch_opts",
    "fcl_enqueue_ndrange",
    "fcl_merge", "fcl_merge_raw", "fcl_finish", "fcl_get_launch_info", "fcl_get_counters", "fcl_slice_range",
    "fcl_get_exec_counts", "fcl_buffer_device_written", "fcl_mirror_upper", "fcl_buffer_versions",
    "fcl_status_string", "fcl_last_error", "fcl_version",
]


DEV_ALLOC = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)
DEV_FREE = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p)


class ContextDesc(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("n_host_threads", ctypes.c_int32),
                ("pin_threads", ctypes.c_int32), ("status_location", ctypes.c_int32),
                ("main_stream", ctypes.c_void_p), ("hd_stream", ctypes.c_void_p),
                ("dh_stream", ctypes.c_void_p), ("dev_alloc", DEV_ALLOC), ("dev_free", DEV_FREE),
                ("alloc_user", ctypes.c_void_p)]


class Arg(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("access", ctypes.c_int32), ("buffer", ctypes.c_void_p),
                ("i", ctypes.c_int64), ("f", ctypes.c_double)]


class LaunchOpts(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("forced_split", ctypes.c_int64),
                ("init_chunk_pct", ctypes.c_int32), ("step_pct", ctypes.c_int32),
                ("cpu_wg_split", ctypes.c_int32), ("abort_period", ctypes.c_int32),
                ("defer_merge", ctypes.c_int32), ("n_host_threads", ctypes.c_int32),
                ("host_delay_us", ctypes.c_int32), ("drop_publish", ctypes.c_int32),
                ("wg_lo", ctypes.c_int64), ("wg_hi", ctypes.c_int64),
                ("blocking", ctypes.c_int32), ("flags", ctypes.c_int32), ("host_variant", ctypes.c_int32),
                ("select", ctypes.c_int32), ("gpu_delay_us", ctypes.c_int32),
                ("record_exec_counts", ctypes.c_int32)]


class LaunchInfo(ctypes.Structure):
    _fields_ = [("n_wg", ctypes.c_int64), ("wg_lo", ctypes.c_int64), ("wg_hi", ctypes.c_int64),
                ("gpu_watermark", ctypes.c_int64), ("published_watermark", ctypes.c_int64),
                ("gpu_tasks", ctypes.c_int64), ("gpu_tasks_total", ctypes.c_int64),
                ("cpu_wgs", ctypes.c_int64), ("n_chunks", ctypes.c_int32),
                ("cpu_did_all", ctypes.c_int32), ("merged", ctypes.c_int32),
                ("gpu_launches", ctypes.c_int32), ("merge_bytes", ctypes.c_int64),
                ("h2d_bytes", ctypes.c_int64), ("d2h_bytes", ctypes.c_int64),
                ("t_call_ms", ctypes.c_double), ("t_gpu_kernel_ms", ctypes.c_double),
                ("t_merge_ms", ctypes.c_double), ("t_host_ms", ctypes.c_double),
                ("chunk_sizes", ctypes.c_int32 * 64), ("gpu_path", ctypes.c_int32), ("race", ctypes.c_int32),
                ("host_variant", ctypes.c_int32), ("n_host_variants", ctypes.c_int32),
                ("profile_ms_per_wg", ctypes.c_double * 4), ("selected", ctypes.c_int32), ("probe", ctypes.c_int32),
                ("streamed_wgs", ctypes.c_int64), ("chunk_ms", ctypes.c_double * 64),
                ("n_c11_chunks", ctypes.c_int32), ("seq_host", ctypes.c_int32)]

    def as_dict(self) -> dict:
        d = {k: getattr(self, k) for k, _ in self._fields_ if k not in ("chunk_sizes", "profile_ms_per_wg", "chunk_ms")}
        d["chunk_sizes"] = [int(v) for v in self.chunk_sizes[: min(64, max(0, self.n_chunks))]]
        d["chunk_ms"] = [float(v) for v in self.chunk_ms[: min(64, max(0, self.n_chunks))]]
        d["profile_ms_per_wg"] = [float(v) for v in self.profile_ms_per_wg[: max(0, self.n_host_variants)]]
        return d


_lib = None


def load() -> ctypes.CDLL:
    """Load libfcl.so (raises if it is missing -- no fallback path exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: run __graft_entry__.build() first")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i32, i64, sz = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_size_t
    sig = {
        "fcl_create_context": ([ctypes.POINTER(ContextDesc), ctypes.POINTER(vp)], i32),
        "fcl_release_context": ([vp], i32),
        "fcl_create_buffer": ([vp, ctypes.c_uint32, sz, ctypes.c_uint32, vp, ctypes.POINTER(vp)], i32),
        "fcl_create_buffer_ext": ([vp, ctypes.c_uint32, sz, ctypes.c_uint32, vp, vp, ctypes.POINTER(vp)], i32),
        "fcl_release_buffer": ([vp], i32),
        "fcl_write_buffer": ([vp, vp, sz, sz, vp, i32], i32),
        "fcl_read_buffer": ([vp, vp, sz, sz, vp, i32], i32),
        "fcl_buffer_info": ([vp, ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(sz),
                             ctypes.POINTER(ctypes.c_uint32)], i32),
        "fcl_get_kernel": ([vp, ctypes.c_char_p, ctypes.POINTER(vp)], i32),
        "fcl_kernel_signature": ([vp, ctypes.c_char_p, sz], i32),
        "fcl_kernel_host_variants": ([vp, ctypes.POINTER(i32), ctypes.POINTER(ctypes.c_char_p), i32], i32),
        "fcl_default_launch_opts": ([ctypes.POINTER(LaunchOpts)], i32),
        "fcl_enqueue_ndrange": ([vp, vp, ctypes.c_uint32, ctypes.POINTER(sz), ctypes.POINTER(sz),
                                 ctypes.POINTER(Arg), ctypes.c_uint32, ctypes.POINTER(LaunchOpts),
                                 ctypes.POINTER(LaunchInfo)], i32),
        "fcl_merge": ([vp, vp], i32),
        "fcl_merge_raw": ([vp, vp, vp, sz, ctypes.c_uint32, vp], i32),
        "fcl_finish": ([vp], i32),
        "fcl_get_launch_info": ([vp, ctypes.POINTER(LaunchInfo)], i32),
        "fcl_get_counters": ([vp, ctypes.POINTER(i64), i32], i32),
        "fcl_get_exec_counts": ([vp, i64, vp, vp, vp], i32),
        "fcl_buffer_device_written": ([vp, vp, sz, sz, vp], i32),
        "fcl_mirror_upper": ([vp, sz, ctypes.c_uint32, vp], i32),
        "fcl_buffer_versions": ([vp, ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64),
                                 ctypes.POINTER(ctypes.c_uint64)], i32),
        "fcl_slice_range": ([vp, ctypes.c_uint32, ctypes.POINTER(sz), ctypes.POINTER(sz), i32, i32,
                             ctypes.POINTER(i64), ctypes.POINTER(i64)], i32),
        "fcl_status_string": ([i32], ctypes.c_char_p),
        "fcl_last_error": ([vp], ctypes.c_char_p),
        "fcl_version": ([], ctypes.c_char_p),
    }
    for name, (argt, rest) in sig.items():
        f = getattr(lib, name)
        f.argtypes = argt
        f.restype = rest
    _lib = lib
    return lib


class FclError(RuntimeError):
    def __init__(self, status: int, what: str, detail: str = ""):
        self.status = status
        name = load().fcl_status_string(status).decode()
        super().__init__(f"{what}: {name} ({status}) {detail}".rstrip())


def _check(status: int, what: str, ctx: Optional[int] = None):
    if status != SUCCESS:
        detail = load().fcl_last_error(ctx).decode() if ctx else ""
        raise FclError(status, what, detail)


def version() -> str:
    return load().fcl_version().decode()


def _sizes3(v: Sequence[int]):
    a = (ctypes.c_size_t * 3)(1, 1, 1)
    for k, x in enumerate(v):
        a[k] = int(x)
    return a


class Buffer:
    """A dual-resident buffer (host mirror + device copy)."""

    def __init__(self, ctx: "Context", handle: int, nbytes: int, elem_size: int, keep=()):
        self.ctx, self.handle, self.nbytes, self.elem_size = ctx, handle, nbytes, elem_size
        self._keep = list(keep)   # torch tensors backing caller-owned memory

    def info(self):
        h, d = ctypes.c_void_p(), ctypes.c_void_p()
        n, e = ctypes.c_size_t(), ctypes.c_uint32()
        _check(load().fcl_buffer_info(self.handle, ctypes.byref(h), ctypes.byref(d), ctypes.byref(n),
                                      ctypes.byref(e)), "fcl_buffer_info")
        return h.value, d.value, n.value, e.value

    @property
    def host_ptr(self) -> int:
        return self.info()[0]

    @property
    def device_ptr(self) -> int:
        return self.info()[1]

    def write(self, src_ptr: int, nbytes: Optional[int] = None, offset: int = 0, blocking: bool = True):
        n = self.nbytes - offset if nbytes is None else nbytes
        _check(load().fcl_write_buffer(self.ctx.handle, self.handle, offset, n, src_ptr, int(blocking)),
               "fcl_write_buffer", self.ctx.handle)

    def read(self, dst_ptr: int, nbytes: Optional[int] = None, offset: int = 0):
        n = self.nbytes - offset if nbytes is None else nbytes
        _check(load().fcl_read_buffer(self.ctx.handle, self.handle, offset, n, dst_ptr, 1),
               "fcl_read_buffer", self.ctx.handle)

    def write_array(self, arr, blocking: bool = True):
        import numpy as np
        a = np.ascontiguousarray(arr)
        assert a.nbytes == self.nbytes, (a.nbytes, self.nbytes)
        self.write(a.ctypes.data, a.nbytes, 0, blocking)

    def read_array(self, dtype, count: Optional[int] = None):
        import numpy as np
        out = np.empty(self.nbytes // np.dtype(dtype).itemsize if count is None else count, dtype)
        self.read(out.ctypes.data, out.nbytes)
        return out

    def device_written(self, offset: int = 0, nbytes: Optional[int] = None, stream: int = 0):
        """The device copy's [offset, offset+nbytes) was written outside the runtime (e.g. an
        all-gather of other ranks' slices); the host mirror is refreshed on demand."""
        n = self.nbytes - offset if nbytes is None else nbytes
        _check(load().fcl_buffer_device_written(self.ctx.handle, self.handle, int(offset), int(n), stream or None),
               "fcl_buffer_device_written", self.ctx.handle)

    def versions(self) -> tuple:
        """(expected, host, device) buffer versions (fcl_buffer_versions; 0 = that copy is stale)."""
        e, h, d = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
        _check(load().fcl_buffer_versions(self.handle, ctypes.byref(e), ctypes.byref(h), ctypes.byref(d)),
               "fcl_buffer_versions")
        return e.value, h.value, d.value

    def release(self):
        if self.handle:
            _check(load().fcl_release_buffer(self.handle), "fcl_release_buffer")
            self.handle = None


class Kernel:
    def __init__(self, ctx: "Context", name: str):
        h = ctypes.c_void_p()
        _check(load().fcl_get_kernel(ctx.handle, name.encode(), ctypes.byref(h)), f"fcl_get_kernel({name})")
        self.name, self.handle = name, h.value
        buf = ctypes.create_string_buffer(256)
        _check(load().fcl_kernel_signature(self.handle, buf, 256), "fcl_kernel_signature")
        self.signature = buf.value.decode()
        self.params = [tuple(p.split(":")) for p in self.signature.split()]
        n = ctypes.c_int32()
        names = (ctypes.c_char_p * 4)()
        _check(load().fcl_kernel_host_variants(self.handle, ctypes.byref(n), names, 4), "fcl_kernel_host_variants")
        self.host_variants = [names[v].decode() for v in range(min(4, n.value))]


def make_opts(mode="coop", forced_split=-1, init_chunk_pct=2, step_pct=2, cpu_wg_split=1,
              abort_period=0, defer_merge=0, n_host_threads=0, host_delay_us=0, drop_publish=0,
              wg_lo=0, wg_hi=-1, blocking=0, timing=0, host_variant=-1, select=0, gpu_delay_us=0,
              record_exec_counts=0) -> LaunchOpts:
    o = LaunchOpts()
    load().fcl_default_launch_opts(ctypes.byref(o))
    o.mode = MODES[mode] if isinstance(mode, str) else int(mode)
    o.forced_split = int(forced_split)
    o.init_chunk_pct, o.step_pct, o.cpu_wg_split = int(init_chunk_pct), int(step_pct), int(cpu_wg_split)
    o.abort_period, o.defer_merge, o.n_host_threads = int(abort_period), int(defer_merge), int(n_host_threads)
    o.host_delay_us, o.drop_publish = int(host_delay_us), int(drop_publish)
    o.wg_lo, o.wg_hi = int(wg_lo), int(wg_hi)
    o.blocking = int(blocking)
    o.flags = LAUNCH_TIMING if timing else 0
    o.host_variant = int(host_variant)
    o.select = int(select)
    o.gpu_delay_us, o.record_exec_counts = int(gpu_delay_us), int(record_exec_counts)
    return o


class Context:
    """A FluidiCL context on one CUDA device plus the host executor threads."""

    def __init__(self, device: int = 0, n_host_threads: int = 0, status_location: str = "device",
                 streams: Optional[Sequence[int]] = None, pin_threads: bool = True, allocator=None):
        """allocator: optional (alloc(nbytes) -> device pointer, free(pointer)) pair for buffers and
        the twin/stage pool, e.g. torch_allocator(); the callables must outlive the context."""
        d = ContextDesc()
        d.device, d.n_host_threads, d.pin_threads = int(device), int(n_host_threads), int(pin_threads)
        d.status_location = STATUS_HOST_MAPPED if status_location == "host_mapped" else STATUS_DEVICE
        if streams:
            d.main_stream, d.hd_stream, d.dh_stream = [int(s) if s else None for s in streams]
        self._alloc_cbs = None
        if allocator is not None:
            alloc, free = allocator
            self._alloc_cbs = (DEV_ALLOC(lambda n, u: int(alloc(int(n)) or 0)),
                               DEV_FREE(lambda p, u: free(int(p))))
            d.dev_alloc, d.dev_free = self._alloc_cbs
        h = ctypes.c_void_p()
        _check(load().fcl_create_context(ctypes.byref(d), ctypes.byref(h)), "fcl_create_context")
        self.handle = h.value
        self.device = device
        self._kernels: Dict[str, Kernel] = {}

    # ---- buffers
    def create_buffer(self, nbytes: int, elem_size: int = 4, host_init: Optional[int] = None,
                      flags: int = MEM_READ_WRITE) -> Buffer:
        h = ctypes.c_void_p()
        _check(load().fcl_create_buffer(self.handle, flags, int(nbytes), int(elem_size), host_init,
                                        ctypes.byref(h)), "fcl_create_buffer", self.handle)
        return Buffer(self, h.value, int(nbytes), int(elem_size))

    def buffer_from_array(self, arr) -> Buffer:
        import numpy as np
        a = np.ascontiguousarray(arr)
        return self.create_buffer(a.nbytes, a.itemsize, a.ctypes.data)

    def buffer_ext(self, nbytes: int, elem_size: int, host_ptr: Optional[int], device_ptr: Optional[int],
                   keep=()) -> Buffer:
        h = ctypes.c_void_p()
        _check(load().fcl_create_buffer_ext(self.handle, MEM_READ_WRITE, int(nbytes), int(elem_size),
                                            host_ptr, device_ptr, ctypes.byref(h)),
               "fcl_create_buffer_ext", self.handle)
        return Buffer(self, h.value, int(nbytes), int(elem_size), keep)

    def buffer_from_torch(self, host_pinned, device=None) -> Buffer:
        """Adopt a pinned host tensor (and optionally a CUDA tensor) as the two copies."""
        nbytes = host_pinned.numel() * host_pinned.element_size()
        dptr = device.data_ptr() if device is not None else None
        keep = (host_pinned,) if device is None else (host_pinned, device)
        return self.buffer_ext(nbytes, host_pinned.element_size(), host_pinned.data_ptr(), dptr, keep)

    def kernel(self, name: str) -> Kernel:
        if name not in self._kernels:
            self._kernels[name] = Kernel(self, name)
        return self._kernels[name]

    # ---- launches
    def enqueue_ndrange(self, kernel, gws: Sequence[int], lws: Sequence[int], args: Iterable,
                        opts: Optional[LaunchOpts] = None, **kw) -> dict:
        """args: Buffers, ints and floats in the kernel's signature order."""
        k = self.kernel(kernel) if isinstance(kernel, str) else kernel
        args = list(args)
        if len(args) != len(k.params):
            raise ValueError(f"{k.name} takes {k.signature}")
        arr = (Arg * len(args))()
        for n, (v, (pname, pkind)) in enumerate(zip(args, k.params)):
            if isinstance(v, Buffer):
                arr[n].kind, arr[n].buffer = ARG_BUFFER, v.handle
                arr[n].access = {"in": ACCESS_IN, "out": ACCESS_OUT, "inout": ACCESS_INOUT}[pkind]
            elif pkind == "i":
                arr[n].kind, arr[n].i = ARG_INT, int(v)
            else:
                arr[n].kind, arr[n].f = ARG_FLOAT, float(v)
        o = opts if opts is not None else make_opts(**kw)
        info = LaunchInfo()
        _check(load().fcl_enqueue_ndrange(self.handle, k.handle, len(gws), _sizes3(gws), _sizes3(lws), arr,
                                          len(args), ctypes.byref(o), ctypes.byref(info)),
               f"fcl_enqueue_ndrange({k.name})", self.handle)
        return info.as_dict()

    def prepare(self, kernel, gws: Sequence[int], lws: Sequence[int], args: Iterable, **kw) -> "PreparedLaunch":
        """Marshal a launch once; calling the result enqueues it with one C call."""
        return PreparedLaunch(self, kernel, gws, lws, args, **kw)

    def merge(self, buf: Buffer):
        _check(load().fcl_merge(self.handle, buf.handle), "fcl_merge", self.handle)

    def finish(self):
        _check(load().fcl_finish(self.handle), "fcl_finish", self.handle)

    def launch_info(self) -> dict:
        info = LaunchInfo()
        _check(load().fcl_get_launch_info(self.handle, ctypes.byref(info)), "fcl_get_launch_info", self.handle)
        return info.as_dict()

    COUNTERS = ("coop", "probe", "sel_gpu", "sel_cpu", "gpu_only", "cpu_only", "h2d_bytes", "d2h_bytes",
                "launch_drains", "seq_host", "seq_trials")

    def counters(self) -> dict:
        """Cumulative launch counters (fcl_get_counters): how COOP launches ran under device selection."""
        c = (ctypes.c_int64 * len(self.COUNTERS))()
        _check(load().fcl_get_counters(self.handle, c, len(self.COUNTERS)), "fcl_get_counters", self.handle)
        return {k: int(c[i]) for i, k in enumerate(self.COUNTERS)}

    def exec_counts(self, n_wg: int) -> dict:
        """Per-work-group execution counts of the last launch made with record_exec_counts=1
        (fcl_get_exec_counts): numpy int32 arrays gpu_done, gpu_frags, cpu_done."""
        import numpy as np
        out = {k: np.zeros(int(n_wg), np.int32) for k in ("gpu_done", "gpu_frags", "cpu_done")}
        _check(load().fcl_get_exec_counts(self.handle, int(n_wg), out["gpu_done"].ctypes.data,
                                          out["gpu_frags"].ctypes.data, out["cpu_done"].ctypes.data),
               "fcl_get_exec_counts", self.handle)
        return out

    def slice_range(self, kernel, gws, lws, rank: int, nranks: int):
        k = self.kernel(kernel) if isinstance(kernel, str) else kernel
        lo, hi = ctypes.c_int64(), ctypes.c_int64()
        _check(load().fcl_slice_range(k.handle, len(gws), _sizes3(gws), _sizes3(lws), int(rank), int(nranks),
                                      ctypes.byref(lo), ctypes.byref(hi)), "fcl_slice_range")
        return lo.value, hi.value

    def last_error(self) -> str:
        return load().fcl_last_error(self.handle).decode()

    def release(self):
        if self.handle:
            _check(load().fcl_release_context(self.handle), "fcl_release_context")
            self.handle = None


class PreparedLaunch:
    """A launch whose C structs are built once (argument marshalling off the critical path)."""

    def __init__(self, ctx: Context, kernel, gws, lws, args, **kw):
        k = ctx.kernel(kernel) if isinstance(kernel, str) else kernel
        args = list(args)
        if len(args) != len(k.params):
            raise ValueError(f"{k.name} takes {k.signature}")
        self.ctx, self.k = ctx, k
        self.arr = (Arg * len(args))()
        for n, (v, (pname, pkind)) in enumerate(zip(args, k.params)):
            if isinstance(v, Buffer):
                self.arr[n].kind, self.arr[n].buffer = ARG_BUFFER, v.handle
                self.arr[n].access = {"in": ACCESS_IN, "out": ACCESS_OUT, "inout": ACCESS_INOUT}[pkind]
            elif pkind == "i":
                self.arr[n].kind, self.arr[n].i = ARG_INT, int(v)
            else:
                self.arr[n].kind, self.arr[n].f = ARG_FLOAT, float(v)
        self.nargs = len(args)
        self.wd = len(gws)
        self.gws, self.lws = _sizes3(gws), _sizes3(lws)
        self.opts = make_opts(**kw)
        self.info = LaunchInfo()
        self._fn = load().fcl_enqueue_ndrange
        self._args = (ctx.handle, k.handle, self.wd, self.gws, self.lws, self.arr, self.nargs,
                      ctypes.byref(self.opts), ctypes.byref(self.info))

    def __call__(self):
        st = self._fn(*self._args)
        if st != SUCCESS:
            _check(st, f"fcl_enqueue_ndrange({self.k.name})", self.ctx.handle)
        return self.info


def merge_raw(gpu_ptr: int, cpu_ptr: int, twin_ptr: int, nbytes: int, elem_size: int, stream: int = 0):
    """The Fig 9 diff-merge kernel on raw device pointers (asynchronous on `stream`)."""
    _check(load().fcl_merge_raw(gpu_ptr, cpu_ptr, twin_ptr, int(nbytes), int(elem_size), stream or None),
           "fcl_merge_raw")


def mirror_upper(ptr: int, n: int, elem_size: int = 4, stream: int = 0):
    """a[j][i] = a[i][j] for i < j on an n x n row-major device matrix (asynchronous on `stream`)."""
    _check(load().fcl_mirror_upper(ptr, int(n), int(elem_size), stream or None), "fcl_mirror_upper")


def torch_allocator(device: int = 0):
    """(alloc, free) over the torch caching allocator (the context's device memory
    from the framework's allocator), for Context(allocator=...)."""
    import torch

    def alloc(n: int) -> int:
        return torch.cuda.caching_allocator_alloc(n, device)

    def free(p: int) -> None:
        torch.cuda.caching_allocator_delete(p)

    return alloc, free
