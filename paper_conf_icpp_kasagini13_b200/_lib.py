"""Thin ctypes binding of libperm (include/perm.h): argument marshalling only.

Every step of the permutation runs in libperm's C++ planner and sm_100a
kernels. PyTorch supplies device memory and streams (data_ptr / cuda_stream).
There is no Python or CPU fallback: if libperm.so is missing this module
raises on import.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libperm.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is not built; run `python -m paper_conf_icpp_kasagini13_b200.build` "
        "or __graft_entry__.build() (there is no CPU fallback)")

_lib = ctypes.CDLL(LIB_PATH)

PERM_OK = 0
STATUS = {0: "PERM_OK", -1: "PERM_EINVAL", -2: "PERM_ENOTPERM", -3: "PERM_EUNSUPPORTED",
          -4: "PERM_ENOMEM", -5: "PERM_ECUDA", -6: "PERM_ENCCL", -7: "PERM_ENODEVICE"}


class PermError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class PlanOptions(ctypes.Structure):
    _fields_ = [("passes", ctypes.c_int32), ("h1", ctypes.c_int32), ("h2", ctypes.c_int32),
                ("h3", ctypes.c_int32), ("layout", ctypes.c_int32), ("stages", ctypes.c_int32),
                ("fuse", ctypes.c_int32), ("no_tma", ctypes.c_int32), ("direct", ctypes.c_int32),
                ("log2c", ctypes.c_int32), ("sched_format", ctypes.c_int32), ("gpu_planner", ctypes.c_int32),
                ("cluster", ctypes.c_int32)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("rows", ctypes.c_int64), ("cols", ctypes.c_int64),
                ("sched_bytes", ctypes.c_int64), ("scratch_bytes", ctypes.c_int64),
                ("elem_bytes", ctypes.c_int32), ("passes", ctypes.c_int32),
                ("kernels_per_apply", ctypes.c_int32), ("entry_bits", ctypes.c_int32 * 3),
                ("h", ctypes.c_int32 * 3), ("planner_threads", ctypes.c_int32),
                ("build_ms_colour", ctypes.c_double), ("build_ms_bank", ctypes.c_double),
                ("build_ms_upload", ctypes.c_double), ("world", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("shard_elems", ctypes.c_int64),
                ("block_elems", ctypes.c_int64), ("distribution", ctypes.c_int64),
                ("direct", ctypes.c_int32), ("gpu_planner", ctypes.c_int32)]

    def as_dict(self) -> dict:
        d = {}
        for name, _ in self._fields_:
            v = getattr(self, name)
            d[name] = list(v) if isinstance(v, ctypes.Array) else v
        return d


_vp, _i64, _i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32


def _sig(name, res, *args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = list(args)
    return f


_plan_create = _sig("perm_plan_create", _vp, _vp, _i64, _i32)
_plan_create_ex = _sig("perm_plan_create_ex", _vp, _vp, _i64, _i32, ctypes.POINTER(PlanOptions))
_plan_create_host = _sig("perm_plan_create_host", _vp, _vp, _i64, _i32, ctypes.POINTER(PlanOptions))
_plan_create_sharded = _sig("perm_plan_create_sharded_ex", _vp, _vp, _i64, _i32, _i32, _i32, _vp,
                            ctypes.POINTER(PlanOptions))
_nccl_uid = _sig("perm_nccl_unique_id", ctypes.c_int, _vp)
_apply_sharded = _sig("perm_apply_sharded", ctypes.c_int, _vp, _vp, _vp, _vp)
_sharded_exchange = _sig("perm_sharded_exchange", ctypes.c_int, _vp, _vp, _vp, _vp)
_plan_create_sharded_host = _sig("perm_plan_create_sharded_host", _vp, _vp, _i64, _i32, _i32, _i32,
                                 ctypes.POINTER(PlanOptions))
_sharded_step = _sig("perm_sharded_step", ctypes.c_int, _vp, _i32, _vp, _vp, _vp)
_run_pass = _sig("perm_plan_run_pass", ctypes.c_int, _vp, _i32, _vp, _vp, _vp)
_plan_destroy = _sig("perm_plan_destroy", None, _vp)
_plan_get_info = _sig("perm_plan_get_info", ctypes.c_int, _vp, ctypes.POINTER(PlanInfo))
_plan_describe = _sig("perm_plan_describe", _i64, _vp, ctypes.c_char_p, _i64)
_plan_export = _sig("perm_plan_export", ctypes.c_int, _vp, _vp, _vp, _vp, _vp)
_apply = _sig("perm_apply", ctypes.c_int, _vp, _vp, _vp, _vp)
_apply_host = _sig("perm_apply_host", ctypes.c_int, _vp, _vp, _vp, _vp)
_apply_host_async = _sig("perm_apply_host_async", ctypes.c_int, _vp, _vp, _vp, _vp)
_set_prof = _sig("perm_plan_set_profiling", ctypes.c_int, _vp, ctypes.c_int)
_pass_times = _sig("perm_plan_pass_times", ctypes.c_int, _vp, ctypes.POINTER(ctypes.c_float), ctypes.c_int)
_set_tracing = _sig("perm_plan_set_tracing", ctypes.c_int, _vp, ctypes.c_int)
_trace = _sig("perm_plan_trace", _i64, _vp, _vp, _i64)
_scatter = _sig("perm_scatter_baseline", ctypes.c_int, _vp, _vp, _vp, _i64, _i32, _vp)
_gather = _sig("perm_gather_baseline", ctypes.c_int, _vp, _vp, _vp, _i64, _i32, _vp)
_copy = _sig("perm_copy_kernel", ctypes.c_int, _vp, _vp, _i64, _i32, _vp)
_last_error = _sig("perm_last_error", ctypes.c_int)
_last_error_string = _sig("perm_last_error_string", ctypes.c_char_p)
_version = _sig("perm_version", ctypes.c_char_p)


def version() -> str:
    return _version().decode()


def _raise(status: int | None = None):
    st = _last_error() if status is None else status
    raise PermError(st, _last_error_string().decode())


def _check(status: int):
    if status != PERM_OK:
        _raise(status)


def _stream_handle(stream) -> int | None:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _ptr(x) -> int:
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return int(x)


def _check_buf(x, nbytes: int, what: str):
    """Device buffers handed to libperm: CUDA, contiguous, exactly nbytes (torch tensors);
    raw integers are passed through as pointers (the caller vouches for them)."""
    if not hasattr(x, "data_ptr"):
        return
    if not getattr(x, "is_cuda", False):
        raise PermError(-1, f"{what} must be a CUDA tensor")
    if not x.is_contiguous():
        raise PermError(-1, f"{what} must be contiguous")
    got = x.numel() * x.element_size()
    if got != nbytes:
        raise PermError(-1, f"{what} holds {got} bytes, the plan needs {nbytes}")


def nccl_unique_id() -> bytes:
    """A fresh ncclUniqueId (128 bytes) for perm_plan_create_sharded (rank 0 makes it,
    every rank passes the same bytes)."""
    buf = ctypes.create_string_buffer(128)
    _check(_nccl_uid(buf))
    return buf.raw


def _as_int32_host(p) -> np.ndarray:
    if hasattr(p, "detach"):       # torch tensor
        p = p.detach().cpu().numpy()
    return np.ascontiguousarray(p, dtype=np.int32)


class Plan:
    """perm_plan: the offline schedule of permutation p (int32, host)."""

    def __init__(self, p, elem_bytes: int = 4, passes: int = 0, h=(0, 0, 0),
                 device: bool = True, layout: int = 0, stages: int = 0, fuse: int = 0,
                 world: int = 0, rank: int = 0, no_tma: int = 0, direct: int = 0, log2c: int = 0,
                 sched_format: int = 0, gpu_planner: int = 0, nccl_uid: bytes | None = None,
                 cluster: int = 0):
        """world > 0: row-sharded plan of rank `rank` (see perm_plan_create_sharded);
        nccl_uid (128 bytes, the same on every rank) also joins the plan's NCCL
        communicator, so apply_sharded() runs the whole sharded apply in libperm."""
        p = _as_int32_host(p)
        self.n = int(p.size)
        self.elem_bytes = elem_bytes
        opt = PlanOptions(passes, h[0], h[1], h[2], layout, stages, fuse, no_tma, direct, log2c,
                          sched_format, gpu_planner, cluster)
        if world > 0:
            if device:
                uid = None
                if nccl_uid is not None:
                    if len(nccl_uid) != 128:
                        raise ValueError("nccl_uid must be 128 bytes")
                    uid = ctypes.create_string_buffer(bytes(nccl_uid), 128)
                handle = _plan_create_sharded(p.ctypes.data, self.n, elem_bytes, world, rank, uid,
                                              ctypes.byref(opt))
            else:
                handle = _plan_create_sharded_host(p.ctypes.data, self.n, elem_bytes, world, rank,
                                                   ctypes.byref(opt))
        elif device:
            handle = _plan_create_ex(p.ctypes.data, self.n, elem_bytes, ctypes.byref(opt))
        else:
            handle = _plan_create_host(p.ctypes.data, self.n, elem_bytes, ctypes.byref(opt))
        if not handle:
            _raise()
        self._h = handle
        self.on_device = device
        self.world = world if world > 0 else 1
        self.nbytes = self.n * elem_bytes
        self.shard_bytes = self.nbytes // self.world

    # -- lifecycle
    def close(self):
        if getattr(self, "_h", None):
            _plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # -- introspection
    def info(self) -> dict:
        inf = PlanInfo()
        _check(_plan_get_info(self._h, ctypes.byref(inf)))
        return inf.as_dict()

    def describe(self) -> dict:
        import json
        need = _plan_describe(self._h, None, 0)
        if need < 0:
            _raise(int(need))
        buf = ctypes.create_string_buffer(int(need))
        _plan_describe(self._h, buf, need)
        return json.loads(buf.value.decode())

    def export(self):
        """(kappa[n] uint16, [sched1 (r,c), sched2 (c,r), sched3 (r,c)] uint32 (sigma<<16)|t)."""
        inf = self.info()
        r, c = inf["rows"], inf["cols"]
        G = inf["world"]
        kappa = np.empty(r * c, dtype=np.uint16)        # words (2n for 8-byte elements)
        s1 = np.empty((r // G, c), dtype=np.uint32)     # sharded plans: this rank's lines
        s2 = np.empty((c // G, r), dtype=np.uint32)
        s3 = np.empty((r // G, c), dtype=np.uint32)
        _check(_plan_export(self._h, kappa.ctypes.data, s1.ctypes.data, s2.ctypes.data,
                            s3.ctypes.data))
        return kappa, [s1, s2, s3]

    # -- hot path
    def apply(self, a, b, stream=None):
        """b[p[i]] = a[i]; a, b CUDA tensors of n * elem_bytes bytes, stream-ordered."""
        _check_buf(a, self.nbytes, "a")
        _check_buf(b, self.nbytes, "b")
        _check(_apply(self._h, _ptr(a), _ptr(b), _stream_handle(stream)))
        return b

    def apply_sharded(self, a_shard, b_shard, stream=None):
        """This rank's b shard of a sharded plan created with nccl_uid (NCCL collective:
        every rank calls it); a_shard / b_shard: n/world elements on the plan's device."""
        _check_buf(a_shard, self.shard_bytes, "a_shard")
        _check_buf(b_shard, self.shard_bytes, "b_shard")
        _check(_apply_sharded(self._h, _ptr(a_shard), _ptr(b_shard), _stream_handle(stream)))
        return b_shard

    def sharded_exchange(self, send, recv, stream=None):
        """The plan communicator's all-to-all of the perm_sharded_step block contract."""
        _check_buf(send, self.shard_bytes, "send")
        _check_buf(recv, self.shard_bytes, "recv")
        _check(_sharded_exchange(self._h, _ptr(send), _ptr(recv), _stream_handle(stream)))
        return recv

    def apply_host(self, a_host, b_host, stream=None):
        """End-to-end: host a -> device -> apply -> host b (synchronises the stream)."""
        for x, what in ((a_host, "a_host"), (b_host, "b_host")):
            nb = x.nbytes if isinstance(x, np.ndarray) else (
                x.numel() * x.element_size() if hasattr(x, "numel") else self.nbytes)
            if nb != self.nbytes or getattr(x, "is_cuda", False):
                raise PermError(-1, f"{what}: host buffer of {self.nbytes} bytes expected")
        _check(_apply_host(self._h, _ptr(a_host), _ptr(b_host), _stream_handle(stream)))
        return b_host

    def apply_host_async(self, a_host, b_host, stream=None):
        """perm_apply_host_async: enqueue H2D, apply, D2H on `stream` without synchronising.
        a_host / b_host must be pinned torch tensors (checked); b_host is valid after the
        stream is synchronised. Calls on the same plan must share one stream."""
        for x, what in ((a_host, "a_host"), (b_host, "b_host")):
            if not hasattr(x, "is_pinned") or not x.is_pinned() or \
                    x.numel() * x.element_size() != self.nbytes:
                raise PermError(-1, f"{what}: pinned host tensor of {self.nbytes} bytes expected")
        _check(_apply_host_async(self._h, _ptr(a_host), _ptr(b_host), _stream_handle(stream)))
        return b_host

    def sharded_step(self, step: int, inp, out, stream=None):
        """One local step of a row-sharded apply (see include/perm.h perm_sharded_step)."""
        _check_buf(inp, self.shard_bytes, "in")
        _check_buf(out, self.shard_bytes, "out")
        _check(_sharded_step(self._h, step, _ptr(inp), _ptr(out), _stream_handle(stream)))
        return out

    def run_pass(self, k: int, inp, out=None, stream=None):
        """Launch row pass k alone (TLC plans; see include/perm.h perm_plan_run_pass)."""
        _check(_run_pass(self._h, k, _ptr(inp) if inp is not None else None,
                         _ptr(out) if out is not None else None, _stream_handle(stream)))

    def set_profiling(self, on: bool = True):
        _check(_set_prof(self._h, 1 if on else 0))

    def set_tracing(self, on: bool = True):
        _check(_set_tracing(self._h, 1 if on else 0))

    def trace(self) -> np.ndarray:
        """[3, ctas, 16] uint64 %globaltimer stamps (ns) of the last apply (0 = not recorded)."""
        n = _trace(self._h, None, 0)
        if n < 0:
            _raise(int(n))
        if n == 0:
            return np.zeros((3, 0, 16), dtype=np.uint64)
        buf = np.zeros(n, dtype=np.uint64)
        k = _trace(self._h, buf.ctypes.data, n)
        if k < 0:
            _raise(int(k))
        return buf.reshape(3, -1, 16)

    def pass_times(self) -> list[float]:
        buf = (ctypes.c_float * 8)()
        k = _pass_times(self._h, buf, 8)
        if k < 0:
            _raise(k)
        return [float(buf[i]) for i in range(k)]


def scatter_baseline(p_dev, a, b, stream=None, elem_bytes: int = 4):
    """D-designated b[p[i]] = a[i], one kernel. p_dev: int32 CUDA tensor."""
    n = p_dev.numel()
    _check(_scatter(_ptr(p_dev), _ptr(a), _ptr(b), n, elem_bytes, _stream_handle(stream)))
    return b


def gather_baseline(q_dev, a, b, stream=None, elem_bytes: int = 4):
    """S-designated b[i] = a[q[i]], q = P^{-1} on the device."""
    n = q_dev.numel()
    _check(_gather(_ptr(q_dev), _ptr(a), _ptr(b), n, elem_bytes, _stream_handle(stream)))
    return b


def copy_kernel(a, b, stream=None):
    _check(_copy(_ptr(a), _ptr(b), a.numel(), a.element_size(), _stream_handle(stream)))
    return b


def last_error() -> tuple[int, str]:
    return int(_last_error()), _last_error_string().decode()
