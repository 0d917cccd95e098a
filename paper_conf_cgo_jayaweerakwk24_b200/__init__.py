"""EATSS on B200 -- Python binding of libeatss.so (include/eatss.h).

Same names as the C ABI without the ``eatss_`` prefix; this layer only marshals
arguments (device buffers are passed as pointers, e.g. ``tensor.data_ptr()``;
streams as ``torch.cuda.Stream`` or raw ``cudaStream_t`` integers).  Every step
of the hot path runs in libeatss.so; there is no Python or CPU fallback.

    import paper_conf_cgo_jayaweerakwk24_b200 as eatss
    d = eatss.desc_builtin("gemm", (4000, 4000, 4000))
    tiles, rep = eatss.select_tiles(d, eatss.gpu_params_b200(), split_pct=50, waf=16)
    eatss.run(d, tiles, [C, A, B])        # torch CUDA tensors, on the current stream
"""
from __future__ import annotations

import ctypes
from typing import List, Optional, Sequence, Tuple

from . import _abi

_lib = _abi.load()

__all__ = [
    "EatssError", "Desc", "desc_builtin", "gpu_params_query", "gpu_params_b200", "gpu_params_ga100",
    "select_tiles", "plan", "run", "run_nest", "coverage", "launches_per_run", "last_kernel_ms", "last_carveout",
    "energy_mj",
    "power_sample", "sweep", "last_error", "abi_version", "lib_path",
]

lib_path = _abi.LIB_PATH


class EatssError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = _lib.eatss_last_error().decode(errors="replace")
        super().__init__(f"{where}: {_abi.STATUS_NAMES.get(status, status)}: {msg}")


def _check(st: int, where: str) -> None:
    if st != _abi.EATSS_OK:
        raise EatssError(st, where)


def _i64s(vals) -> ctypes.Array:
    vals = [int(v) for v in vals]
    return (ctypes.c_int64 * max(1, len(vals)))(*vals)


def _ptr(x) -> int:
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return int(x.data_ptr())
    raise TypeError(f"cannot take a device pointer of {type(x)}")


def _stream(s) -> Optional[int]:
    if s is None:
        try:
            import torch
            return int(torch.cuda.current_stream().cuda_stream)
        except Exception:  # no torch / no device: legacy default stream
            return None
    if isinstance(s, int):
        return s
    return int(s.cuda_stream)


class Desc:
    """Owning handle of an ``eatss_kernel_desc``."""

    def __init__(self, handle: int, kind: str):
        self._h = ctypes.c_void_p(handle)
        self.kind = kind

    @property
    def handle(self) -> ctypes.c_void_p:
        return self._h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            if _lib is not None:  # interpreter shutdown may have cleared module globals
                _lib.eatss_desc_destroy(h)
            self._h = None

    @property
    def num_loops(self) -> int:
        return _lib.eatss_desc_num_loops(self._h)

    @property
    def num_nests(self) -> int:
        return _lib.eatss_desc_num_nests(self._h)

    @property
    def num_buffers(self) -> int:
        return _lib.eatss_desc_num_buffers(self._h)

    def buffer_elems(self, i: int) -> int:
        return _lib.eatss_desc_buffer_elems(self._h, i)

    @property
    def flops(self) -> float:
        return _lib.eatss_desc_flops(self._h)

    @property
    def bytes(self) -> float:
        return _lib.eatss_desc_bytes(self._h)

    def set_scalars(self, alpha: float, beta: float) -> None:
        _check(_lib.eatss_desc_set_scalars(self._h, float(alpha), float(beta)), "desc_set_scalars")

    def set_exec(self, split_pct: int = 50, engine: int = 0, use_graph: int = 1, time_kernels: int = 0,
                 warp_align: int = 0, carveout_exact: int = 0) -> None:
        o = _abi.ExecOpts(split_pct, engine, use_graph, time_kernels, warp_align, carveout_exact)
        _check(_lib.eatss_desc_set_exec(self._h, ctypes.byref(o)), "desc_set_exec")

    def model_info(self, nest: int = 0, waf: int = 16):
        ls1 = ctypes.c_int32(); nrefs = ctypes.c_int32()
        H = (ctypes.c_int64 * _abi.MAX_LOOPS)()
        _check(_lib.eatss_desc_model_info(self._h, nest, waf, ctypes.byref(ls1), ctypes.byref(nrefs), H),
               "desc_model_info")
        return ls1.value, nrefs.value, list(H)[: self.num_loops]


def desc_builtin(kind: str, dims: Sequence[int], dtype: str = "f32", tsteps: int = 0) -> Desc:
    if kind not in _abi.BUILTINS:
        raise ValueError(f"unknown builtin {kind!r}; one of {sorted(_abi.BUILTINS)}")
    dt = {"f32": _abi.F32, "f64": _abi.F64}[dtype]
    out = ctypes.c_void_p()
    dv = _i64s(dims)
    _check(_lib.eatss_desc_builtin(_abi.BUILTINS[kind], dv, len(dims), dt, int(tsteps), ctypes.byref(out)),
           "desc_builtin")
    return Desc(out.value, kind)


def gpu_params_query(device: int = 0) -> _abi.GpuParams:
    g = _abi.GpuParams()
    _check(_lib.eatss_gpu_params_query(device, ctypes.byref(g)), "gpu_params_query")
    return g


def gpu_params_b200() -> _abi.GpuParams:
    g = _abi.GpuParams()
    _check(_lib.eatss_gpu_params_b200(ctypes.byref(g)), "gpu_params_b200")
    return g


def gpu_params_ga100() -> _abi.GpuParams:
    g = _abi.GpuParams()
    _check(_lib.eatss_gpu_params_ga100(ctypes.byref(g)), "gpu_params_ga100")
    return g


def select_tiles(d: Desc, gpu: _abi.GpuParams, split_pct: int = 50, waf: int = 16,
                 mode: int = 1) -> Tuple[Tuple[int, ...], _abi.ModelReport]:
    """Returns (tiles, report); raises EatssError(E_INFEASIBLE) on an empty space."""
    o = _abi.ModelOpts(split_pct, waf, mode)
    t = (ctypes.c_int64 * d.num_loops)()
    rep = _abi.ModelReport()
    _check(_lib.eatss_select_tiles(d.handle, ctypes.byref(gpu), ctypes.byref(o), t, ctypes.byref(rep)),
           "select_tiles")
    return tuple(t), rep


def plan(d: Desc, tiles: Sequence[int]) -> List[_abi.LaunchPlan]:
    arr = (_abi.LaunchPlan * _abi.MAX_NESTS)()
    n = ctypes.c_int()
    _check(_lib.eatss_plan(d.handle, _i64s(tiles), arr, _abi.MAX_NESTS, ctypes.byref(n)), "plan")
    return [arr[i] for i in range(n.value)]


def _bufs(d: Desc, buffers) -> ctypes.Array:
    if len(buffers) != d.num_buffers:
        raise ValueError(f"{d.kind}: expected {d.num_buffers} buffers, got {len(buffers)}")
    return (ctypes.c_void_p * len(buffers))(*[_ptr(b) for b in buffers])


def run(d: Desc, tiles: Sequence[int], buffers, stream=None) -> None:
    _check(_lib.eatss_run(d.handle, _i64s(tiles), _bufs(d, buffers), _stream(stream)), "run")


def _host_ptr(x) -> int:
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr") and hasattr(x, "is_cuda"):
        if x.is_cuda:
            raise TypeError("run_host takes host buffers")
        return int(x.data_ptr())
    if hasattr(x, "ctypes"):  # numpy array
        return int(x.ctypes.data)
    raise TypeError(f"cannot take a host pointer of {type(x)}")


def run_host(d: Desc, tiles: Sequence[int], host_buffers, row_blocks: int = 1, stream=None) -> None:
    """eatss_run_host: host buffers in, outputs copied back; complete when `stream` reaches the end."""
    if len(host_buffers) != d.num_buffers:
        raise ValueError(f"{d.kind}: expected {d.num_buffers} buffers, got {len(host_buffers)}")
    arr = (ctypes.c_void_p * len(host_buffers))(*[_host_ptr(b) for b in host_buffers])
    _check(_lib.eatss_run_host(d.handle, _i64s(tiles), arr, int(row_blocks), _stream(stream)), "run_host")


def run_nest(d: Desc, nest: int, tiles: Sequence[int], buffers, stream=None) -> None:
    _check(_lib.eatss_run_nest(d.handle, nest, _i64s(tiles), _bufs(d, buffers), _stream(stream)), "run_nest")


def coverage(d: Desc, nest: int, tiles: Sequence[int], counts, stream=None) -> None:
    _check(_lib.eatss_coverage(d.handle, nest, _i64s(tiles), _ptr(counts), _stream(stream)), "coverage")


def launches_per_run(d: Desc, tiles: Sequence[int]) -> int:
    return int(_lib.eatss_launches_per_run(d.handle, _i64s(tiles)))


def last_kernel_ms(d: Desc) -> List[float]:
    """Device ms of each nest's main compute kernel in the last run with time_kernels=1 (blocks)."""
    cap = max(1, d.num_nests)
    ms = (ctypes.c_float * cap)(); n = ctypes.c_int32()
    _check(_lib.eatss_last_kernel_ms(d.handle, ms, cap, ctypes.byref(n)), "last_kernel_ms")
    return list(ms)[: n.value]


def last_carveout(d: Desc) -> List[int]:
    """Carve-out percent each nest's main kernel requested in the last run (-1: none set)."""
    cap = max(1, d.num_nests)
    v = (ctypes.c_int32 * cap)(); n = ctypes.c_int32()
    _check(_lib.eatss_last_carveout(d.handle, v, cap, ctypes.byref(n)), "last_carveout")
    return list(v)[: n.value]


def energy_mj(device: int = 0) -> int:
    v = ctypes.c_uint64()
    _check(_lib.eatss_energy_mj(device, ctypes.byref(v)), "energy_mj")
    return v.value


def power_sample(device: int = 0) -> Tuple[int, int]:
    mw = ctypes.c_uint32(); mhz = ctypes.c_uint32()
    _check(_lib.eatss_power_sample(device, ctypes.byref(mw), ctypes.byref(mhz)), "power_sample")
    return mw.value, mhz.value


def sweep(d: Desc, variants: Sequence[Sequence[int]], buffers, device: int = 0, warmup: int = 3,
          min_window_s: float = 0.5) -> List[_abi.Measurement]:
    L = d.num_loops
    flat = [int(v) for row in variants for v in row]
    if len(flat) != L * len(variants):
        raise ValueError("each variant needs num_loops entries")
    res = (_abi.Measurement * max(1, len(variants)))()
    _check(_lib.eatss_sweep(d.handle, _i64s(flat), len(variants), _bufs(d, buffers), device, warmup,
                            float(min_window_s), res), "sweep")
    return [res[i] for i in range(len(variants))]


def last_error() -> str:
    return _lib.eatss_last_error().decode(errors="replace")


def abi_version() -> int:
    return int(_lib.eatss_abi_version())
