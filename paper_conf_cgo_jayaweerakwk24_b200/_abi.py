"""ctypes declarations of include/eatss.h (argument marshalling only).

Loads the in-tree ``libeatss.so``.  There is no fallback of any kind: if the
library is missing or fails to load, importing the package raises.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libeatss.so")

EATSS_OK = 0
EATSS_E_INVALID = -1
EATSS_E_INFEASIBLE = -2
EATSS_E_CUDA = -3
EATSS_E_NVML = -4
EATSS_E_UNSUPPORTED = -5
EATSS_E_NOMEM = -6
STATUS_NAMES = {0: "OK", -1: "E_INVALID", -2: "E_INFEASIBLE", -3: "E_CUDA", -4: "E_NVML",
                -5: "E_UNSUPPORTED", -6: "E_NOMEM"}

F32, F64 = 1, 2
BUILTINS = {"gemm": 0, "2mm": 1, "3mm": 2, "syrk": 3, "jacobi-2d": 4, "heat-3d": 5, "ccsd_t_d1": 6,
            "mvt": 7, "atax": 8, "bicg": 9, "gemver": 10, "mttkrp": 11, "conv-2d": 12}
ENGINE_AUTO, ENGINE_SIMT, ENGINE_TENSOR, ENGINE_UNTILED, ENGINE_TENSOR_F16 = 0, 1, 2, 3, 4
MAX_LOOPS = 8
MAX_NESTS = 4
MAX_BUFFERS = 16

I64 = ctypes.c_int64
I32 = ctypes.c_int32
P = ctypes.c_void_p


class GpuParams(ctypes.Structure):
    _fields_ = [("threads_per_block", I64), ("threads_per_warp", I64), ("regs_per_thread", I64),
                ("regs_per_sm", I64), ("regs_per_block", I64), ("l1_shared_bytes", I64),
                ("l2_bytes", I64), ("num_sms", I64), ("max_smem_per_block", I64)]


class ModelOpts(ctypes.Structure):
    _fields_ = [("split_pct", I32), ("warp_align", I32), ("mode", I32)]


class ModelReport(ctypes.Structure):
    _fields_ = [("ls1_loop", I32), ("nrefs", I32), ("obj", I64), ("n_feasible", I64), ("n_ties", I64),
                ("m_l1", I64), ("m_sh", I64), ("b_size", I64), ("reg_sm", I64),
                ("solve_seconds", ctypes.c_double)]


class ExecOpts(ctypes.Structure):
    _fields_ = [("split_pct", I32), ("engine", I32), ("use_graph", I32), ("time_kernels", I32),
                ("warp_align", I32), ("carveout_exact", I32)]


class LaunchPlan(ctypes.Structure):
    _fields_ = [("nest", I32), ("engine", I32), ("grid_x", I64), ("grid_y", I64), ("grid_z", I64),
                ("block_x", I32), ("block_y", I32), ("rm", I32), ("rn", I32), ("vec", I32),
                ("passes", I32), ("smem_bytes", I32), ("a_in_smem", I32), ("b_in_smem", I32),
                ("carveout_pct", I32), ("simt_x", I32), ("tile", I64 * MAX_LOOPS)]


class Measurement(ctypes.Structure):
    _fields_ = [("ms_per_run", ctypes.c_double), ("joules_per_run", ctypes.c_double),
                ("avg_watts", ctypes.c_double), ("tflops", ctypes.c_double),
                ("gflops_per_watt", ctypes.c_double), ("sm_mhz_median", ctypes.c_double),
                ("runs", I64), ("status", I32), ("reserved", I32)]


# (name, restype, argtypes) -- one line per declaration in include/eatss.h
DECLS = [
    ("eatss_desc_builtin", I32, [I32, ctypes.POINTER(I64), ctypes.c_int, I32, I64, ctypes.POINTER(P)]),
    ("eatss_desc_destroy", None, [P]),
    ("eatss_desc_num_loops", ctypes.c_int, [P]),
    ("eatss_desc_num_nests", ctypes.c_int, [P]),
    ("eatss_desc_num_buffers", ctypes.c_int, [P]),
    ("eatss_desc_buffer_elems", I64, [P, ctypes.c_int]),
    ("eatss_desc_flops", ctypes.c_double, [P]),
    ("eatss_desc_bytes", ctypes.c_double, [P]),
    ("eatss_desc_set_scalars", I32, [P, ctypes.c_double, ctypes.c_double]),
    ("eatss_desc_set_exec", I32, [P, ctypes.POINTER(ExecOpts)]),
    ("eatss_desc_model_info", I32, [P, ctypes.c_int, ctypes.c_int, ctypes.POINTER(I32), ctypes.POINTER(I32),
                                    ctypes.POINTER(I64)]),
    ("eatss_gpu_params_query", I32, [ctypes.c_int, ctypes.POINTER(GpuParams)]),
    ("eatss_gpu_params_b200", I32, [ctypes.POINTER(GpuParams)]),
    ("eatss_gpu_params_ga100", I32, [ctypes.POINTER(GpuParams)]),
    ("eatss_select_tiles", I32, [P, ctypes.POINTER(GpuParams), ctypes.POINTER(ModelOpts), ctypes.POINTER(I64),
                                 ctypes.POINTER(ModelReport)]),
    ("eatss_plan", I32, [P, ctypes.POINTER(I64), ctypes.POINTER(LaunchPlan), ctypes.c_int,
                         ctypes.POINTER(ctypes.c_int)]),
    ("eatss_run", I32, [P, ctypes.POINTER(I64), ctypes.POINTER(P), P]),
    ("eatss_run_host", I32, [P, ctypes.POINTER(I64), ctypes.POINTER(P), I64, P]),
    ("eatss_run_nest", I32, [P, ctypes.c_int, ctypes.POINTER(I64), ctypes.POINTER(P), P]),
    ("eatss_coverage", I32, [P, ctypes.c_int, ctypes.POINTER(I64), P, P]),
    ("eatss_launches_per_run", I64, [P, ctypes.POINTER(I64)]),
    ("eatss_last_kernel_ms", I32, [P, ctypes.POINTER(ctypes.c_float), I32, ctypes.POINTER(I32)]),
    ("eatss_last_carveout", I32, [P, ctypes.POINTER(I32), I32, ctypes.POINTER(I32)]),
    ("eatss_energy_mj", I32, [ctypes.c_int, ctypes.POINTER(ctypes.c_uint64)]),
    ("eatss_power_sample", I32, [ctypes.c_int, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]),
    ("eatss_sweep", I32, [P, ctypes.POINTER(I64), ctypes.c_int, ctypes.POINTER(P), ctypes.c_int, ctypes.c_int,
                          ctypes.c_double, ctypes.POINTER(Measurement)]),
    ("eatss_last_error", ctypes.c_char_p, []),
    ("eatss_abi_version", ctypes.c_int, []),
]


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    if not os.path.exists(path):
        raise ImportError(
            f"{path} not found: build it with `python paper_conf_cgo_jayaweerakwk24_b200/build.py` "
            "(there is no CPU fallback)")
    lib = ctypes.CDLL(path)
    for name, res, args in DECLS:
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib
