#!/usr/bin/env python
"""bench.py -- headline benchmark: EATSS-tiled gemm N=4000 fp32 on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

One step = one pass of the whole hot path on one problem: build the kernel
descriptor's model inputs -> select the tile vector with the EATSS model
(host enumeration) -> execute the tiled gemm N=4000 (SIMT contraction executor)
in libeatss.so.  Metric (BASELINE.json): TFLOP/s and GFLOP/s per Watt.
For N > 1 (torchrun, one process per GPU, NCCL) every rank runs its own
N=4000 problem (weak scaling, no data-path collective); timing is the max over
ranks of the device-timed region, energy the sum over ranks.

Prints ONE JSON line on rank 0 (see DESIGN.md §6 for every key).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N = 4000
METRIC = "GFLOP/s per Watt and TFLOP/s of EATSS-tiled affine kernels (gemm N=4000)"
FLOPS = 2.0 * N ** 3
SM_COUNT, FP32_LANES = 148, 128


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    return ap.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except Exception:
        return {}


# ------------------------------------------------------------------ CPU oracle leg
def cpu_oracle_sample(target_s: float = 12.0):
    """Time the fp64 oracle on a bounded row block of the same gemm N=4000."""
    import synth
    from oracle import numeric as O

    A = synth.uniform((N, N), 0)
    B = synth.uniform((N, N), 1)
    C = synth.uniform((N, N), 2)
    O.lib()

    def run_rows(r):
        t0 = time.perf_counter()
        O.gemm(1.5, 1.2, C[:r], A[:r], B)
        return time.perf_counter() - t0

    t = run_rows(16)
    rows = int(min(N, max(16, 16 * target_s / max(t, 1e-3))))
    t = run_rows(rows)
    flops = 2.0 * rows * N * N
    return {"value": flops / t / 1e12, "unit": "TFLOP/s", "cores": O.num_threads(), "kind": "oracle",
            "sample": f"fp64 oracle (oracle/oracle.c, OpenMP) on rows 0..{rows - 1} of gemm N=4000 "
                      f"({flops:.3g} flop, {t:.2f} s)"}


def reference_arm(args, ws, rank):
    if rank != 0:
        return
    import synth
    from oracle import numeric as O

    A = synth.uniform((N, N), 0)
    B = synth.uniform((N, N), 1)
    C = synth.uniform((N, N), 2)
    rows = 32
    flops = 2.0 * rows * N * N
    for _ in range(args.warmup):
        O.gemm(1.5, 1.2, C[:rows], A[:rows], B)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        O.gemm(1.5, 1.2, C[:rows], A[:rows], B)
    dt = time.perf_counter() - t0
    value = flops * args.steps / dt / 1e12
    sample = f"each step: fp64 oracle on rows 0..{rows - 1} of gemm N=4000 ({flops:.3g} flop)"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic U[-1,1) PCG64 seeds 0,1,2",
        "config": {"workload": "gemm N=4000 (row-block sample on host cores)", "rows_per_step": rows},
        "cpu_baseline": {"value": value, "unit": "TFLOP/s", "cores": O.num_threads(), "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": value, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """NVML sampler of SM clock / power / throttle reasons during the timed region."""
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device_index: int):
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            import torch
            # match the CUDA device to its NVML handle by UUID (CUDA_VISIBLE_DEVICES safe)
            want = "GPU-" + str(torch.cuda.get_device_properties(device_index).uuid)
            h = None
            for i in range(pynvml.nvmlDeviceGetCount()):
                hi = pynvml.nvmlDeviceGetHandleByIndex(i)
                u = pynvml.nvmlDeviceGetUUID(hi)
                u = u.decode() if isinstance(u, bytes) else u
                if u == want:
                    h = hi
                    break
            if h is None:
                h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.nv, self.h, self.ok = pynvml, h, True
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.max_mhz = None
        self.mhz, self.mw, self.reasons = [], [], 0
        self._stop = threading.Event()

    def energy_mj(self):
        if not self.ok:
            return None
        try:
            return self.nv.nvmlDeviceGetTotalEnergyConsumption(self.h)
        except Exception:
            return None

    def _loop(self):
        while not self._stop.is_set():
            try:
                self.mhz.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.mw.append(self.nv.nvmlDeviceGetPowerUsage(self.h))
                self.reasons |= self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(0.05)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._loop, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        reasons = [n for b, n in self.REASONS.items() if self.reasons & b and n != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.mhz) if self.mhz else None, "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(self.mhz),
                "power_w_median": statistics.median(self.mw) / 1e3 if self.mw else None}


# ------------------------------------------------------------------ our arm
def main():
    args = parse()
    ws, rank, local = dist_env()
    if args.impl == "reference":
        reference_arm(args, ws, rank)
        return
    import torch
    import torch.distributed as dist

    import paper_conf_cgo_jayaweerakwk24_b200 as E
    import synth

    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (there is no CPU fallback)")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if ws > 1:
        dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream()

    # inputs: U[-1,1) PCG64 seeds 0,1,2 (same generator as the oracle side), resident in HBM
    A_h = synth.uniform((N, N), 0); B_h = synth.uniform((N, N), 1); C_h = synth.uniform((N, N), 2)
    A = torch.from_numpy(A_h).to(dev); B = torch.from_numpy(B_h).to(dev); C = torch.from_numpy(C_h).to(dev)
    gpu = E.gpu_params_query(local)
    alpha, beta = 1.5, 1.2

    def step():
        d = E.desc_builtin("gemm", (N, N, N))                      # a1 kernel descriptor
        d.set_scalars(alpha, beta)
        tiles, rep = E.select_tiles(d, gpu, split_pct=50, waf=16)  # a2-a4 model + tile selection
        d.set_exec(split_pct=50)                                   # a5 carve-out from the split
        E.run(d, tiles, [C, A, B], stream)                         # a5-a6 launch plan + tiled execution
        return d, tiles, rep

    for _ in range(max(3, args.warmup)):
        d, tiles, rep = step()
    torch.cuda.synchronize()
    plans = E.plan(d, tiles)
    launches_per_step = E.launches_per_run(d, tiles)

    clk = ClockSampler(local)
    K = args.steps
    ev_s = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    ev_e = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    t_start = torch.cuda.Event(enable_timing=True); t_end = torch.cuda.Event(enable_timing=True)
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with clk:
        e0 = clk.energy_mj()
        t_start.record(stream)
        for i in range(K):
            dd = E.desc_builtin("gemm", (N, N, N))
            dd.set_scalars(alpha, beta)
            tt, _ = E.select_tiles(dd, gpu, split_pct=50, waf=16)
            dd.set_exec(split_pct=50)
            ev_s[i].record(stream)
            E.run(dd, tt, [C, A, B], stream)
            ev_e[i].record(stream)
        t_end.record(stream)
        torch.cuda.synchronize()
        e1 = clk.energy_mj()
    if ws > 1:
        dist.barrier()
    ms_total = t_start.elapsed_time(t_end)
    kern_ms = [ev_s[i].elapsed_time(ev_e[i]) for i in range(K)]
    joules = (e1 - e0) / 1e3 if (e0 is not None and e1 is not None) else float("nan")

    # e2e through the public API with host buffers (pinned), copies inside the timed region
    A_p = torch.from_numpy(A_h).pin_memory(); B_p = torch.from_numpy(B_h).pin_memory()
    C_p = torch.from_numpy(C_h).pin_memory(); C_out = torch.empty_like(C_p).pin_memory()
    A2 = torch.empty_like(A); B2 = torch.empty_like(B); C2 = torch.empty_like(C)
    Ke = args.e2e_steps
    for _ in range(2):
        A2.copy_(A_p, non_blocking=True); B2.copy_(B_p, non_blocking=True); C2.copy_(C_p, non_blocking=True)
        step_d, step_t, _ = step()
        E.run(step_d, step_t, [C2, A2, B2], stream)
        C_out.copy_(C2, non_blocking=True)
    torch.cuda.synchronize()
    e2s = torch.cuda.Event(enable_timing=True); e2e_ev = torch.cuda.Event(enable_timing=True)
    if ws > 1:
        dist.barrier()
    e2s.record(stream)
    for _ in range(Ke):
        A2.copy_(A_p, non_blocking=True); B2.copy_(B_p, non_blocking=True); C2.copy_(C_p, non_blocking=True)
        dd = E.desc_builtin("gemm", (N, N, N)); dd.set_scalars(alpha, beta)
        tt, _ = E.select_tiles(dd, gpu, split_pct=50, waf=16)
        E.run(dd, tt, [C2, A2, B2], stream)
        C_out.copy_(C2, non_blocking=True)
    e2e_ev.record(stream)
    torch.cuda.synchronize()
    e2e_ms = e2s.elapsed_time(e2e_ev) / Ke

    # max over ranks (time), sum over ranks (energy)
    vals = torch.tensor([ms_total, e2e_ms, float(np.mean(kern_ms))], dtype=torch.float64, device=dev)
    en = torch.tensor([joules], dtype=torch.float64, device=dev)
    if ws > 1:
        dist.all_reduce(vals, op=dist.ReduceOp.MAX)
        dist.all_reduce(en, op=dist.ReduceOp.SUM)
    ms_total, e2e_ms, kern_avg_ms = vals.tolist()
    joules = en.item()

    if rank == 0:
        total_flops = FLOPS * K * ws
        value = total_flops / (ms_total * 1e-3) / 1e12
        clocks = clk.summary()
        peaks = measured_peaks()
        sm_max = clocks.get("sm_max_mhz") or peaks.get("sm_max_mhz") or 1965.0
        fp32_peak = SM_COUNT * FP32_LANES * 2 * sm_max * 1e6 / 1e12
        achieved = FLOPS / (kern_avg_ms * 1e-3) / 1e12
        traffic = None
        tp = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tp):
            try:
                traffic = json.load(open(tp)).get("gemm_eatss_tile", {}).get("dram_bytes_per_launch")
            except Exception:
                traffic = None
        p0 = plans[0]
        out = {
            "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": ws, "steps": K,
            "warmup": max(3, args.warmup), "ms_per_step": ms_total / K, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic: A, B, C ~ U[-1,1) numpy PCG64 seeds 0,1,2; alpha=1.5 beta=1.2",
            "config": {"workload": "gemm N=4000 fp32 (BASELINE configs[1]), EATSS-selected tile",
                       "tiles": list(tiles), "model": {"split_pct": 50, "waf": 16, "mode": "B200",
                                                        "obj": rep.obj, "n_ties": rep.n_ties},
                       "engine": "SIMT contraction executor (FFMA)",
                       "launch": {"grid": [p0.grid_x, p0.grid_y], "block": [p0.block_x, p0.block_y],
                                  "micro_tile": [p0.rm, p0.rn], "vec": p0.vec, "smem_bytes": p0.smem_bytes},
                       "l2": "inputs 192 MB (A,B,C) > 126 MB L2; no flush",
                       "parallelism": f"dp{ws} independent problems"},
            "energy": {"joules_per_step": joules / K / ws if joules == joules else None,
                       "avg_watts_per_gpu": joules / (ms_total * 1e-3) / ws if joules == joules else None,
                       "gflops_per_watt": total_flops / joules / 1e9 if joules == joules and joules > 0 else None,
                       "source": "NVML total-energy counter over the timed region, summed over ranks"},
            "roofline": {"bound": "alu", "achieved": achieved, "peak": fp32_peak, "unit": "TFLOP/s",
                         "frac": achieved / fp32_peak, "traffic": traffic,
                         "kernel": (f"contract_staged_kernel<float,{p0.rm},{p0.rn},{p0.vec},false>"
                                    if (p0.b_in_smem and p0.passes == 1) else
                                    f"contract_kernel<float,{p0.rm},{p0.rn},{p0.vec},false>"),
                         "peak_source": f"148 SMs x 128 FP32 lanes x 2 flop x {sm_max:.0f} MHz (sm max clock)",
                         "frac_at_observed_clock": (achieved / (SM_COUNT * FP32_LANES * 2 * clocks["sm_mhz"] * 1e-6))
                         if clocks.get("sm_mhz") else None},
            "e2e": {"value": FLOPS * ws / (e2e_ms * 1e-3) / 1e12, "unit": "TFLOP/s",
                    "h2d_bytes_per_step": int(3 * N * N * 4), "d2h_bytes_per_step": int(N * N * 4)},
            "gpu_launches": int(K * launches_per_step),
            "clocks": clocks,
        }
        if not args.no_cpu_baseline:
            out["cpu_baseline"] = cpu_oracle_sample()
        print(json.dumps(out), flush=True)
    if ws > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
