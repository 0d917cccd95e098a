#!/usr/bin/env python
"""NVML energy-counter validation (SURVEY §8(d) "NVML calibration"; the a9 protocol).

    python harness/nvml_check.py [--seconds 3] [--out nvml_check.json]

Before any energy window is trusted: (1) poll nvmlDeviceGetTotalEnergyConsumption every 1 ms for a
while under load to measure the counter's update interval; (2) keep the GPU busy with back-to-back
EATSS runs (gemm N=4000, the tensor-mode pick) for --seconds while a 10 ms sampler records the
board power (eatss_power_sample), and compare the counter's energy delta over the window with the
trapezoidal integral of the sampled power; (3) the same at idle.  The a9 windows are >= 0.5 s
(>= 5 counter updates) and aligned to counter updates, so the counter's quantisation does not enter.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seconds", type=float, default=3.0)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "nvml_check.json"))
    return ap.parse_args()


def window(E, busy, seconds, device=0):
    """Energy counter delta vs integral of 10 ms power samples over [first update, last update]."""
    samples = []
    stop = threading.Event()

    def sampler():
        while not stop.is_set():
            mw, mhz = E.power_sample(device)
            samples.append((time.perf_counter(), mw / 1e3))
            time.sleep(0.01)

    th = threading.Thread(target=sampler, daemon=True)
    # align the window to counter updates (as the a9 protocol does)
    e_prev = E.energy_mj(device)
    while True:
        e0 = E.energy_mj(device)
        if e0 != e_prev:
            t0 = time.perf_counter()
            break
    th.start()
    t_end = t0 + seconds
    while time.perf_counter() < t_end:
        busy()
    e_last = E.energy_mj(device)
    while True:  # close at the next counter update
        busy()
        e1 = E.energy_mj(device)
        if e1 != e_last:
            t1 = time.perf_counter()
            break
    stop.set()
    th.join()
    pts = [(t, w) for t, w in samples if t0 <= t <= t1]
    integ = sum((b[0] - a[0]) * (a[1] + b[1]) / 2 for a, b in zip(pts, pts[1:]))
    integ += (pts[0][0] - t0) * pts[0][1] + (t1 - pts[-1][0]) * pts[-1][1] if pts else 0.0
    counter_j = (e1 - e0) / 1e3
    return {"seconds": t1 - t0, "counter_joules": counter_j, "integral_joules": integ,
            "avg_watts_counter": counter_j / (t1 - t0), "samples": len(pts),
            "rel_diff": (counter_j - integ) / integ if integ > 0 else None}


def main():
    a = parse()
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    torch.cuda.set_device(0)
    n = 4000
    d = E.desc_builtin("gemm", (n, n, n))
    gpu = E.gpu_params_query(0)
    tiles, _ = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=2)
    d.set_exec(split_pct=50, engine=2)
    g = torch.Generator(device="cuda").manual_seed(0)
    bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=g) * 2 - 1 for i in range(3)]

    def busy():
        for _ in range(4):
            E.run(d, tiles, bufs)
        torch.cuda.synchronize()

    # (1) counter update interval under load: 1 ms polls
    busy()
    changes, last, t_start = [], E.energy_mj(0), time.perf_counter()
    while time.perf_counter() - t_start < 1.5:
        E.run(d, tiles, bufs)
        v = E.energy_mj(0)
        if v != last:
            changes.append(time.perf_counter())
            last = v
        time.sleep(0.001)
    torch.cuda.synchronize()
    gaps = [(b - a) * 1e3 for a, b in zip(changes, changes[1:])]
    interval = sorted(gaps)[len(gaps) // 2] if gaps else None
    out = {"counter_update_ms_median": interval, "counter_updates_seen": len(changes)}
    # (2) loaded window, (3) idle window
    out["loaded"] = window(E, busy, a.seconds)
    out["idle"] = window(E, lambda: time.sleep(0.002), a.seconds)
    out["pass_within_5pct"] = all(abs(out[k]["rel_diff"]) < 0.05 for k in ("loaded", "idle")
                                  if out[k]["rel_diff"] is not None)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
