#!/usr/bin/env python
"""BASELINE config 4 on the paper's metric: EATSS-tiled vs untiled stencils, time and energy (a9
protocol: eatss_sweep, >= --window s of back-to-back runs aligned to NVML counter updates),
PPW = FLOP/J.  jacobi-2d N=4000 and heat-3d N=120, 500 time steps, U[-1,1) fields."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--window", type=float, default=1.0)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "untiled_ppw.json"))
    a = ap.parse_args()
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    gpu = E.gpu_params_query(0)
    res = {}
    for kind, n in (("jacobi-2d", 4000), ("heat-3d", 120)):
        d = E.desc_builtin(kind, (n,), tsteps=500)
        tiles, _ = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=1)
        g = torch.Generator(device="cuda").manual_seed(0)
        bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=g) * 2 - 1 for i in range(2)]
        row = {}
        for name, engine in (("eatss", 1), ("untiled", 3)):
            d.set_exec(split_pct=50, engine=engine)
            m = E.sweep(d, [tiles], bufs, device=0, warmup=2, min_window_s=a.window)[0]
            row[name] = dict(tiles=list(tiles) if engine == 1 else None, ms=m.ms_per_run, tflops=m.tflops,
                             watts=m.avg_watts, joules=m.joules_per_run, ppw=m.gflops_per_watt, status=m.status)
        row["speedup"] = row["untiled"]["ms"] / row["eatss"]["ms"]
        row["ppw_gain"] = row["eatss"]["ppw"] / row["untiled"]["ppw"]
        res[f"{kind} n={n} T=500"] = row
        print(kind, json.dumps(row), flush=True)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
