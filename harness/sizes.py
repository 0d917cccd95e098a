#!/usr/bin/env python
"""Problem-size sensitivity of EATSS-tiled gemm, conv-2d and mttkrp (Figs. 1, 12, 13).

    python harness/sizes.py [--kind gemm|conv-2d|mttkrp] [--sizes 512,1024,...] [--out sizes.jsonl]

Fig. 13 repeats the study for the non-PolyBench kernels ("for conv-2d, the performance-per-Watt
is higher than observed using the baseline PPCG"): --kind conv-2d sweeps the image size n (5 x 5
filter, reading R-N9) and --kind mttkrp the tensor extent I = K = L (rank J = 32, reading R-N8), EATSS
(B200 mode, WAF 16; mttkrp also at its tensor-pipe point) against the default tile 32 per loop.

The paper's model is problem-size agnostic and its Figs. 12-13 show how performance and
average power move with the input size.  For each N the model selects the tile in
both EATSS modes (B200 mode -> SIMT executor; tensor-core mode, reading T -> tcgen05 3xTF32) and
the a9 protocol (eatss_sweep: warm-up, >= --window s of back-to-back runs, NVML energy counter,
P:225) measures time, average power and PPW.  The PPCG default tile 32^3 on the
SIMT executor is measured alongside as the paper's baseline.  Inputs U[-1,1).
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kind", default="gemm", choices=["gemm", "conv-2d", "mttkrp"])
    ap.add_argument("--sizes", default="")
    ap.add_argument("--window", type=float, default=1.0)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sizes.jsonl"))
    return ap.parse_args()


def main():
    a = parse()
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    gpu = E.gpu_params_query(0)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    rows = []
    default_sizes = {"gemm": "512,1024,2048,4000,8192", "conv-2d": "1024,2048,4096,8192,16384",
                     "mttkrp": "128,256,384,512,768"}[a.kind]
    with open(a.out, "a") as f:
        for n in [int(x) for x in (a.sizes or default_sizes).split(",")]:
            dims = {"gemm": (n, n, n), "conv-2d": (n, 5), "mttkrp": (n, 32, n, n)}[a.kind]
            d = E.desc_builtin(a.kind, dims)
            g = torch.Generator(device="cuda").manual_seed(n)
            bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=g) * 2 - 1 for i in range(d.num_buffers)]
            arms = []
            if a.kind == "gemm":
                for name, mode, engine in (("eatss-tensor", 2, 2), ("eatss-simt", 1, 1)):
                    tiles, rep = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=mode)
                    arms.append((name, tuple(tiles), engine))
            else:
                tiles, rep = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=1)
                arms.append(("eatss-simt", tuple(tiles), 1))
                if a.kind == "mttkrp":
                    arms.append(("mma-legal-tensor", (1, 32, 128, 32), 2))
            arms.append(("ppcg-default", tuple([32] * d.num_loops), 1))
            for name, tiles, engine in arms:
                d.set_exec(split_pct=50, engine=engine)
                m = E.sweep(d, [tiles], bufs, warmup=3, min_window_s=a.window)[0]
                rec = dict(kind=a.kind, n=n, arm=name, tiles=list(tiles), ms=m.ms_per_run, tflops=m.tflops, watts=m.avg_watts,
                           ppw=m.gflops_per_watt, sm_mhz=m.sm_mhz_median, status=m.status)
                rows.append(rec)
                f.write(json.dumps(rec) + "\n")
                f.flush()
                print(json.dumps(rec), flush=True)
            del bufs
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
