#!/usr/bin/env python
"""Problem-size sensitivity of EATSS-tiled gemm (paper Figs. 1, 12, 13).

    python harness/sizes.py [--sizes 512,1024,2048,4000,8192] [--out sizes.jsonl]

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
    ap.add_argument("--sizes", default="512,1024,2048,4000,8192")
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
    with open(a.out, "w") as f:
        for n in [int(x) for x in a.sizes.split(",")]:
            d = E.desc_builtin("gemm", (n, n, n))
            g = torch.Generator(device="cuda").manual_seed(n)
            bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=g) * 2 - 1 for i in range(3)]
            arms = []
            for name, mode, engine in (("eatss-tensor", 2, 2), ("eatss-simt", 1, 1)):
                tiles, rep = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=mode)
                arms.append((name, tuple(tiles), engine))
            arms.append(("ppcg-default", (32, 32, 32), 1))
            for name, tiles, engine in arms:
                d.set_exec(split_pct=50, engine=engine)
                m = E.sweep(d, [tiles], bufs, warmup=3, min_window_s=a.window)[0]
                rec = dict(n=n, arm=name, tiles=list(tiles), ms=m.ms_per_run, tflops=m.tflops, watts=m.avg_watts,
                           ppw=m.gflops_per_watt, sm_mhz=m.sm_mhz_median, status=m.status)
                rows.append(rec)
                f.write(json.dumps(rec) + "\n")
                f.flush()
                print(json.dumps(rec), flush=True)
            del bufs
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
