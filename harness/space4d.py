#!/usr/bin/env python
"""Where EATSS lands in the explored tile space of the 4-D kernels (paper Fig. 11).

    python harness/space4d.py [--kinds mttkrp,conv-2d] [--count 150] [--window 0.3] [--out space.jsonl]

Fig. 11 places three markers in the performance / energy distribution of the
explored tile space of conv-2d, heat-3d and mttkrp: P = PPCG's default tile (32 per loop),
M = the median variant, U = the best EATSS candidate.  Here: --count seeded random variants of the
15-size space per loop (reading Q19; filter loops of conv-2d range over 1..f), each executed by the
library's SIMT executor at the 50% carve-out and measured with the a9 protocol (eatss_sweep,
P:225), plus the default tile and every EATSS candidate (the split x warp-fraction protocol at 50%).
The summary gives the percentile of P, of U and of the EATSS WAF-16 pick within the space, on
TFLOP/s and on PPW (GFLOP/s/W).  Inputs U[-1,1).
"""
from __future__ import annotations

import argparse
import json
import os
import random
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SIZES = [4, 8, 16, 24, 32, 48, 64, 96, 128, 192, 256, 384, 512, 768, 1024]
KINDS = {"mttkrp": (512, 32, 512, 512), "conv-2d": (8192, 5)}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kinds", default="mttkrp,conv-2d")
    ap.add_argument("--count", type=int, default=150)
    ap.add_argument("--window", type=float, default=0.3)
    ap.add_argument("--max-ms", type=float, default=20.0, help="skip variants slower than this per run")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "space4d.jsonl"))
    return ap.parse_args()


def main():
    a = parse()
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    gpu = E.gpu_params_query(0)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    summary = {}
    with open(a.out, "a") as f:
        for kind in a.kinds.split(","):
            dims = KINDS[kind]
            d = E.desc_builtin(kind, dims)
            d.set_exec(split_pct=50, engine=1)
            ext = [E.plan(d, [1 << 30] * 4)[0].tile[p] for p in range(4)]  # loop extents (tiles clip to them)
            doms = [sorted({min(s, e) for s in SIZES}) for e in ext]
            space = [tuple(v) for v in np.array(np.meshgrid(*doms, indexing="ij")).reshape(4, -1).T.tolist()]
            rng = random.Random(a.seed)
            sample = rng.sample(space, min(a.count, len(space)))
            default = tuple(min(32, e) for e in ext)
            cands = {}
            for w in (4, 8, 16, 32):
                try:
                    t, _ = E.select_tiles(d, gpu, split_pct=50, waf=w, mode=1)
                    cands[tuple(t)] = w
                except E.EatssError:
                    pass
            gen = torch.Generator(device="cuda").manual_seed(0)
            bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=gen) * 2 - 1 for i in range(d.num_buffers)]
            rows = []
            for role, v in [("default", default)] + [("eatss", t) for t in cands] + [("space", t) for t in sample]:
                # quick probe: skip pathological variants (they would dominate the GPU time)
                E.run(d, v, bufs)
                torch.cuda.synchronize()
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record(); E.run(d, v, bufs); e.record(); torch.cuda.synchronize()
                if s.elapsed_time(e) > a.max_ms and role == "space":
                    rec = dict(kind=kind, role=role, tiles=list(v), skipped_ms=s.elapsed_time(e))
                    f.write(json.dumps(rec) + "\n")
                    continue
                m = E.sweep(d, [v], bufs, device=0, warmup=2, min_window_s=a.window)[0]
                rec = dict(kind=kind, role=role, tiles=list(v), ms=m.ms_per_run, tflops=m.tflops, watts=m.avg_watts,
                           ppw=m.gflops_per_watt, status=m.status, waf=cands.get(tuple(v)))
                rows.append(rec)
                f.write(json.dumps(rec) + "\n"); f.flush()
            sp = [r for r in rows if r["role"] == "space" and r["status"] == 0]
            tfs = np.array([r["tflops"] for r in sp]); ppws = np.array([r["ppw"] for r in sp])

            def pct(x, arr):
                return float((arr < x).mean() * 100)

            dflt = next(r for r in rows if r["role"] == "default")
            eat = [r for r in rows if r["role"] == "eatss"]
            best = max(eat, key=lambda r: r["ppw"])
            pick = next((r for r in eat if r["waf"] == 16), best)
            summary[kind] = dict(
                n_space=len(sp), n_skipped=len(sample) - len(sp),
                median=dict(tflops=float(np.median(tfs)), ppw=float(np.median(ppws))),
                best_in_space=dict(tflops=float(tfs.max()), ppw=float(ppws.max())),
                P=dict(tiles=dflt["tiles"], tflops=dflt["tflops"], ppw=dflt["ppw"], pct_tflops=pct(dflt["tflops"], tfs),
                       pct_ppw=pct(dflt["ppw"], ppws)),
                U=dict(tiles=best["tiles"], tflops=best["tflops"], ppw=best["ppw"], pct_tflops=pct(best["tflops"], tfs),
                       pct_ppw=pct(best["ppw"], ppws)),
                eatss_waf16=dict(tiles=pick["tiles"], tflops=pick["tflops"], ppw=pick["ppw"],
                                 pct_tflops=pct(pick["tflops"], tfs), pct_ppw=pct(pick["ppw"], ppws)),
                U_over_P_ppw=best["ppw"] / dflt["ppw"], U_over_M_ppw=best["ppw"] / float(np.median(ppws)))
            print(kind, json.dumps(summary[kind]), flush=True)
            del bufs
            torch.cuda.empty_cache()
    with open(a.out.replace(".jsonl", ".summary.json"), "w") as f:
        json.dump(summary, f, indent=1)


if __name__ == "__main__":
    main()
