#!/usr/bin/env python
"""EATSS candidate protocol across shared-memory splits and warp fractions.

    python harness/candidates.py [--kinds gemm,2mm,...] [--window 0.6] [--out cand.jsonl]

The paper does not use one EATSS tile per kernel: it generates candidates over the L1/shared
split (SPLIT_FACTOR; "three configurations", "0%, 50% or 67%, and 100%")
and the warp fraction (WARP_ALIGNMENT_FACTOR = warp_frac * 32, "as small as 4"),
runs each candidate with the matching carve-out, and keeps the best measured PPW (Figs. 8, 10).
This harness does that on B200 with the library's own model (B200 mode, mode = 1) and the SIMT
executor family the sweep uses (engine = SIMT; the paper's code class):

  * candidates: sigma in {0, 50, 100} % (reading Q17) x WAF in {4, 8, 16, 32}; infeasible
    pairs are recorded (e.g. heat-3d at WAF 32; the 6-D contraction at WAF >= 8);
  * each distinct (tile, sigma, WAF) is measured with eatss_sweep (warm-up, then back-to-back runs
    for >= --window s, CUDA-event time, NVML energy counter) at carve-out sigma requested
    EXACTLY (exec.carveout_exact; the carve-out each run requested is recorded from
    eatss_last_carveout) and, for the gemm family, with WAF lanes of every warp along l_s1
    (exec.warp_align: the executor's SIMT length);
  * baseline: PPCG's default tile (32 per tiled loop) at the same three carve-outs.

The summary gives, per kernel, the best candidate's PPW (GFLOP/s/W = FLOP/J) over
the best default's PPW -- the quantity behind the paper's "median 1.5x / 1.2x, peak 6.3x" PPW
gains over PPCG (context only: other GPUs, other code generator).
Inputs are U[-1,1) on the device (energy must be measured on random data).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SPLITS = (0, 50, 100)
WAFS = (4, 8, 16, 32)
# BASELINE.json configs (reading Q22 sizes)
KINDS = {
    "gemm": dict(dims=(4000, 4000, 4000)),
    "2mm": dict(dims=(4000, 4000, 4000, 4000)),
    "3mm": dict(dims=(4000, 4000, 4000, 4000, 4000)),
    "syrk": dict(dims=(4000, 4000)),
    "jacobi-2d": dict(dims=(4000,), tsteps=500),
    "heat-3d": dict(dims=(120,), tsteps=500),
    "ccsd_t_d1": dict(dims=(48,)),
    # low-dimensional PolyBench kernels (PolyBench EXTRALARGE-like n = 4000)
    "mvt": dict(dims=(4000,)),
    "atax": dict(dims=(4000, 4000)),
    "bicg": dict(dims=(4000, 4000)),
    "gemver": dict(dims=(4000,)),
    # non-PolyBench 4-D kernels of Figs. 10-11 (readings R-N8, R-N9: our sizes)
    "mttkrp": dict(dims=(512, 32, 512, 512)),
    "conv-2d": dict(dims=(8192, 5)),
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kinds", default=",".join(KINDS))
    ap.add_argument("--window", type=float, default=0.6)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--device", type=int, default=0)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "candidates.jsonl"))
    ap.add_argument("--confirm", type=int, default=5,
                    help="when the PPW-best and the fastest candidate differ, re-measure both this many "
                         "times, interleaved, and report mean and 95%% interval of the PPW (0 = off)")
    return ap.parse_args()


CONTRACTIONS = ("gemm", "2mm", "3mm", "syrk")


def candidates(E, d, gpu):
    """{(tile, sigma, waf): [(sigma, waf, obj), ...]} plus the infeasible (sigma, waf) pairs; the WAF is
    part of the key only where the executor honours it (the gemm family)."""
    out, infeasible = {}, []
    for s in SPLITS:
        for w in WAFS:
            try:
                t, rep = E.select_tiles(d, gpu, split_pct=s, waf=w, mode=1)
            except E.EatssError as e:
                if e.status != -2:
                    raise
                infeasible.append((s, w))
                continue
            out.setdefault((tuple(t), s, w if d.kind in CONTRACTIONS else 0), []).append((s, w, int(rep.obj)))
    return out, infeasible


def measure(E, d, tiles, split, bufs, a, waf=0):
    d.set_exec(split_pct=split, engine=1, warp_align=waf, carveout_exact=1)
    m = E.sweep(d, [tiles], bufs, device=a.device, warmup=a.warmup, min_window_s=a.window)[0]
    try:
        cv = E.last_carveout(d)
    except E.EatssError:
        cv = None
    return dict(ms=m.ms_per_run, joules=m.joules_per_run, watts=m.avg_watts, tflops=m.tflops,
                ppw=m.gflops_per_watt, sm_mhz=m.sm_mhz_median, status=m.status, carveout_requested=cv)


def confirm(E, d, bufs, a, cands):
    """Interleaved repeats of the given candidates (DVFS / thermal drift hits both alike)."""
    import numpy as np

    ppw = {i: [] for i in range(len(cands))}
    tf = {i: [] for i in range(len(cands))}
    for _ in range(a.confirm):
        for i, c in enumerate(cands):
            r = measure(E, d, tuple(c["tiles"]), c["split"], bufs, a, c.get("waf", 0))
            if r["status"] == 0 and r["ppw"] > 0:
                ppw[i].append(r["ppw"]); tf[i].append(r["tflops"])
    out = []
    for i, c in enumerate(cands):
        x = np.array(ppw[i]); t = np.array(tf[i])
        half = 1.96 * x.std(ddof=1) / np.sqrt(len(x)) if len(x) > 1 else float("nan")
        out.append(dict(tiles=c["tiles"], split=c["split"], role="ppw-best" if i == 0 else "fastest",
                        ppw_mean=float(x.mean()) if len(x) else None, ppw_ci95=[float(x.mean() - half), float(x.mean() + half)]
                        if len(x) > 1 else None, tflops_mean=float(t.mean()) if len(t) else None, n=len(x)))
    lo0, hi1 = (out[0]["ppw_ci95"] or [None])[0], (out[1]["ppw_ci95"] or [None, None])[1]
    return dict(repeats=out, ppw_best_separated=(lo0 is not None and hi1 is not None and lo0 > hi1))


def main():
    a = parse()
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    torch.cuda.set_device(a.device)
    gpu = E.gpu_params_query(a.device)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    summary = {}
    with open(a.out, "a") as f:
        for kind in a.kinds.split(","):
            cfg = KINDS[kind]
            d = E.desc_builtin(kind, cfg["dims"], tsteps=cfg.get("tsteps", 0))
            gen = torch.Generator(device="cuda").manual_seed(0)
            bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=gen) * 2 - 1 for i in range(d.num_buffers)]
            cands, infeasible = candidates(E, d, gpu)
            default = tuple([32] * d.num_loops)
            rows = []
            for (tiles, s, w), origin in sorted(cands.items(), key=lambda kv: (kv[0][1], kv[0][2], kv[0][0])):
                r = measure(E, d, tiles, s, bufs, a, w)
                rec = dict(kind=kind, role="eatss", tiles=list(tiles), split=s, waf=w, origin=origin, **r)
                rows.append(rec)
                f.write(json.dumps(rec) + "\n"); f.flush()
            for s in SPLITS:
                r = measure(E, d, default, s, bufs, a)
                rec = dict(kind=kind, role="default", tiles=list(default), split=s, **r)
                rows.append(rec)
                f.write(json.dumps(rec) + "\n"); f.flush()
            ok = [r for r in rows if r["status"] == 0 and r["ppw"] > 0]
            ea = [r for r in ok if r["role"] == "eatss"]
            de = [r for r in ok if r["role"] == "default"]
            if ea:
                be = max(ea, key=lambda r: r["ppw"])
                pe = max(ea, key=lambda r: r["tflops"])
                bd = max(de, key=lambda r: r["ppw"]) if de else None
                summary[kind] = dict(
                    best_candidate=dict(tiles=be["tiles"], split=be["split"], waf=be["waf"], origin=be["origin"],
                                        ppw=be["ppw"], tflops=be["tflops"], watts=be["watts"]),
                    fastest_candidate=dict(tiles=pe["tiles"], split=pe["split"], ppw=pe["ppw"], tflops=pe["tflops"]),
                    best_default=(dict(split=bd["split"], ppw=bd["ppw"], tflops=bd["tflops"], watts=bd["watts"])
                                  if bd else "default tile not executable (launch configuration rejected)"),
                    ppw_gain_vs_default=be["ppw"] / bd["ppw"] if bd else None,
                    ppw_spread_over_candidates=be["ppw"] / min(r["ppw"] for r in ea),
                    n_candidates=len(ea), infeasible=infeasible)
            if ea and a.confirm > 0:
                be = max(ea, key=lambda r: r["ppw"]); pe = max(ea, key=lambda r: r["tflops"])
                if (be["tiles"], be["split"], be["waf"]) != (pe["tiles"], pe["split"], pe["waf"]):
                    summary[kind]["confirm"] = confirm(E, d, bufs, a, [be, pe])
            print(kind, json.dumps(summary.get(kind)), flush=True)
            del bufs
            torch.cuda.empty_cache()
    with open(a.out.replace(".jsonl", ".summary.json"), "w") as g:
        json.dump(dict(created=time.time(), window_s=a.window, splits=SPLITS, wafs=WAFS, kinds=summary), g, indent=1)


if __name__ == "__main__":
    main()
