#!/usr/bin/env python
"""Tensor-core tile space sweep: does the energy-vs-performance finding hold
on the tensor pipe?

    python harness/tensor_sweep.py [--kinds gemm,2mm,syrk] [--repeats 5] [--window 1.0] [--out ts.jsonl]

The tcgen05 3xTF32 executor accepts the tiles Ti in {128 (one CTA), 256 (a CTA pair)}, Tj in
{16, 32, ..., 256} (UMMA N), Tk in {8, 16, 32, 64} (k per pipeline stage) that fit its shared memory;
reading T is the subset with Tk in {32, 64} (whole 128-byte swizzle atoms).
Every executable vector of gemm (2mm / syrk: the reading-T subset) at N = 4000 is measured with the
a9 protocol (eatss_sweep:
warm-up, >= --window s of back-to-back runs, NVML energy counter) in --repeats interleaved
rounds, so DVFS and thermal drift hit every variant alike; each variant is first checked for
exactness on small-integer inputs (sampled entries vs the fp64 oracle).  The summary gives per
kernel the performance-optimal and the PPW-optimal variant with 95% intervals, and whether they
differ beyond the noise -- the paper's finding is that the energy-optimal tile
beats the performance-optimal one on GFLOP/s/W.  The EATSS tensor-mode pick is marked.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

N = 4000
KINDS = {"gemm": (N, N, N), "2mm": (N, N, N, N), "syrk": (N, N)}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kinds", default="gemm")
    ap.add_argument("--repeats", type=int, default=5)
    ap.add_argument("--window", type=float, default=1.0)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--engine", type=int, choices=[2, 4], default=2,
                    help="2 = 3xTF32 (reading T mode 2), 4 = 3xFP16 (mode 3; Tk counts fp16 elements)")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "tensor_sweep.jsonl"))
    return ap.parse_args()


def exact_gemm(E, torch, tiles, engine=2):
    """Small-integer gemm through the tensor engine: 512 sampled entries equal the fp64 oracle."""
    import synth
    from oracle import numeric as O

    n = N
    d = E.desc_builtin("gemm", (n, n, n))
    d.set_scalars(1.0, 1.0)
    d.set_exec(split_pct=50, engine=engine)
    Ah, Bh, Ch = synth.small_int((n, n), 1), synth.small_int((n, n), 2), synth.small_int((n, n), 3)
    C = torch.from_numpy(Ch).cuda()
    E.run(d, tiles, [C, torch.from_numpy(Ah).cuda(), torch.from_numpy(Bh).cuda()])
    g = synth.rng(7)
    ii, jj = g.integers(0, n, 512), g.integers(0, n, 512)
    got = C[torch.from_numpy(ii).cuda(), torch.from_numpy(jj).cuda()].double().cpu().numpy()
    return bool(np.array_equal(got, O.gemm_entries(ii, jj, Ch, Ah, Bh, 1.0, 1.0)))


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
            d.set_exec(split_pct=50, engine=a.engine)
            mode = 2 if a.engine == 2 else 3
            pick, _ = E.select_tiles(d, gpu, split_pct=50, waf=16, mode=mode)
            tks = (8, 16, 32, 64) if a.engine == 2 else (16, 32, 64, 128)  # 32 .. 256 bytes of k per stage row
            tk_t = 32 if a.engine == 2 else 64                               # reading T: whole 128-byte atoms
            space = [(ti, tj, tk) for ti in (128, 256) for tj in range(16, 257, 16) for tk in tks]
            if kind != "gemm":
                space = [v for v in space if v[2] >= tk_t]
            nl = 2 if a.engine == 2 else 3  # launches per nest on the engine: executable there
            variants = [v for v in space if E.launches_per_run(d, v) == nl]
            gen = torch.Generator(device="cuda").manual_seed(0)
            bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=gen) * 2 - 1 for i in range(d.num_buffers)]
            exact = {v: exact_gemm(E, torch, v, a.engine) for v in variants} if kind == "gemm" else {}
            ppw = {v: [] for v in variants}
            tf = {v: [] for v in variants}
            watts = {v: [] for v in variants}
            for rep in range(a.repeats):
                order = variants if rep % 2 == 0 else variants[::-1]
                for v in order:
                    m = E.sweep(d, [v], bufs, device=0, warmup=a.warmup, min_window_s=a.window)[0]
                    rec = dict(kind=kind, tiles=list(v), rep=rep, ms=m.ms_per_run, tflops=m.tflops,
                               watts=m.avg_watts, ppw=m.gflops_per_watt, joules=m.joules_per_run,
                               sm_mhz=m.sm_mhz_median, status=m.status, eatss_pick=tuple(v) == tuple(pick),
                               reading_t=v[2] >= tk_t, exact=exact.get(v), engine=a.engine)
                    f.write(json.dumps(rec) + "\n"); f.flush()
                    if m.status == 0 and m.gflops_per_watt > 0:
                        ppw[v].append(m.gflops_per_watt); tf[v].append(m.tflops); watts[v].append(m.avg_watts)

            def stats(x):
                x = np.array(x)
                h = 1.96 * x.std(ddof=1) / np.sqrt(len(x)) if len(x) > 1 else float("nan")
                return float(x.mean()), [float(x.mean() - h), float(x.mean() + h)]

            rows = {v: dict(ppw=stats(ppw[v]), tflops=stats(tf[v]), watts=float(np.mean(watts[v]))) for v in variants
                    if ppw[v]}
            perf = max(rows, key=lambda v: rows[v]["tflops"][0])
            eff = max(rows, key=lambda v: rows[v]["ppw"][0])
            s = dict(engine=a.engine, eatss_pick=list(pick), n_variants=len(rows), perf_optimal=dict(tiles=list(perf), **rows[perf]),
                     ppw_optimal=dict(tiles=list(eff), **rows[eff]),
                     distinct=perf != eff,
                     separated=perf != eff and rows[eff]["ppw"][1][0] > rows[perf]["ppw"][1][1],
                     all={str(list(v)): r for v, r in rows.items()},
                     exact_all=all(exact.values()) if exact else None)
            summary[kind] = s
            print(kind, json.dumps({k: s[k] for k in ("eatss_pick", "perf_optimal", "ppw_optimal", "distinct",
                                                      "separated", "exact_all")}), flush=True)
    with open(a.out.replace(".jsonl", ".summary.json"), "w") as f:
        json.dump(summary, f, indent=1)


if __name__ == "__main__":
    main()
