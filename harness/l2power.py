#!/usr/bin/env python
"""L2 read-sector traffic vs average power over tile variants (paper Fig. 9).

The paper grounds its model in the observation that, across tile variants, a BLAS3 kernel's
power tracks its L2 read traffic -- Pearson r = 0.85 (2mm) and 0.75 (gemm) between the
`lts__t_sectors_srcunit_tex_op_read` count and power -- while jacobi-2d shows no such
correlation (Fig. 9: '0.85 and 0.75 for 2mm and gemm, respectively').  This harness repeats that on B200 with the SIMT executor family:

  1. ``--phase power``: for a seeded sample of tile variants (the 15-per-dimension space of
     harness/sweep.py, reading Q19), measure time and average power with eatss_sweep
     (warm-up, >= --window s of back-to-back runs, NVML energy counter);
  2. ``--phase l2`` (run under ncu, one launch per variant and nest):
        ncu --metrics lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_op_read.sum,gpu__time_duration.sum \
            -k regex:'contract|jacobi2d|lowdim_kernel' --csv --log-file l2.csv python harness/l2power.py --phase l2 ...
  3. ``--phase report``: join both, Pearson r of power vs L2 read sectors per second (and per run).

Power comes only from phase 1 (ncu serialises and replays kernels, so it never measures time
or power here).  Inputs are U[-1,1) on the device.
"""
from __future__ import annotations

import argparse
import csv
import itertools
import json
import os
import random
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SIZES = [4, 8, 16, 24, 32, 48, 64, 96, 128, 192, 256, 384, 512, 768, 1024]
KINDS = {"gemm": ((4000, 4000, 4000), 0), "2mm": ((4000, 4000, 4000, 4000), 0), "jacobi-2d": ((4000,), 1),
         "mvt": ((4000,), 0)}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--phase", choices=["power", "l2", "report"], required=True)
    ap.add_argument("--kinds", default="gemm,2mm,jacobi-2d,mvt")
    ap.add_argument("--count", type=int, default=120, help="variants per kind (jacobi-2d: at most 225)")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--window", type=float, default=0.5)
    ap.add_argument("--max-ms", type=float, default=60.0, help="skip variants slower than this (ms per run)")
    ap.add_argument("--power", default=os.path.join(ROOT, "gpurun_out", "l2power_power.jsonl"))
    ap.add_argument("--l2csv", default=os.path.join(ROOT, "gpurun_out", "l2power_l2.csv"))
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "l2power_summary.json"))
    return ap.parse_args()


def variants(kind, count, seed):
    dims, _ = KINDS[kind]
    depth = 2 if kind in ("jacobi-2d", "mvt") else 3
    space = list(itertools.product(SIZES, repeat=depth))
    random.Random(seed).shuffle(space)
    return space[: min(count, len(space))]


def nest_kernels(kind):
    """Kernel launches matched by the ncu filter per run of one variant."""
    return {"gemm": 1, "2mm": 2, "jacobi-2d": 1, "mvt": 1}[kind]


def make(E, torch, kind):
    dims, tsteps = KINDS[kind]
    d = E.desc_builtin(kind, dims, tsteps=tsteps)
    d.set_exec(split_pct=50, engine=1, use_graph=0)
    g = torch.Generator(device="cuda").manual_seed(0)
    bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=g) * 2 - 1 for i in range(d.num_buffers)]
    return d, bufs


def phase_power(a):
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    os.makedirs(os.path.dirname(a.power), exist_ok=True)
    with open(a.power, "w") as f:
        for kind in a.kinds.split(","):
            d, bufs = make(E, torch, kind)
            for v in variants(kind, a.count, a.seed):
                # cheap pre-timing: skip pathological variants (e.g. 4x4 tiles of gemm take seconds)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record(); E.run(d, v, bufs); e.record(); torch.cuda.synchronize()
                if s.elapsed_time(e) > a.max_ms:
                    f.write(json.dumps(dict(kind=kind, tiles=list(v), skipped=True)) + "\n")
                    continue
                m = E.sweep(d, [v], bufs, warmup=1, min_window_s=a.window)[0]
                f.write(json.dumps(dict(kind=kind, tiles=list(v), ms=m.ms_per_run, watts=m.avg_watts,
                                        ppw=m.gflops_per_watt, tflops=m.tflops, sm_mhz=m.sm_mhz_median,
                                        status=m.status)) + "\n")
                f.flush()
            del bufs
            torch.cuda.empty_cache()


def phase_l2(a):
    """One run per measured variant, in file order (ncu counts the sectors of each launch)."""
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    recs = [json.loads(x) for x in open(a.power)]
    for kind in a.kinds.split(","):
        d, bufs = make(E, torch, kind)
        for r in recs:
            if r["kind"] == kind and not r.get("skipped"):
                E.run(d, r["tiles"], bufs)
        torch.cuda.synchronize()
        del bufs
        torch.cuda.empty_cache()


def pearson(x, y):
    x, y = np.asarray(x, float), np.asarray(y, float)
    if len(x) < 3 or x.std() == 0 or y.std() == 0:
        return None
    return float(np.corrcoef(x, y)[0, 1])


def phase_report(a):
    recs = [json.loads(x) for x in open(a.power)]
    rows = list(csv.reader(open(a.l2csv)))
    hdr = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hdr]
    per_id = {}
    for r in rows[hdr + 1:]:
        if len(r) != len(h):
            continue
        d = dict(zip(h, r))
        v = float(d["Metric Value"].replace(",", ""))
        unit = d["Metric Unit"]
        if d["Metric Name"] == "gpu__time_duration.sum":
            v *= {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3}.get(unit, 1.0)
        per_id.setdefault(int(d["ID"]), {})[d["Metric Name"]] = v
    launches = [per_id[i] for i in sorted(per_id)]
    out, pos = {}, 0
    for kind in a.kinds.split(","):
        k = nest_kernels(kind)
        pts = []
        for r in recs:
            if r["kind"] != kind or r.get("skipped"):
                continue
            ls = launches[pos: pos + k]
            pos += k
            if r.get("status", 0) != 0 or r["watts"] <= 0:
                continue
            sectors = sum(x.get("lts__t_sectors_srcunit_tex_op_read.sum", 0.0) for x in ls)
            allrd = sum(x.get("lts__t_sectors_op_read.sum", 0.0) for x in ls)
            pts.append((r["watts"], sectors, sectors / (r["ms"] * 1e-3), r["tiles"], r["ppw"], allrd / (r["ms"] * 1e-3)))
        if not pts:
            continue
        w = [p[0] for p in pts]
        out[kind] = dict(n=len(pts), r_power_vs_sectors_per_s=pearson(w, [p[2] for p in pts]),
                         r_power_vs_sectors_per_run=pearson(w, [p[1] for p in pts]),
                         r_power_vs_all_l2_read_sectors_per_s=pearson(w, [p[5] for p in pts]),
                         watts_range=[min(w), max(w)],
                         paper_r={"gemm": 0.75, "2mm": 0.85, "jacobi-2d": "no correlation", "mvt": "no correlation"}.get(kind))
    out["launches_parsed"] = len(launches)
    out["launches_used"] = pos
    json.dump(out, open(a.out, "w"), indent=1)
    print(json.dumps(out, indent=1))


def main():
    a = parse()
    {"power": phase_power, "l2": phase_l2, "report": phase_report}[a.phase](a)


if __name__ == "__main__":
    main()
