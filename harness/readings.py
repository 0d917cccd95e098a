#!/usr/bin/env python
"""Reading -> tile -> PPW: what the unpinned readings of the model text would cost on B200.

    python harness/readings.py [--repeats 7] [--window 1.0] [--out gpurun_out/readings.jsonl]

tests/golden/reading_table.json (written from oracle/model.py only) lists, for every alternative
reading of the ambiguous model text (Q6 H counting, Q7 2-D rule, Q12 B-set order,
Q16 tie-break, ...), the tile it picks for BASELINE configs 4-5 and the set of tiles tied at the
optimum.  The readings that some printed fact excludes (
tests/test_oracle_model.py) are not measured; for the rest, every distinct tile -- each reading's
pick and every tied optimum -- runs through the C ABI with the a9 protocol (eatss_sweep: warm-up, then
back-to-back runs for >= --window s metered by the NVML energy counter) in --repeats interleaved
rounds (order reversed every other round) on U[-1,1) inputs, so drift hits all tiles alike.  The summary
gives per config and reading: tile, GFLOP/s/W with a 95% interval, TFLOP/s, and the best tile in the tie
set -- i.e. how far each reading's choice is from the best choice the model could have made.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CONFIGS = {  # (kernel, waf) -> descriptor (BASELINE configs 4-5; reading Q22 sizes)
    ("jacobi-2d", 16): dict(kind="jacobi-2d", dims=(4000,), tsteps=500),
    ("heat-3d", 16): dict(kind="heat-3d", dims=(120,), tsteps=500),
    ("heat-3d", 8): dict(kind="heat-3d", dims=(120,), tsteps=500),
    ("heat-3d", 4): dict(kind="heat-3d", dims=(120,), tsteps=500),
    ("ccsd_t_d1", 4): dict(kind="ccsd_t_d1", dims=(48,), tsteps=0),
}
UNPINNED = ["R", "h_count=array", "h_count=ref", "rule2d=none", "rule2d=scaled", "bset=outer", "bset=ls1_inner",
            "tiebreak=lexmin", "tiebreak=lexmax"]


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--repeats", type=int, default=7)
    ap.add_argument("--window", type=float, default=1.0)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "readings.jsonl"))
    return ap.parse_args()


def main():
    a = parse()
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E

    table = json.load(open(os.path.join(ROOT, "tests", "golden", "reading_table.json")))["readings"]
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    summary = {}
    with open(a.out, "a") as f:
        for key, cfg in CONFIGS.items():
            picks = {}
            tiles = []
            for name in UNPINNED:
                t = next(x for x in table[name]["tiles"] if (x["kernel"], x["waf"]) == key)
                picks[name] = tuple(t["pick"])
                for tt in [t["pick"]] + t["ties"]:
                    if tuple(tt) not in tiles:
                        tiles.append(tuple(tt))
            d = E.desc_builtin(cfg["kind"], cfg["dims"], tsteps=cfg["tsteps"])
            d.set_exec(split_pct=50, engine=1)
            g = torch.Generator(device="cuda").manual_seed(0)
            bufs = [torch.rand(d.buffer_elems(i), device="cuda", generator=g) * 2 - 1 for i in range(d.num_buffers)]
            vals = {t: [] for t in tiles}
            for rep in range(a.repeats):
                for t in (tiles if rep % 2 == 0 else tiles[::-1]):
                    m = E.sweep(d, [t], bufs, device=0, warmup=a.warmup, min_window_s=a.window)[0]
                    rec = dict(kernel=key[0], waf=key[1], tiles=list(t), rep=rep, ms=m.ms_per_run, tflops=m.tflops,
                               watts=m.avg_watts, ppw=m.gflops_per_watt, sm_mhz=m.sm_mhz_median, status=m.status)
                    f.write(json.dumps(rec) + "\n"); f.flush()
                    if m.status == 0 and m.gflops_per_watt > 0:
                        vals[t].append((m.gflops_per_watt, m.tflops, m.avg_watts))

            def stats(t):
                x = np.array([v[0] for v in vals[t]])
                h = 1.96 * x.std(ddof=1) / np.sqrt(len(x)) if len(x) > 1 else float("nan")
                return dict(ppw=float(x.mean()), ci=[float(x.mean() - h), float(x.mean() + h)],
                            tflops=float(np.mean([v[1] for v in vals[t]])), watts=float(np.mean([v[2] for v in vals[t]])))

            st = {t: stats(t) for t in tiles if vals[t]}
            best = max(st, key=lambda t: st[t]["ppw"])
            rows = {}
            for name in UNPINNED:
                t = picks[name]
                rows[name] = dict(tiles=list(t), **st[t], vs_best=st[t]["ppw"] / st[best]["ppw"],
                                  separated_from_best=t != best and st[t]["ci"][1] < st[best]["ci"][0])
            summary[f"{key[0]} waf={key[1]}"] = dict(best=dict(tiles=list(best), **st[best]), readings=rows,
                                                    all={str(list(t)): s for t, s in st.items()})
            print(key, json.dumps(summary[f"{key[0]} waf={key[1]}"]["best"]), flush=True)
            del bufs
            torch.cuda.empty_cache()
    with open(a.out.replace(".jsonl", ".summary.json"), "w") as f:
        json.dump(summary, f, indent=1)


if __name__ == "__main__":
    main()
