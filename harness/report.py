#!/usr/bin/env python
"""Summarise a sweep JSONL (harness/sweep.py): performance- vs energy-optimal tiles.

    python harness/report.py run.jsonl [--json out.json]

Reports (P:225 energy = P_avg * t; P:231-234 PPW = FLOP/s / W = FLOP/J):
  * the performance-optimal variant (max TFLOP/s) and the energy-optimal one (min J/run
    == max GFLOP/s/W) among variants that passed the exactness check;
  * whether they differ and by how much PPW differs, against the anchor-estimated noise
    (spread of the repeated default / EATSS anchors);
  * where the EATSS pick and the default 32^3 tile rank, and the share of variants that
    beat the default (the paper: 15% for gemm on GA100).
"""
import argparse
import json
import statistics

import numpy as np


def load(path):
    """Records of a sweep JSONL; a tile measured again later (sweep.py --only) keeps its LAST record."""
    meta, var, anc = None, {}, {"anchor_default": [], "anchor_eatss": []}
    for line in open(path):
        r = json.loads(line)
        k = r.get("kind")
        if k == "meta":
            meta = meta or r
        elif k == "variant":
            var[(tuple(r["tile"]), r.get("rank", 0))] = r
        elif k in anc:
            anc[k].append(r)
    return meta, list(var.values()), anc


def summarise(path):
    meta, var, anc = load(path)
    ok = [r for r in var if r.get("status") == 0 and r.get("exact", True) and (r.get("joules") or 0) > 0]
    bad = [r for r in var if not r.get("exact", True)]
    out = {"file": path, "variants": len(var), "measured_ok": len(ok), "inexact": len(bad),
           "eatss_tile": meta.get("eatss_tile") if meta else None, "nvml_update_ms": meta.get("nvml_update_ms") if meta else None}
    if not ok:
        return out
    perf = max(ok, key=lambda r: r["tflops"])
    energy = min(ok, key=lambda r: r["joules"])
    ppw = sorted(ok, key=lambda r: -r["gflops_per_watt"])
    out["perf_optimal"] = {k: perf[k] for k in ("tile", "tflops", "joules", "watts", "gflops_per_watt", "ms")}
    out["energy_optimal"] = {k: energy[k] for k in ("tile", "tflops", "joules", "watts", "gflops_per_watt", "ms")}
    out["energy_optimal_differs"] = perf["tile"] != energy["tile"]
    out["ppw_gain_energy_vs_perf_optimal"] = energy["gflops_per_watt"] / perf["gflops_per_watt"]
    for name, key in (("default", "anchor_default"), ("eatss", "anchor_eatss")):
        a = [r for r in anc[key] if r.get("status") == 0 and (r.get("joules") or 0) > 0]
        if a:
            p = [r["gflops_per_watt"] for r in a]
            t = [r["tflops"] for r in a]
            out[f"anchor_{name}"] = {"tile": a[0]["tile"], "n": len(a), "ppw_median": statistics.median(p),
                                     "ppw_rel_spread": (max(p) - min(p)) / statistics.median(p),
                                     "tflops_median": statistics.median(t),
                                     "tflops_rel_spread": (max(t) - min(t)) / statistics.median(t)}
    noise = max([out.get(f"anchor_{n}", {}).get("ppw_rel_spread", 0) for n in ("default", "eatss")] or [0])
    out["ppw_noise_rel"] = noise
    out["finding_energy_beats_perf_on_ppw"] = bool(out["energy_optimal_differs"] and
                                                   out["ppw_gain_energy_vs_perf_optimal"] - 1 > noise)
    tiles_by_ppw = [tuple(r["tile"]) for r in ppw]
    tiles_by_perf = [tuple(r["tile"]) for r in sorted(ok, key=lambda r: -r["tflops"])]
    for name, key in (("eatss", "eatss_tile"),):
        t = tuple(meta.get(key) or ())
        if t in tiles_by_ppw:
            out[f"{name}_rank_ppw"] = tiles_by_ppw.index(t) + 1
            out[f"{name}_rank_perf"] = tiles_by_perf.index(t) + 1
    d = out.get("anchor_default")
    if d:
        out["share_beating_default_perf"] = float(np.mean([r["tflops"] > d["tflops_median"] for r in ok]))
        out["share_beating_default_ppw"] = float(np.mean([r["gflops_per_watt"] > d["ppw_median"] for r in ok]))
    # drift correction: scale each variant's PPW / TFLOP/s by the EATSS anchor interpolated at its
    # measurement time (DVFS / thermal drift over the ~50 min sweep) -- on the variant's OWN GPU when the
    # sweep ran on several (per-GPU anchor normalisation: GPUs differ in clocks, power and drift)
    ae_all = [r for r in anc["anchor_eatss"] if r.get("status") == 0 and (r.get("joules") or 0) > 0]
    ranks = sorted({r.get("rank", 0) for r in ae_all})
    per_rank = {}
    for rk in ranks:
        ae = sorted([r for r in ae_all if r.get("rank", 0) == rk], key=lambda r: r["t"])
        if len(ae) >= 2:
            per_rank[rk] = (np.array([r["t"] for r in ae]), np.array([r["gflops_per_watt"] for r in ae]),
                            np.array([r["tflops"] for r in ae]))
    if per_rank:
        p_med = float(np.median([r["gflops_per_watt"] for r in ae_all]))
        t_med = float(np.median([r["tflops"] for r in ae_all]))
        corr = [r for r in ok if r.get("rank", 0) in per_rank]
        for r in corr:
            ts, pp, tf = per_rank[r.get("rank", 0)]
            r["ppw_drift_corr"] = r["gflops_per_watt"] * p_med / float(np.interp(r["t"], ts, pp))
            r["tflops_drift_corr"] = r["tflops"] * t_med / float(np.interp(r["t"], ts, tf))
        perf_c = max(corr, key=lambda r: r["tflops_drift_corr"])
        ener_c = max(corr, key=lambda r: r["ppw_drift_corr"])
        out["drift_corrected"] = {
            "per_gpu_anchors": {str(k): int(len(v[0])) for k, v in per_rank.items()},
            "perf_optimal": {"tile": perf_c["tile"], "tflops": perf_c["tflops_drift_corr"], "ppw": perf_c["ppw_drift_corr"]},
            "energy_optimal": {"tile": ener_c["tile"], "tflops": ener_c["tflops_drift_corr"], "ppw": ener_c["ppw_drift_corr"]},
            "ppw_gain": ener_c["ppw_drift_corr"] / perf_c["ppw_drift_corr"],
            "top10_ppw": [r["tile"] for r in sorted(corr, key=lambda r: -r["ppw_drift_corr"])[:10]],
            "top10_perf": [r["tile"] for r in sorted(corr, key=lambda r: -r["tflops_drift_corr"])[:10]],
        }
    out["top5_ppw"] = [{"tile": r["tile"], "gflops_per_watt": r["gflops_per_watt"], "tflops": r["tflops"],
                        "watts": r["watts"]} for r in ppw[:5]]
    out["top5_perf"] = [{"tile": r["tile"], "gflops_per_watt": r["gflops_per_watt"], "tflops": r["tflops"],
                         "watts": r["watts"]} for r in sorted(ok, key=lambda r: -r["tflops"])[:5]]
    return out


T975 = {2: 12.71, 3: 4.30, 4: 3.18, 5: 2.78, 6: 2.57, 7: 2.45, 8: 2.36, 9: 2.31, 10: 2.26}


def confirm_summary(path):
    """Per-tile mean and 95% CI (Student t) of repeated interleaved measurements."""
    by = {}
    for line in open(path):
        r = json.loads(line)
        if r.get("kind") == "confirm" and r.get("status") == 0 and (r.get("joules") or 0) > 0:
            by.setdefault(tuple(r["tile"]), []).append(r)
    rows = []
    for tile, rs in by.items():
        n = len(rs)
        stats = {"tile": list(tile), "n": n}
        for key in ("gflops_per_watt", "tflops", "watts"):
            v = np.array([r[key] for r in rs])
            half = T975.get(n, 1.96) * v.std(ddof=1) / np.sqrt(n) if n > 1 else float("nan")
            stats[key] = {"mean": float(v.mean()), "ci95": [float(v.mean() - half), float(v.mean() + half)]}
        rows.append(stats)
    rows.sort(key=lambda s: -s["gflops_per_watt"]["mean"])
    if not rows:
        return {"file": path, "tiles": []}
    best_ppw = rows[0]
    best_perf = max(rows, key=lambda s: s["tflops"]["mean"])
    sep = best_ppw["gflops_per_watt"]["ci95"][0] > best_perf["gflops_per_watt"]["ci95"][1]
    return {"file": path, "energy_optimal": best_ppw["tile"], "perf_optimal": best_perf["tile"],
            "ppw_energy_opt": best_ppw["gflops_per_watt"], "ppw_perf_opt": best_perf["gflops_per_watt"],
            "tflops_energy_opt": best_ppw["tflops"], "tflops_perf_opt": best_perf["tflops"],
            "finding_energy_beats_perf_on_ppw_ci_separated": bool(best_ppw["tile"] != best_perf["tile"] and sep),
            "tiles": rows}


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("path")
    ap.add_argument("--json", default="")
    ap.add_argument("--confirm", action="store_true")
    a = ap.parse_args()
    s = confirm_summary(a.path) if a.confirm else summarise(a.path)
    txt = json.dumps(s, indent=1)
    print(txt)
    if a.json:
        open(a.json, "w").write(txt)
