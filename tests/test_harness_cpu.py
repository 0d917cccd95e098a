"""Host logic of the measurement harness on synthetic records:
harness/report.py must pick the performance- and energy-optimal variants, rank the EATSS tile, use
the anchor spread as the noise bar for the paper's finding, drift-correct by the
interpolated EATSS anchor, and give Student-t intervals for confirmation repeats.  No GPU."""
import json
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "harness"))

import report  # noqa: E402


def _write(tmp_path, rows):
    p = tmp_path / "sweep.jsonl"
    with open(p, "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    return str(p)


def _variant(tile, tflops, watts, t, exact=True, status=0):
    ms = 2 * 4000 ** 3 / (tflops * 1e12) * 1e3
    joules = watts * ms * 1e-3
    return {"kind": "variant", "tile": list(tile), "tflops": tflops, "watts": watts, "ms": ms, "joules": joules,
            "gflops_per_watt": tflops * 1e3 / watts, "status": status, "exact": exact, "t": t}


def _anchor(kind, tile, tflops, watts, t):
    r = _variant(tile, tflops, watts, t)
    r["kind"] = kind
    return r


def test_report_finds_optima_ranks_and_noise(tmp_path):
    rows = [{"kind": "meta", "eatss_tile": [16, 1024, 16], "nvml_update_ms": 100.0}]
    rows += [_variant((16, 1024, 16), 36.0, 700.0, 1.0),      # EATSS pick
             _variant((32, 512, 48), 40.0, 760.0, 2.0),       # fastest
             _variant((64, 256, 128), 38.0, 640.0, 3.0),      # lowest energy per run: PPW 59.4 > 52.6
             _variant((32, 32, 32), 7.0, 500.0, 4.0),         # default class
             _variant((4, 4, 4), 99.0, 100.0, 5.0, exact=False),  # inexact: never ranked
             _variant((8, 8, 8), 99.0, 100.0, 6.0, status=-3)]    # failed: never ranked
    rows += [_anchor("anchor_default", (32, 32, 32), 7.0, 500.0, t) for t in (0.5, 3.5)]
    rows += [_anchor("anchor_eatss", (16, 1024, 16), x, 700.0, t) for x, t in ((36.0, 0.5), (35.0, 6.5))]
    s = report.summarise(_write(tmp_path, rows))
    assert s["variants"] == 6 and s["measured_ok"] == 4 and s["inexact"] == 1
    assert s["perf_optimal"]["tile"] == [32, 512, 48]
    assert s["energy_optimal"]["tile"] == [64, 256, 128]
    assert s["energy_optimal_differs"]
    gain = (38.0 / 640.0) / (40.0 / 760.0)
    assert s["ppw_gain_energy_vs_perf_optimal"] == pytest.approx(gain)
    # EATSS anchor spread (36 vs 35 TF at equal power) is the noise bar; the 12.8% gain clears it
    assert s["ppw_noise_rel"] == pytest.approx((36.0 - 35.0) / (35.5), rel=1e-6)
    assert s["finding_energy_beats_perf_on_ppw"]
    assert s["eatss_rank_perf"] == 3 and s["eatss_rank_ppw"] == 3
    assert s["share_beating_default_perf"] == pytest.approx(0.75)
    assert "drift_corrected" in s and len(s["top5_ppw"]) == 4


def test_report_drift_correction_uses_interpolated_anchor(tmp_path):
    # the EATSS anchor drifts linearly 40 -> 20 TF over the run; a variant measured mid-run at 30 TF
    # is as fast as the anchor median (30): drift-corrected it equals 30
    rows = [{"kind": "meta", "eatss_tile": [16, 1024, 16]}]
    rows += [_anchor("anchor_eatss", (16, 1024, 16), x, 500.0, t) for x, t in ((40.0, 0.0), (30.0, 5.0), (20.0, 10.0))]
    rows += [_variant((32, 512, 48), 30.0, 500.0, 5.0), _variant((64, 64, 64), 25.0, 500.0, 9.0)]
    s = report.summarise(_write(tmp_path, rows))
    dc = s["drift_corrected"]
    # (64,64,64) at t=9 ran while the anchor was at 22: corrected 25 * 30 / 22 = 34.1 > 30
    assert dc["perf_optimal"]["tile"] == [64, 64, 64]
    assert dc["perf_optimal"]["tflops"] == pytest.approx(25.0 * 30.0 / 22.0)


def test_confirm_summary_student_t_and_separation(tmp_path):
    rows = []
    g = np.random.default_rng(0)
    for tile, ppw_mu, tf_mu in (((32, 512, 48), 53.7, 35.0), ((48, 256, 48), 52.9, 33.0)):
        for _ in range(7):
            ppw = ppw_mu + g.normal(0, 0.2)
            tf = tf_mu + g.normal(0, 0.1)
            rows.append({"kind": "confirm", "tile": list(tile), "gflops_per_watt": ppw, "tflops": tf,
                         "watts": tf * 1e3 / ppw, "joules": 1.0, "status": 0})
    s = report.confirm_summary(_write(tmp_path, rows))
    assert s["energy_optimal"] == [32, 512, 48] and s["perf_optimal"] == [32, 512, 48]
    assert not s["finding_energy_beats_perf_on_ppw_ci_separated"]  # same tile: no split to confirm
    t = s["tiles"][0]
    assert t["n"] == 7
    lo, hi = t["gflops_per_watt"]["ci95"]
    assert lo < t["gflops_per_watt"]["mean"] < hi and hi - lo < 1.0
