#!/usr/bin/env python
"""Tile-space sweep with energy measurement (BASELINE config 2).

    python harness/sweep.py --kind gemm --n 4000 [--sizes 4,8,...] [--limit K] [--out run.jsonl]
    torchrun --nproc-per-node G harness/sweep.py ...     (variants round-robin over ranks)

For each tile vector of the space (15 sizes per dimension -> 3,375 variants for the
3-deep gemm nest; sizes = reading Q19) the variant is executed by
libeatss.so through ``eatss_sweep`` (warm-up, then back-to-back runs for a window of
>= --window seconds, CUDA-event time, NVML energy-counter delta, 10 ms power / clock
sampler), after an exactness check on small-integer inputs (sampled entries vs
the fp64 oracle -- every fp32 partial sum is an exact integer, so any tiling must match
bit for bit).  Variants run in a seeded random order with two anchors -- the default
PPCG tile 32^3 and the EATSS pick -- re-measured every --anchor-every variants
to track DVFS / thermal drift.  Records are appended to a JSONL file (resumable).

The summary reports the performance-optimal and energy-optimal variants, their PPW
(GFLOP/s/W = FLOP/J) and where the EATSS pick ranks -- the paper's finding
to reproduce is that the energy-optimal tiles beat the performance-optimal ones on
PPW.
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import random
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SIZES = [4, 8, 16, 24, 32, 48, 64, 96, 128, 192, 256, 384, 512, 768, 1024]


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kind", default="gemm")
    ap.add_argument("--n", type=int, default=4000)
    ap.add_argument("--sizes", default=",".join(map(str, SIZES)))
    ap.add_argument("--limit", type=int, default=0, help="measure only the first K variants (after shuffling)")
    ap.add_argument("--window", type=float, default=0.5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--anchor-every", type=int, default=50)
    ap.add_argument("--split", type=int, default=50)
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep_gemm.jsonl"))
    ap.add_argument("--resume", default="", help="existing JSONL whose variants are skipped")
    ap.add_argument("--no-parity", action="store_true")
    ap.add_argument("--tiles", default="", help="confirmation mode: 'a,b,c;d,e,f' measured --repeats times, interleaved")
    ap.add_argument("--repeats", type=int, default=5)
    ap.add_argument("--only", default="", help="re-measure just these variants ('a,b,c;d,e,f') as variant records "
                                               "(harness/report.py keeps the last record of a tile)")
    ap.add_argument("--dtype", choices=["f32", "f64"], default="f32",
                    help="f64: the paper's precision (P:117 FP_factor 2, P:202): model and executor in fp64")
    return ap.parse_args()


REC_FIELDS = ["ms", "joules", "watts", "tflops", "gflops_per_watt", "sm_mhz", "runs", "status", "t"]
REC_KINDS = {"variant": 0, "anchor_default": 1, "anchor_eatss": 2, "confirm": 3}


def gather_records(recs, rank, ws, dist, torch, device):
    """All ranks' sweep records on rank 0 (list of dicts; [] elsewhere): fixed-size float64 rows
    (kind, tile[3], exact, REC_FIELDS incl. the wall-clock time t) padded to the longest rank and
    gathered with all_gather_into_tensor -- the per-rank timestamps let harness/report.py normalise
    each variant by ITS GPU's interpolated EATSS anchor (GPUs differ in clocks, power and drift)."""
    rows = [[REC_KINDS[r["kind"]], *r["tile"], float(r.get("exact", 1)),
             *[float(r.get(f, -1) if r.get(f) is not None else -1) for f in REC_FIELDS]] for r in recs]
    width = 5 + len(REC_FIELDS)
    cnt = torch.tensor([len(rows)], device=device)
    dist.all_reduce(cnt, op=dist.ReduceOp.MAX)
    buf = torch.full((int(cnt.item()), width), float("nan"), dtype=torch.float64, device=device)
    if rows:
        buf[: len(rows)] = torch.tensor(rows, dtype=torch.float64, device=device)
    allb = torch.empty((ws * buf.shape[0], width), dtype=torch.float64, device=device)  # rank blocks, concatenated
    dist.all_gather_into_tensor(allb, buf)
    out = []
    if rank == 0:
        inv = {v: k for k, v in REC_KINDS.items()}
        for rr, block in enumerate(allb.reshape(ws, buf.shape[0], width).cpu().numpy()):
            for x in block:
                if np.isnan(x[0]):
                    continue
                r = {"kind": inv[int(x[0])], "tile": [int(v) for v in x[1:4]], "exact": bool(x[4]), "rank": rr}
                r.update({f: float(v) for f, v in zip(REC_FIELDS, x[5:])})
                r["status"] = int(r["status"])
                out.append(r)
    return out


def nvml_interval_ms(E, device, seconds=1.0):
    """Calibrate the NVML energy-counter update interval."""
    try:
        last = E.energy_mj(device)
    except Exception:
        return None
    changes, t0 = [], time.perf_counter()
    while time.perf_counter() - t0 < seconds:
        v = E.energy_mj(device)
        if v != last:
            changes.append(time.perf_counter())
            last = v
        time.sleep(0.0005)
    if len(changes) < 2:
        return None
    return float(np.median(np.diff(changes)) * 1e3)


def main():
    a = parse()
    import torch
    import torch.distributed as dist

    import paper_conf_cgo_jayaweerakwk24_b200 as E
    import synth
    from oracle import numeric as O

    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if ws > 1:
        dist.init_process_group("nccl", device_id=dev)

    n = a.n
    assert a.kind == "gemm", "the sweep driver covers the gemm nest (config 2)"
    d = E.desc_builtin("gemm", (n, n, n), a.dtype)
    d.set_exec(split_pct=a.split)
    gpu = E.gpu_params_query(local)
    tdt = torch.float64 if a.dtype == "f64" else torch.float32
    ndt = np.float64 if a.dtype == "f64" else np.float32
    eatss_tile, rep = E.select_tiles(d, gpu, a.split, 16)
    default_tile = (32, 32, 32)
    sizes = [int(x) for x in a.sizes.split(",")]
    variants = list(itertools.product(sizes, sizes, sizes))
    random.Random(a.seed).shuffle(variants)
    if a.limit:
        variants = variants[: a.limit]
    if a.only:
        variants = [tuple(int(x) for x in t.split(",")) for t in a.only.split(";") if t]
    done = set()
    if a.resume and os.path.exists(a.resume):
        for line in open(a.resume):
            r = json.loads(line)
            if r.get("kind") == "variant":
                done.add(tuple(r["tile"]))
    mine = [v for i, v in enumerate(variants) if i % ws == rank and v not in done]

    # inputs: U(0..2) for energy/speed (data-dependent power), I(1..3) for exact parity
    A = torch.from_numpy(synth.uniform((n, n), 0, dtype=ndt)).to(dev)
    B = torch.from_numpy(synth.uniform((n, n), 1, dtype=ndt)).to(dev)
    C = torch.from_numpy(synth.uniform((n, n), 2, dtype=ndt)).to(dev)
    Ai_h = synth.small_int((n, n), 1, dtype=ndt); Bi_h = synth.small_int((n, n), 2, dtype=ndt)
    Ci_h = synth.small_int((n, n), 3, dtype=ndt)
    Ai, Bi = torch.from_numpy(Ai_h).to(dev), torch.from_numpy(Bi_h).to(dev)
    g = synth.rng(7)
    ii = g.integers(0, n, 512); jj = g.integers(0, n, 512)
    ref = O.gemm_entries(ii, jj, Ci_h, Ai_h, Bi_h, 1.0, 1.0) if not a.no_parity else None
    iit, jjt = torch.from_numpy(ii).to(dev), torch.from_numpy(jj).to(dev)
    dpar = E.desc_builtin("gemm", (n, n, n), a.dtype); dpar.set_scalars(1.0, 1.0); dpar.set_exec(split_pct=a.split)

    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    out = open(a.out if ws == 1 else a.out.replace(".jsonl", f".rank{rank}.jsonl"), "a")
    interval = nvml_interval_ms(E, local) if rank == 0 or ws > 1 else None
    meta = {"kind": "meta", "rank": rank, "world": ws, "n": n, "split_pct": a.split, "eatss_tile": list(eatss_tile),
            "default_tile": list(default_tile), "variants_total": len(variants), "variants_mine": len(mine),
            "window_s": a.window, "nvml_update_ms": interval, "sizes": sizes, "dtype": a.dtype,
            "gpu": torch.cuda.get_device_name(local), "time": time.time()}
    out.write(json.dumps(meta) + "\n"); out.flush()

    def measure(tile, tag):
        rec = {"kind": tag, "tile": list(tile), "rank": rank}
        if ref is not None and tag == "variant":
            Ci = torch.from_numpy(Ci_h).to(dev)
            try:
                E.run(dpar, tile, [Ci, Ai, Bi])
                torch.cuda.synchronize()
                got = Ci[iit, jjt].double().cpu().numpy()
                rec["exact"] = bool(np.array_equal(got, ref))
            except Exception as e:  # recorded, not fatal
                rec["exact"] = False
                rec["error"] = str(e)[:200]
        try:
            (m,) = E.sweep(d, [tile], [C, A, B], device=local, warmup=a.warmup, min_window_s=a.window)
            rec.update(ms=m.ms_per_run, joules=m.joules_per_run, watts=m.avg_watts, tflops=m.tflops,
                       gflops_per_watt=m.gflops_per_watt, sm_mhz=m.sm_mhz_median, runs=int(m.runs),
                       status=int(m.status))
        except Exception as e:
            rec.update(status=-99, error=str(e)[:200])
        rec["t"] = time.time()
        out.write(json.dumps(rec) + "\n"); out.flush()
        return rec

    t0 = time.time()
    if a.tiles:
        # confirmation mode: the candidate tiles, re-measured round-robin
        conf = [tuple(int(x) for x in s.split(",")) for s in a.tiles.split(";") if s]
        for rep_i in range(a.repeats):
            for tile in conf:
                r = measure(tile, "confirm")
        out.close()
        if rank == 0:
            print(f"[sweep] confirmation: {len(conf)} tiles x {a.repeats} in {time.time() - t0:.0f} s", flush=True)
        return
    measure(default_tile, "anchor_default"); measure(eatss_tile, "anchor_eatss")
    for k, v in enumerate(mine):
        measure(v, "variant")
        if (k + 1) % a.anchor_every == 0:
            measure(default_tile, "anchor_default"); measure(eatss_tile, "anchor_eatss")
            if rank == 0:
                print(f"[sweep] {k + 1}/{len(mine)} variants, {time.time() - t0:.0f} s", flush=True)
    measure(default_tile, "anchor_default"); measure(eatss_tile, "anchor_eatss")
    out.close()
    if ws > 1:
        # gather fixed-size records to rank 0 over NCCL (the only collective of the sweep)
        mine_path = a.out.replace(".jsonl", f".rank{rank}.jsonl")
        recs = [json.loads(l) for l in open(mine_path) if '"kind": "meta"' not in l]
        allrecs = gather_records(recs, rank, ws, dist, torch, dev)
        if rank == 0:
            with open(a.out, "a") as fo:
                fo.write(json.dumps(dict(meta, rank="all", world=ws)) + "\n")
                for r in allrecs:
                    fo.write(json.dumps(r) + "\n")
        dist.barrier()
        dist.destroy_process_group()
    if rank == 0:
        print(f"[sweep] done: {len(mine)} variants in {time.time() - t0:.0f} s -> {a.out}", flush=True)


if __name__ == "__main__":
    main()
