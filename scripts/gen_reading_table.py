#!/usr/bin/env python
"""Write tests/golden/reading_table.json by calling ONLY oracle/model.py: for the alternative readings of
the ambiguous model text (oracle.model.Reading) --

  * "p282": the paper-pinned feasibility counts of P:282 (GA100 paper mode, warp_frac x shared quota):
    heat-3d 9 of 12, mttkrp and conv-2d 11 of 12 -- recomputed under every alternative, conv-2d at every
    filter size 3..11, so P:282 is a pin that discriminates readings instead of a fit of the filter;
  * "worked_example": the P:117-121 example under every alternative (tile and objective printed at P:121);
  * "fdtd_nrefs": no.references of fdtd-2d (P:153 prints 4);
  * "tiles": the tile each reading picks for the BASELINE configs 4-5 (jacobi-2d, heat-3d, ccsd_t_d1) on
    B200 (mode 1, split 50%), with the tie set -- what harness/readings.py measures on the GPU.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from oracle import model as M  # noqa: E402

ALTS = {
    "R": M.R,
    "footprint=halo": M.Reading(footprint="halo"),
    "split=literal": M.Reading(split="literal"),
    "nrefs=array": M.Reading(nrefs="array"),
    "nrefs=ref": M.Reading(nrefs="ref"),
    "units=KB": M.Reading(units="KB"),
    "waf_scale=warp": M.Reading(waf_scale="warp"),
    "h_count=array": M.Reading(h_count="array"),
    "h_count=ref": M.Reading(h_count="ref"),
    "rule2d=none": M.Reading(rule2d="none"),
    "rule2d=scaled": M.Reading(rule2d="scaled"),
    "bset=outer": M.Reading(bset="outer"),
    "bset=ls1_inner": M.Reading(bset="ls1_inner"),
    "tiebreak=lexmin": M.Reading(tiebreak="lexmin"),
    "tiebreak=lexmax": M.Reading(tiebreak="lexmax"),
}


def p282(prog, rd):
    miss = []
    n = 0
    for wf in (0.125, 0.25, 0.5, 1.0):
        for split in (0, 50, 100):
            ok = M.select_tiles(prog, M.GA100, M.Opts(split, int(wf * 32), 0), keep_ties=False, rd=rd).tiles is not None
            n += ok
            if not ok:
                miss.append([wf, split])
    return {"feasible": n, "missing": miss}


def main():
    out = {"generator": "scripts/gen_reading_table.py (oracle/model.py only)", "readings": {}}
    progs = {"heat-3d n=120 fp64": M.heat3d(120, 8), "heat-3d n=120 fp32": M.heat3d(120, 4),
             "mttkrp 512x32x512x512": M.mttkrp(512, 32, 512, 512), "mttkrp 64x32x64x64": M.mttkrp(64, 32, 64, 64)}
    for f in range(3, 12):
        progs[f"conv-2d n=8192 f={f}"] = M.conv2d(8192, f)
    cfg = [("jacobi-2d", M.jacobi2d(4000), 16), ("heat-3d", M.heat3d(120), 16), ("heat-3d", M.heat3d(120), 8),
           ("heat-3d", M.heat3d(120), 4), ("ccsd_t_d1", M.ccsd_t_d1(48), 4), ("gemm", M.gemm(), 16)]
    for name, rd in ALTS.items():
        rec = {"reading": rd.__dict__ if hasattr(rd, "__dict__") else str(rd), "p282": {}, "tiles": []}
        for pn, prog in progs.items():
            rec["p282"][pn] = p282(prog, rd)
        r = M.select_tiles(M.matmul_paper(1024, 8), M.GA100, M.Opts(50, 16, 0), rd=rd)
        rec["worked_example"] = {"tiles": list(r.tiles) if r.tiles else None, "obj": r.obj,
                                 "H": M.derive(M.matmul_paper().nests[0], 16, rd).H}
        rec["fdtd_nrefs"] = max(M.derive(n, 16, rd).nrefs for n in M.fdtd2d().nests)
        for kname, prog, waf in cfg:
            r = M.select_tiles(prog, M.B200, M.Opts(50, waf, 1), rd=rd)
            rec["tiles"].append({"kernel": kname, "waf": waf, "pick": list(r.tiles) if r.tiles else None,
                                 "obj": r.obj, "n_ties": r.n_ties, "ties": [list(t) for t in r.ties]})
        out["readings"][name] = rec
        print(name, {k: v["feasible"] for k, v in rec["p282"].items()}, rec["worked_example"], flush=True)
    path = os.path.join(ROOT, "tests", "golden", "reading_table.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=0)
    print("wrote", path)


if __name__ == "__main__":
    main()
