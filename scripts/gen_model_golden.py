#!/usr/bin/env python
"""Write tests/golden/model_golden.json by calling ONLY oracle/model.py (brute force).

The C++ enumerator in libeatss.so is checked against this file bit-exactly
(tiles, OBJ, #ties, #feasible).  Re-run after any change of reading.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import model as M  # noqa: E402

CASES = []


def add(kernel, dims, dtype_bytes, gpu, split, waf, mode):
    CASES.append(dict(kernel=kernel, dims=list(dims), dtype_bytes=dtype_bytes, gpu=gpu,
                      split_pct=split, waf=waf, mode=mode))


# the paper-mode pin first
add("gemm", (1024, 1024, 1024), 8, "GA100", 50, 16, 0)
for split in (0, 25, 50, 75, 100):
    add("gemm", (4000, 4000, 4000), 4, "B200", split, 16, 1)
add("gemm", (4000, 4000, 4000), 8, "B200", 50, 16, 1)
add("gemm", (256, 256, 256), 4, "B200", 50, 16, 1)
add("gemm", (4000, 4000, 4000), 4, "B200", 50, 32, 1)
add("gemm", (4000, 4000, 4000), 4, "B200", 50, 8, 1)
add("gemm", (1000, 3000, 200), 4, "B200", 50, 16, 1)
add("2mm", (4000, 4000, 4000, 4000), 4, "B200", 50, 16, 1)
add("2mm", (4000, 4000, 4000, 4000), 4, "B200", 100, 16, 1)
add("3mm", (4000, 4000, 4000, 4000, 4000), 4, "B200", 50, 16, 1)
add("3mm", (4000, 4000, 4000, 4000, 4000), 4, "B200", 0, 16, 1)
add("syrk", (4000, 4000), 4, "B200", 50, 16, 1)
add("syrk", (4000, 4000), 4, "B200", 100, 8, 1)
add("jacobi-2d", (4000,), 4, "B200", 50, 16, 1)
add("jacobi-2d", (4000,), 4, "B200", 0, 32, 1)
for waf in (4, 8, 16, 32):
    add("heat-3d", (120,), 4, "B200", 50, waf, 1)
for waf in (4, 8, 16, 32):
    for split in (0, 50, 100):
        add("heat-3d", (120,), 8, "GA100", split, waf, 0)
# tensor-core mode (reading T)
add("gemm", (4000, 4000, 4000), 4, "B200", 50, 16, 2)
add("2mm", (4000, 4000, 4000, 4000), 4, "B200", 50, 16, 2)
add("3mm", (4000, 4000, 4000, 4000, 4000), 4, "B200", 50, 16, 2)
add("syrk", (4000, 4000), 4, "B200", 50, 16, 2)
add("gemm", (100, 40, 20), 4, "B200", 50, 16, 2)
add("gemm", (300, 1100, 204), 4, "B200", 50, 16, 2)
add("gemm", (4000, 4000, 4000), 4, "GA100", 50, 16, 2)
# tensor-core mode of the 3xFP16 engine (mode 3: 2-byte operands, K-major B, Tk in {64, 128})
add("gemm", (4000, 4000, 4000), 4, "B200", 50, 16, 3)
add("syrk", (4000, 4000), 4, "B200", 50, 16, 3)
add("3mm", (4000, 4000, 4000, 4000, 4000), 4, "B200", 50, 16, 3)
add("gemm", (100, 40, 20), 4, "B200", 50, 16, 3)
add("ccsd_t_d1", (48,), 4, "B200", 50, 4, 2)   # reading T4
add("ccsd_t_d1", (16,), 4, "B200", 50, 16, 2)
add("ccsd_t_d1", (24,), 4, "B200", 50, 4, 2)
add("ccsd_t_d1", (48,), 4, "B200", 50, 4, 1)
add("ccsd_t_d1", (48,), 4, "B200", 50, 8, 1)
add("ccsd_t_d1", (16,), 4, "B200", 50, 4, 1)
# low-dimensional PolyBench kernels
for kern, dims in (("mvt", (4000,)), ("atax", (4000, 4000)), ("bicg", (4000, 4000)), ("gemver", (4000,)),
                   ("atax", (1900, 2100)), ("bicg", (2100, 1900))):
    for split, waf in ((50, 16), (0, 4), (100, 32)):
        add(kern, dims, 4, "B200", split, waf, 1)
add("gemver", (4000,), 8, "GA100", 50, 16, 0)
# non-PolyBench 4-D kernels (readings R-N8, R-N9): B200 at the config sizes,
# GA100 paper mode over the P:282 space (warp_frac x shared-memory quota)
for waf in (4, 8, 16, 32):
    add("mttkrp", (512, 32, 512, 512), 4, "B200", 50, waf, 1)
    add("conv-2d", (8192, 5), 4, "B200", 50, waf, 1)
    for split in (0, 50, 100):
        add("mttkrp", (512, 32, 512, 512), 4, "GA100", split, waf, 0)
        add("conv-2d", (8192, 5), 4, "GA100", split, waf, 0)
add("mttkrp", (60, 20, 36, 44), 4, "B200", 0, 4, 1)
add("conv-2d", (514, 3), 4, "B200", 100, 8, 1)


def main():
    out = []
    for c in CASES:
        prog = M.BUILTINS[c["kernel"]](*c["dims"], dtype_bytes=c["dtype_bytes"])
        gpu = M.GA100 if c["gpu"] == "GA100" else M.B200
        r = M.select_tiles(prog, gpu, M.Opts(c["split_pct"], c["waf"], c["mode"]), keep_ties=False)
        c = dict(c, tiles=list(r.tiles) if r.tiles else None, obj=r.obj, n_ties=r.n_ties,
                 n_feasible=r.n_feasible)
        print(c)
        out.append(c)
    path = os.path.join(ROOT, "tests", "golden", "model_golden.json")
    with open(path, "w") as f:
        json.dump({"generator": "scripts/gen_model_golden.py (oracle/model.py brute force only)",
                   "gpus": {"GA100": M.GA100.__dict__, "B200": M.B200.__dict__},
                   "cases": out}, f, indent=1)
    print("wrote", path)


if __name__ == "__main__":
    main()
