#!/usr/bin/env python
"""Development measurement: normwise error of the tensor engines at N = 4000 against an fp64 torch
reference computed on the GPU (the plain definitions -- no oracle/ code), for several accumulator chunk
lengths (EATSS_TCM_CHUNK_K), on gemm, 2mm (D), 3mm (G) and syrk with U[-1,1) inputs.

    python scripts/r02/precision_chunks.py ENGINE TILE CHUNK [CHUNK ...]   # one subprocess per chunk
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)


def one(engine, tiles):
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E
    import synth

    n = 4000
    dev = lambda x: torch.from_numpy(x).cuda()
    A, B, C, D = (dev(synth.uniform((n, n), s)) for s in (50, 51, 52, 53))
    a64, b64, c64, d64 = (x.double() for x in (A, B, C, D))
    err = lambda x, r: float(torch.linalg.norm(x.double() - r) / torch.linalg.norm(r))
    out = {}
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, engine)
    Cd = C.clone(); E.run(d, tiles, [Cd, A, B])
    out["gemm"] = err(Cd, 1.5 * a64 @ b64 + 1.2 * c64)
    d = E.desc_builtin("2mm", (n, n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, engine)
    tmp = torch.empty_like(A); Dd = D.clone(); E.run(d, tiles, [tmp, A, B, C, Dd])
    out["2mm"] = err(Dd, (1.5 * a64 @ b64) @ c64 + 1.2 * d64)
    d = E.desc_builtin("3mm", (n, n, n, n, n)); d.set_exec(50, engine)
    bufs = [torch.empty_like(A), A, B, torch.empty_like(A), C, D, torch.empty_like(A)]
    E.run(d, tiles, bufs)
    out["3mm"] = err(bufs[6], (a64 @ b64) @ (c64 @ d64))
    d = E.desc_builtin("syrk", (n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, engine)
    Cd = C.clone(); E.run(d, tiles, [Cd, A])
    out["syrk"] = err(Cd, 1.5 * a64 @ a64.T + 1.2 * c64)
    torch.cuda.synchronize()
    return out


if __name__ == "__main__":
    if os.environ.get("_PC_CHILD"):
        t = tuple(int(x) for x in sys.argv[2].split(","))
        print(json.dumps(one(int(sys.argv[1]), t)))
        sys.exit(0)
    eng, tile = sys.argv[1], sys.argv[2]
    for ck in sys.argv[3:]:
        env = dict(os.environ, _PC_CHILD="1", EATSS_TCM_CHUNK_K=ck)
        r = subprocess.run([sys.executable, __file__, eng, tile], env=env, capture_output=True, text=True)
        line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr[-400:]
        print(json.dumps({"engine": int(eng), "tiles": tile, "chunk_k": int(ck), "err": json.loads(line) if line.startswith("{") else line}), flush=True)
