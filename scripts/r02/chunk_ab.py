#!/usr/bin/env python
"""A/B of the tcgen05 GEMM's accumulator chunk (k-blocks of 32 per TMEM drain, EATSS_TCM_CHUNK_K) at the
headline size: device time and precision vs the fp64 oracle (development measurement, not the bench).

    python scripts/r02/chunk_ab.py            # runs one subprocess per chunk value
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)


def one():
    import numpy as np
    import torch

    import paper_conf_cgo_jayaweerakwk24_b200 as E
    import synth
    from oracle import numeric as O

    n = 4000
    A = synth.uniform((n, n), 0); B = synth.uniform((n, n), 1); C = synth.uniform((n, n), 2)
    ref_path = "/tmp/eatss_gemm4000_ref.npy"
    if os.path.exists(ref_path):
        ref = np.load(ref_path)
    else:
        ref = O.gemm(1.5, 1.2, C, A, B)
        np.save(ref_path, ref)
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, int(os.environ.get("ENGINE", "2")))
    Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    Cd = torch.from_numpy(C).cuda()
    t = tuple(int(x) for x in os.environ.get("TILE", "256,256,32").split(","))
    E.run(d, t, [Cd, Ad, Bd]); torch.cuda.synchronize()
    out = Cd.double().cpu().numpy()
    err = O.normwise_rel_err(out, ref)
    mx = float(np.max(np.abs(out - ref)) / np.sqrt(np.mean(ref * ref)))
    Cw = torch.from_numpy(C).cuda()
    for _ in range(5):
        E.run(d, t, [Cw, Ad, Bd])
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); s.record()
    for _ in range(50):
        E.run(d, t, [Cw, Ad, Bd])
    e.record(); torch.cuda.synchronize()
    ms = s.elapsed_time(e) / 50
    print(json.dumps({"engine": os.environ.get("ENGINE", "2"), "tiles": t, "chunk_k": os.environ.get("EATSS_TCM_CHUNK_K", "128"), "ms": ms, "tflops": 2 * n ** 3 / ms / 1e9,
                      "normwise_rel_err": err, "max_abs_err_over_rms": mx}), flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "one":
        one()
    else:
        for r in ("64", "128", "256", "512", "4000"):
            env = dict(os.environ, EATSS_TCM_CHUNK_K=r)
            subprocess.run([sys.executable, __file__, "one"], env=env, check=False)
