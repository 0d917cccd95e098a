#!/usr/bin/env python
"""Exactness of every tile of the tensor-engine space (Ti in {128,256}, Tj in 16..256 step 16, Tk in
{8,16,32,64}) on small-integer inputs, gemm (MN-major B) and syrk (K-major B); prints failures and
per-tile time at N=4000 (development check; the tests pin a subset)."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402
import synth  # noqa: E402
from oracle import numeric as O  # noqa: E402


def main():
    ni, nj, nk = 300, 1100, 204
    A = synth.small_int((ni, nk), 10); B = synth.small_int((nk, nj), 11); C = synth.small_int((ni, nj), 12)
    ref = O.gemm(1.0, 1.0, C, A, B)
    As = synth.small_int((ni, nk), 13); Cs = synth.small_int((ni, ni), 14)
    refs = O.syrk(1.0, 1.0, Cs, As)
    Ad, Bd, Asd = (torch.from_numpy(x).cuda() for x in (A, B, As))
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 1.0); d.set_exec(50, 2)
    ds = E.desc_builtin("syrk", (ni, nk)); ds.set_scalars(1.0, 1.0); ds.set_exec(50, 2)
    bad, ok, uns = [], 0, []
    for ti in (128, 256):
        for tj in range(16, 257, 16):
            for tk in (8, 16, 32, 64):
                t = (ti, tj, tk)
                for name, dd, bufs, r in (("gemm", d, lambda: [torch.from_numpy(C).cuda(), Ad, Bd], ref),
                                          ("syrk", ds, lambda: [torch.from_numpy(Cs).cuda(), Asd], refs)):
                    b = bufs()
                    try:
                        E.run(dd, t, b)
                        torch.cuda.synchronize()
                    except E.EatssError as e:
                        uns.append((name, t, str(e)[:60]))
                        continue
                    if np.array_equal(b[0].double().cpu().numpy(), r):
                        ok += 1
                    else:
                        diff = np.abs(b[0].double().cpu().numpy() - r)
                        bad.append((name, t, float(diff.max()), int((diff > 0).sum())))
    print(json.dumps({"exact": ok, "bad": bad, "unsupported": uns[:200], "n_unsupported": len(uns)}), flush=True)
    # timing at N = 4000 (gemm), 10 runs per tile
    n = 4000
    g = E.desc_builtin("gemm", (n, n, n)); g.set_scalars(1.5, 1.2); g.set_exec(50, 2)
    A4 = torch.rand(n, n, device="cuda") * 2 - 1; B4 = torch.rand(n, n, device="cuda") * 2 - 1
    C4 = torch.rand(n, n, device="cuda") * 2 - 1
    for ti in (128, 256):
        for tj in range(16, 257, 16):
            for tk in (8, 16, 32, 64):
                t = (ti, tj, tk)
                try:
                    E.run(g, t, [C4, A4, B4])
                except E.EatssError:
                    continue
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize(); s.record()
                for _ in range(10):
                    E.run(g, t, [C4, A4, B4])
                e.record(); torch.cuda.synchronize()
                ms = s.elapsed_time(e) / 10
                print(json.dumps({"tiles": t, "ms": ms, "tflops": 2 * n ** 3 / ms / 1e9}), flush=True)


if __name__ == "__main__":
    main()
