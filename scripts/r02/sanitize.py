#!/usr/bin/env python
"""One small run of every TMA / tcgen05 / bulk-copy executor (for compute-sanitizer: memcheck, racecheck,
synccheck).  Development tool; the parity of these shapes is covered by the GPU tests."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "all"


def bufs(d):
    g = torch.Generator(device="cuda").manual_seed(0)
    return [torch.rand(d.buffer_elems(i), device="cuda", generator=g) for i in range(d.num_buffers)]


def go(kind, dims, tiles, engine, tsteps=0):
    if which not in ("all", kind):
        return
    d = E.desc_builtin(kind, dims, tsteps=tsteps)
    d.set_exec(split_pct=50, engine=engine)
    E.run(d, tiles, bufs(d))
    torch.cuda.synchronize()
    print("ok", kind, tiles, flush=True)


go("gemm", (300, 520, 200), (256, 256, 32), 2)      # tc_mma, CTA pair, split tail, ragged
go("gemm", (260, 300, 136), (128, 48, 16), 2)       # tc_mma single CTA, SW64
go("gemm", (300, 520, 200), (256, 256, 64), 4)      # tc_mma 3xFP16 (maxima + split launches), CTA pair
go("syrk", (300, 200), (128, 64, 32), 4)            # tc_mma 3xFP16, shared K-major split
go("syrk", (300, 200), (256, 96, 64), 2)            # tc_mma K-major B
go("gemm", (100, 300, 64), (16, 256, 32), 2)        # tc_gemm (narrow-tile TS engine)
go("gemm", (300, 520, 200), (16, 1024, 16), 1)      # SIMT staged (bulk copies)
go("ccsd_t_d1", (2, 3, 4, 32, 4, 8, 48), (1, 2, 2, 32, 4, 8, 48), 2)
go("mttkrp", (64, 32, 128, 64), (1, 32, 128, 32), 2)
go("conv-2d", (260, 5), (16, 64, 5, 5), 1)
go("jacobi-2d", (132,), (16, 64), 1, tsteps=3)
go("heat-3d", (68,), (16, 16, 32), 1, tsteps=2)
