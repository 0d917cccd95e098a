#!/usr/bin/env python
"""Quick device timing of one builtin + tile vector (development tool, not the bench).

    python scripts/time_kernel.py gemm 4000,4000,4000 16,1024,16 [--iters 20]
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_jayaweerakwk24_b200 as E  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("kind")
    ap.add_argument("dims")
    ap.add_argument("tiles")
    ap.add_argument("--tsteps", type=int, default=0)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--split", type=int, default=50)
    ap.add_argument("--engine", type=int, default=0)
    ap.add_argument("--kernel-ms", action="store_true", help="also report the main kernel alone (exec.time_kernels)")
    a = ap.parse_args()
    dims = [int(x) for x in a.dims.split(",")]
    tiles = [int(x) for x in a.tiles.split(",")]
    d = E.desc_builtin(a.kind, dims, tsteps=a.tsteps)
    d.set_exec(split_pct=a.split, engine=a.engine, time_kernels=1 if a.kernel_ms else 0)
    bufs = [torch.rand(d.buffer_elems(i), device="cuda") * 2 - 1 for i in range(d.num_buffers)]
    if a.kind == "ccsd_t_d1":
        bufs[0].zero_()
    for _ in range(3):
        E.run(d, tiles, bufs)
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(a.iters):
        E.run(d, tiles, bufs)
    e.record()
    torch.cuda.synchronize()
    ms = s.elapsed_time(e) / a.iters
    if a.kernel_ms:
        ks = []
        for _ in range(5):
            E.run(d, tiles, bufs)
            torch.cuda.synchronize()
            ks.append(sum(E.last_kernel_ms(d)))
        ks.sort()
        print(f"kernel {ks[2]:.4f} ms (median of 5)  {d.flops / ks[2] / 1e9:.2f} TFLOP/s", flush=True)
    p = E.plan(d, tiles)[0]
    print(f"{a.kind} {dims} tiles {tiles}: {ms:.3f} ms  {d.flops / ms / 1e9:.2f} TFLOP/s  "
          f"{d.bytes / ms / 1e6:.1f} GB/s  grid ({p.grid_x},{p.grid_y}) block ({p.block_x},{p.block_y}) "
          f"mt {p.rm}x{p.rn} v{p.vec} passes {p.passes} smem {p.smem_bytes}", flush=True)


if __name__ == "__main__":
    main()
