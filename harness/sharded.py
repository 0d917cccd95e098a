"""The sharded BASELINE configs on N GPUs (configs 3 and 5), as bench.py runs them at N > 1.

For each config -- 2mm, 3mm (with its one exchange: all_gather of F over NCCL), syrk at N = 4000 and
ccsd_t_d1 at dims 48 (h3 slabs) -- on the tcgen05 engine with the EATSS tensor-mode tile (reading T /
T4), the problem is split over the ranks by harness/multigpu.run_shard (row blocks of whole i-tiles,
h3 slabs).  Per config it reports:
  * ms: device time of one sharded run, max over ranks (barrier + synchronize on both sides, CUDA events);
  * ms_1gpu: the same problem on rank 0 alone, timed the same way (the N = 1 reference) -> speedup,
    strong-scaling efficiency = speedup / N;
  * joules: NVML energy of the sharded run summed over ranks (a window of repeated runs);
  * bit_equal: small-integer inputs (every partial sum exact in fp32 and on the 3xTF32 path: the
    result does not depend on the summation order or the partition), each rank's output rows/slabs
    against rank 0's single-GPU result, compared by 64-bit checksums of the raw fp32 bits per shard;
  * rel_err_vs_1gpu: U[-1,1) inputs (alpha 1.5, beta 1.2), the normwise difference of 4096 sampled
    entries per rank and output against the 1-GPU result (not 0 even at N = 1: the split-k tail adds its
    partial sums with atomics, in no fixed order).
The host logic (partition, exchange, checksum comparison) runs under gloo in tests/test_multigpu_cpu.py.
"""
from __future__ import annotations

import time

import numpy as np

from harness import multigpu as MG

CONFIGS = (("2mm", 4000), ("3mm", 4000), ("syrk", 4000), ("ccsd_t_d1", 48))
OUT_KEYS = {"2mm": ("tmp", "D"), "3mm": ("E", "G"), "syrk": ("C",), "ccsd_t_d1": ("t3",)}


def checksums(torch, t, rows=None, chunk=1 << 26):
    """(sum of the fp32 bit patterns, index-weighted sum) over the rows [r0, r1) of t: int64 arithmetic
    in chunks (the ccsd output is 12G elements), wrapping identically on every rank."""
    x = t.reshape(t.shape[0], -1)
    if rows is not None:
        x = x[rows[0]:rows[1]]
    flat = x.reshape(-1)
    s1 = s2 = 0
    for c0 in range(0, flat.numel(), chunk):
        b = flat[c0:c0 + chunk].contiguous().view(torch.int32).to(torch.int64)
        idx = torch.arange(c0 + 1, c0 + 1 + b.numel(), device=b.device, dtype=torch.int64)
        s1 += int(b.sum().item())
        s2 += int((b * idx).sum().item())
    return s1 & (2 ** 64 - 1), s2 & (2 ** 64 - 1)


def _inputs(kind, dims, torch, dev, small_int, seed):
    X = MG.make_inputs(kind, dims, seed0=seed, small_int=small_int)
    Xd = {k: torch.from_numpy(np.ascontiguousarray(v)).to(dev) for k, v in X.items()}
    if kind == "ccsd_t_d1":
        Xd["t3"] = torch.zeros(tuple(dims[:6]), dtype=torch.float32, device=dev)
    return Xd


def _reset(kind, Xd, X0):
    for k in X0:
        Xd[k].copy_(X0[k])
    if kind == "ccsd_t_d1":
        Xd["t3"].zero_()


def run_config(kind, n, E, torch, dist, rank, ws, dev, gpu, steps=3, window_s=1.0):
    dims = MG.dims_of(kind, n)
    d_full = E.desc_builtin(kind, dims)
    tiles, _ = E.select_tiles(d_full, gpu, 50, 4 if kind == "ccsd_t_d1" else 16, mode=2)
    be = MG.CudaBackend(dev, tiles, dist if ws > 1 else None, engine=2)
    be1 = MG.CudaBackend(dev, tiles, None, engine=2)
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    out = {"tiles": list(tiles), "engine": "tcgen05 3xTF32", "gpus": ws}

    def timed(fn, reps):
        fn()
        torch.cuda.synchronize()
        if ws > 1:
            dist.barrier()
        s, e = ev(), ev()
        s.record()
        for _ in range(reps):
            fn()
        e.record()
        torch.cuda.synchronize()
        ms = s.elapsed_time(e) / reps
        if ws > 1:
            v = torch.tensor([ms], dtype=torch.float64, device=dev)
            dist.all_reduce(v, op=dist.ReduceOp.MAX)
            ms = v.item()
        return ms

    # --- U[-1,1): timing (sharded and, on rank 0 alone, the whole problem -- interleaved, best of 3 so
    # both see the same thermal / power state), then energy of the sharded run
    Xd = _inputs(kind, dims, torch, dev, False, 0)
    shard = lambda: MG.run_shard(kind, dims, tiles, rank, ws, Xd, be)  # noqa: E731
    one = lambda: MG.run_shard(kind, dims, tiles, 0, 1, Xd, be1)  # noqa: E731

    def timed_one():
        ms1 = 0.0
        if rank == 0:
            one(); torch.cuda.synchronize()
            s, e = ev(), ev()
            s.record()
            for _ in range(steps):
                one()
            e.record(); torch.cuda.synchronize()
            ms1 = s.elapsed_time(e) / steps
        if ws > 1:
            dist.barrier()
        v = torch.tensor([ms1], dtype=torch.float64, device=dev)
        if ws > 1:
            dist.broadcast(v, 0)
        return v.item()

    t_sh, t_1 = [], []
    for _ in range(3):
        t_sh.append(timed(shard, steps))
        t_1.append(timed_one())
    out["ms"], out["ms_1gpu"] = min(t_sh), min(t_1)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    mj0, t0, reps = E.energy_mj(dev.index), time.perf_counter(), 0
    while time.perf_counter() - t0 < window_s:
        shard(); reps += 1
        torch.cuda.synchronize()
    mj1 = E.energy_mj(dev.index)
    j = torch.tensor([(mj1 - mj0) / 1e3 / reps], dtype=torch.float64, device=dev)
    if ws > 1:
        dist.all_reduce(j, op=dist.ReduceOp.SUM)
    out["joules"] = j.item()
    out["tflops"] = d_full.flops / (out["ms"] * 1e-3) / 1e12
    out["gflops_per_watt"] = d_full.flops / out["joules"] / 1e9 if out["joules"] > 0 else None
    out["speedup"] = out["ms_1gpu"] / out["ms"]
    out["efficiency"] = out["speedup"] / ws
    del Xd
    # --- bit-equality on small integers, and the U[-1,1) error, shard vs 1-GPU result
    for small in (True, False):
        Xd = _inputs(kind, dims, torch, dev, small, 11)
        X0 = {k: v.clone() for k, v in Xd.items() if k != "t3"}
        # exact pass: exactly representable scalars (alpha = beta = 1), so every value is an integer
        # below 2^24 and the result cannot depend on the order of the (split-k atomic) partial sums
        ab = dict(alpha=1.0, beta=1.0) if small else {}
        res, rr = MG.run_shard(kind, dims, tiles, rank, ws, Xd, be, **ab)
        torch.cuda.synchronize()
        r0, r1 = rr
        if small:  # checksums of this rank's rows / slabs, taken before the buffers are reused
            mine = {k: checksums(torch, res[k]) for k in OUT_KEYS[kind]}
        else:  # 4096 sampled elements of this rank's rows (flat indices into the full output)
            g = torch.Generator(device=dev).manual_seed(5 + rank)
            samp = {}
            for k in OUT_KEYS[kind]:
                x = res[k].reshape(-1)
                per_row = x.numel() // max(1, r1 - r0)
                i = torch.randint(0, max(1, x.numel()), (4096,), device=dev, generator=g)
                samp[k] = (i + r0 * per_row, x[i].double() if x.numel() else torch.zeros(4096, device=dev,
                                                                                            dtype=torch.float64))
        _reset(kind, Xd, X0)
        ref = MG.run_shard(kind, dims, tiles, 0, 1, Xd, be1, **ab)[0] if rank == 0 else None
        torch.cuda.synchronize()
        if small:
            gathered = [None] * ws
            if ws > 1:
                dist.all_gather_object(gathered, (rr, mine))
            else:
                gathered = [(rr, mine)]
            ok = True
            if rank == 0:
                for (q0, q1), cs in gathered:
                    for k in OUT_KEYS[kind]:
                        ok &= cs[k] == checksums(torch, ref[k], (q0, q1))
            flag = torch.tensor([1.0 if ok else 0.0], device=dev, dtype=torch.float64)
            if ws > 1:
                dist.broadcast(flag, 0)
            out["bit_equal"] = bool(flag.item() > 0.5)
            out["bit_equal_inputs"] = "small integers in [-1, 1] (exact in fp32 and 3xTF32)"
        else:
            num = den = 0.0
            for k in OUT_KEYS[kind]:
                idx, val = samp[k]
                live = torch.tensor([1.0 if r1 > r0 else 0.0], device=dev, dtype=torch.float64)
                parts_i = [torch.empty_like(idx) for _ in range(ws)]
                parts_v = [torch.empty_like(val) for _ in range(ws)]
                parts_l = [torch.empty_like(live) for _ in range(ws)]
                if ws > 1:
                    dist.all_gather(parts_i, idx); dist.all_gather(parts_v, val); dist.all_gather(parts_l, live)
                else:
                    parts_i, parts_v, parts_l = [idx], [val], [live]
                if rank == 0:
                    full = ref[k].reshape(-1)
                    for ii, vv, ll in zip(parts_i, parts_v, parts_l):
                        if ll.item() < 0.5:
                            continue
                        rf = full[ii].double()
                        num += float(((vv - rf) ** 2).sum().item()); den += float((rf ** 2).sum().item())
            e = torch.tensor([(num / den) ** 0.5 if den > 0 else 0.0], device=dev, dtype=torch.float64)
            if ws > 1:
                dist.broadcast(e, 0)
            out["rel_err_vs_1gpu"] = e.item()
        del Xd, res, ref
        torch.cuda.empty_cache()
    return out


def sharded_configs(E, torch, dist, rank, ws, dev, gpu, configs=CONFIGS):
    res = {}
    for kind, n in configs:
        res[f"{kind} n={n}"] = run_config(kind, n, E, torch, dist, rank, ws, dev, gpu)
        torch.cuda.empty_cache()
    return res
