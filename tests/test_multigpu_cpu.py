"""World-size-2 gloo tests of the multi-GPU sharding / exchange logic (harness/multigpu.py).

The shard compute is the fp64 oracle (test-only backend); what is under test is the
partition (whole i-tiles per rank), the 3mm all_gather of F between nests and the
reassembly: the union of the shards must equal the single-process oracle result
exactly (the per-element operation order does not depend on the partition).
"""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from harness import multigpu as MG  # noqa: E402
from oracle import numeric as O  # noqa: E402


class OracleBackend:
    """fp64 oracle shard compute + gloo all_gather (test-only)."""

    def gemm(self, alpha, beta, C, A, B, init_zero):
        if init_zero:
            C = np.zeros_like(C, dtype=np.float64)
        return O.gemm(alpha, beta if not init_zero else 0.0, C, A, B)

    def syrk_rows(self, alpha, beta, Crows, Afull, r0):
        rows = Crows.shape[0]
        A = np.asarray(Afull, np.float64)
        out = np.empty((rows, A.shape[0]))
        for i in range(rows):  # row block of the oracle's full square syrk, same k order
            out[i] = O.gemm(alpha, beta, Crows[i:i + 1], A[r0 + i:r0 + i + 1], A.T.copy())[0]
        return out

    def ccsd(self, t3, t2, v2):
        return O.ccsd_t_d1(t3, t2, v2)

    def all_gather_rows(self, local, total_rows, ranges):
        ws = dist.get_world_size()
        maxr = max(r1 - r0 for r0, r1 in ranges)
        buf = torch.zeros((maxr,) + tuple(local.shape[1:]), dtype=torch.float64)
        buf[: local.shape[0]] = torch.from_numpy(np.asarray(local, np.float64))
        parts = [torch.empty_like(buf) for _ in range(ws)]
        dist.all_gather(parts, buf)
        return np.concatenate([p[: r1 - r0].numpy() for p, (r0, r1) in zip(parts, ranges)], 0)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, kind, dims, tiles, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    X = MG.make_inputs(kind, dims)
    if kind == "ccsd_t_d1":
        X["t3"] = MG.make_inputs("gemm", (int(np.prod(dims[:6])), 1, 1), seed0=9)["C"].reshape(dims[:6])
    out, rr = MG.run_shard(kind, dims, tiles, rank, world, X, OracleBackend())
    # gather the shards to rank 0 (object gather over gloo)
    payload = {k: np.asarray(v) for k, v in out.items()}
    gathered = [None] * world
    dist.all_gather_object(gathered, (rr, payload))
    if rank == 0:
        q.put(gathered)
    dist.barrier()
    dist.destroy_process_group()


def _run(kind, dims, tiles, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, kind, dims, tiles, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = q.get(timeout=300)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return res


def test_shard_rows_partition_covers_and_aligns():
    for M, G, Ti in [(4000, 8, 16), (1000, 3, 24), (17, 4, 4), (5, 8, 16)]:
        ranges = [MG.shard_rows(M, G, Ti, r) for r in range(G)]
        assert ranges[0][0] == 0 and ranges[-1][1] == M
        for (a0, a1), (b0, b1) in zip(ranges, ranges[1:]):
            assert a1 == b0
        for r0, r1 in ranges:
            assert r0 % Ti == 0 and r0 <= r1


@pytest.mark.parametrize("kind,dims,tiles", [
    ("gemm", (37, 29, 23), (8, 16, 8)),
    ("2mm", (33, 20, 18, 26), (8, 32, 8)),
    ("3mm", (30, 28, 17, 25, 19), (8, 16, 4)),
    ("syrk", (26, 15), (4, 16, 8)),
    ("ccsd_t_d1", (5, 3, 4, 3, 2, 6, 4), (2, 3, 4, 3, 2, 6, 4)),
])
def test_gloo_world2_shards_equal_single_process(kind, dims, tiles):
    res = _run(kind, dims, tiles)
    X = MG.make_inputs(kind, dims)
    if kind == "gemm":
        ref = {"C": O.gemm(1.5, 1.2, X["C"], X["A"], X["B"])}
    elif kind == "2mm":
        tmp, D = O.two_mm(1.5, 1.2, X["A"], X["B"], X["C"], X["D"])
        ref = {"tmp": tmp, "D": D}
    elif kind == "3mm":
        E, F, G = O.three_mm(X["A"], X["B"], X["C"], X["D"])
        ref = {"E": E, "G": G}
    elif kind == "syrk":
        ref = {"C": O.syrk(1.5, 1.2, X["C"], X["A"])}
    else:
        t3 = MG.make_inputs("gemm", (int(np.prod(dims[:6])), 1, 1), seed0=9)["C"].reshape(dims[:6])
        ref = {"t3": O.ccsd_t_d1(t3, X["t2"], X["v2"])}
    for key, full in ref.items():
        parts = sorted([(rr, p[key]) for rr, p in res], key=lambda t: t[0][0])
        got = np.concatenate([np.asarray(p, np.float64) for _, p in parts], 0)
        assert got.shape == full.shape
        # syrk rows use the same k order as the oracle: exact; others exact by construction
        assert np.array_equal(got, full), key
    if kind == "3mm":  # every rank holds the full gathered F after the exchange
        for _, p in res:
            assert np.array_equal(np.asarray(p["F"]), O.three_mm(X["A"], X["B"], X["C"], X["D"])[1])


# ------------------------------------------------------------------ the sweep's record gather
def _fake_records(rank):
    """Rank r's sweep records: its GPU runs 10% faster per rank (different clocks) and drifts down in
    time; the EATSS anchors see the same drift -- per-GPU anchor normalisation must undo both."""
    g = np.random.default_rng(rank)
    scale = 1.0 + 0.1 * rank
    recs = []
    for k in range(12):
        t = 1000.0 + 10.0 * k + rank
        drift = 1.0 - 0.01 * k
        anchor = k % 4 == 0 or k == 11  # anchors bracket every variant (interpolation, not extrapolation)
        tile = [16, 1024, 16] if anchor else [int(x) for x in g.choice([16, 32, 64], 3)]
        kind = "anchor_eatss" if anchor else "variant"
        base = 50.0 if kind == "anchor_eatss" else 40.0 + tile[0] / 8
        ppw = base * scale * drift
        recs.append({"kind": kind, "tile": tile, "exact": True, "ms": 1.0, "joules": 1.0 / ppw, "watts": 500.0,
                     "tflops": ppw * 0.5, "gflops_per_watt": ppw, "sm_mhz": 1800.0, "runs": 10, "status": 0, "t": t})
    return recs


def _gather_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from harness import sweep as SW
    out = SW.gather_records(_fake_records(rank), rank, world, dist, torch, torch.device("cpu"))
    if rank == 0:
        q.put(out)
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_sweep_gather_keeps_rank_and_time(tmp_path):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_gather_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    got = q.get(timeout=300)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert len(got) == 24
    for rank in (0, 1):
        mine = [r for r in got if r["rank"] == rank]
        want = _fake_records(rank)
        assert [(r["kind"], r["tile"], r["t"]) for r in mine] == [(w["kind"], w["tile"], w["t"]) for w in want]
        assert all(abs(r["gflops_per_watt"] - w["gflops_per_watt"]) < 1e-9 for r, w in zip(mine, want))
    # per-GPU anchor normalisation: after correction a variant's PPW no longer depends on its GPU or time
    sys.path.insert(0, os.path.join(ROOT, "harness"))
    import report
    path = tmp_path / "gathered.jsonl"
    with open(path, "w") as f:
        f.write('{"kind": "meta", "eatss_tile": [16, 1024, 16], "nvml_update_ms": 100.0}\n')
        for r in got:
            f.write(__import__("json").dumps(r) + "\n")
    s = report.summarise(str(path))
    assert s["drift_corrected"]["per_gpu_anchors"] == {"0": 4, "1": 4}
    meta, var, anc = report.load(str(path))
    ok = [r for r in var]
    corr = {}
    for r in ok:
        # reproduce the normalisation for the check: variant PPW / its rank's interpolated anchor
        an = sorted([a for a in anc["anchor_eatss"] if a["rank"] == r["rank"]], key=lambda a: a["t"])
        v = r["gflops_per_watt"] / np.interp(r["t"], [a["t"] for a in an], [a["gflops_per_watt"] for a in an])
        corr.setdefault(r["tile"][0], set()).add(round(v, 6))
    # same tile[0] -> same base PPW on both GPUs -> identical normalised value
    assert all(len(v) == 1 for v in corr.values()), corr


def test_sharded_checksums_compare_row_blocks():
    from harness import sharded as SH
    full = torch.arange(6 * 5, dtype=torch.float32).reshape(6, 5) * 0.5
    a = SH.checksums(torch, full, (2, 4))
    assert a == SH.checksums(torch, full[2:4].clone())
    bad = full[2:4].clone()
    bad[1, 3] = torch.nextafter(bad[1, 3], torch.tensor(1e9))  # one ulp off
    assert SH.checksums(torch, bad) != a
