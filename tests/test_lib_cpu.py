"""CPU-only tests of libeatss.so: ABI surface, the C++ tile model against the
brute-force oracle, error paths and launch-plan invariants.  No compute calls."""
import json
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_cgo_jayaweerakwk24_b200 as E
from paper_conf_cgo_jayaweerakwk24_b200 import _abi
from oracle import model as M

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    src = open(os.path.join(ROOT, "include", "eatss.h")).read()
    return sorted(set(re.findall(r"\b(eatss_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    out = subprocess.run(["nm", "-D", "--defined-only", E.lib_path], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (eatss_\w+)", out))
    declared = header_symbols()
    assert declared and set(declared) <= exported, set(declared) - exported
    # the ctypes table covers exactly the header
    assert sorted(n for n, _, _ in _abi.DECLS) == declared


def test_abi_version():
    assert E.abi_version() == 2


def _gpu(name):
    return E.gpu_params_ga100() if name == "GA100" else E.gpu_params_b200()


def test_gpu_param_tables_match_oracle():
    for name, ref in (("GA100", M.GA100), ("B200", M.B200)):
        g = _gpu(name)
        assert g.threads_per_block == ref.T_P_B and g.regs_per_sm == ref.R_P_S
        assert g.l1_shared_bytes == ref.L1_SH and g.l2_bytes == ref.L2 and g.num_sms == ref.n_SM
        assert g.max_smem_per_block == ref.max_smem_per_block


GOLD = json.load(open(os.path.join(ROOT, "tests", "golden", "model_golden.json")))


@pytest.mark.parametrize("case", GOLD["cases"], ids=lambda c: f"{c['kernel']}-{c['gpu']}-{c['split_pct']}-{c['waf']}-{c['dtype_bytes']}")
def test_cpp_model_bit_exact_vs_bruteforce_golden(case):
    dtype = "f64" if case["dtype_bytes"] == 8 else "f32"
    d = E.desc_builtin(case["kernel"], case["dims"], dtype, tsteps=1 if case["kernel"] in ("jacobi-2d", "heat-3d") else 0)
    g = _gpu(case["gpu"])
    if case["tiles"] is None:
        with pytest.raises(E.EatssError) as ei:
            E.select_tiles(d, g, case["split_pct"], case["waf"], case["mode"])
        assert ei.value.status == _abi.EATSS_E_INFEASIBLE
        return
    tiles, rep = E.select_tiles(d, g, case["split_pct"], case["waf"], case["mode"])
    assert list(tiles) == case["tiles"]
    assert rep.obj == case["obj"]
    assert rep.n_ties == case["n_ties"]
    assert rep.n_feasible == case["n_feasible"]


@pytest.mark.parametrize("seed", range(12))
def test_cpp_model_matches_bruteforce_on_random_small_programs(seed):
    """Random extents / splits / WAF on small spaces: C++ DFS vs unpruned numpy brute force."""
    g = np.random.default_rng(seed)
    kind = ["gemm", "2mm", "3mm", "syrk", "jacobi-2d", "heat-3d"][seed % 6]
    waf = int(g.choice([4, 8, 16]))
    split = int(g.choice([0, 25, 50, 67, 100]))
    mode = int(g.integers(0, 2))
    gpu_name = ["GA100", "B200"][int(g.integers(0, 2))]
    db = int(g.choice([4, 8]))
    if kind == "gemm":
        dims = tuple(int(x) for x in g.integers(20, 300, 3))
    elif kind == "2mm":
        dims = tuple(int(x) for x in g.integers(20, 200, 4))
    elif kind == "3mm":
        dims = tuple(int(x) for x in g.integers(20, 150, 5))
    elif kind == "syrk":
        dims = tuple(int(x) for x in g.integers(20, 300, 2))
    elif kind == "jacobi-2d":
        dims = (int(g.integers(30, 900)),)
    else:
        dims = (int(g.integers(10, 90)),)
    prog = M.BUILTINS[kind](*dims, dtype_bytes=db)
    ref = M.select_tiles(prog, M.GA100 if gpu_name == "GA100" else M.B200, M.Opts(split, waf, mode))
    d = E.desc_builtin(kind, dims, "f64" if db == 8 else "f32", tsteps=1 if kind in ("jacobi-2d", "heat-3d") else 0)
    try:
        tiles, rep = E.select_tiles(d, _gpu(gpu_name), split, waf, mode)
    except E.EatssError as e:
        assert e.status == _abi.EATSS_E_INFEASIBLE and ref.tiles is None
        return
    assert tiles == ref.tiles
    assert (rep.obj, rep.n_ties, rep.n_feasible) == (ref.obj, ref.n_ties, ref.n_feasible)


def test_model_info_matches_paper_example():
    d = E.desc_builtin("gemm", (1024, 1024, 1024), "f64")
    ls1, nrefs, H = d.model_info(0, 16)
    assert ls1 == 1 and nrefs == 3 and H == [0, 32, 0]


def test_error_paths():
    with pytest.raises(E.EatssError) as e:
        E.desc_builtin("gemm", (4000, 4000))
    assert e.value.status == _abi.EATSS_E_INVALID
    with pytest.raises(E.EatssError):
        E.desc_builtin("gemm", (4000, 0, 4000))
    with pytest.raises(E.EatssError):
        E.desc_builtin("jacobi-2d", (2,), tsteps=1)
    d = E.desc_builtin("gemm", (64, 64, 64))
    with pytest.raises(E.EatssError) as e:
        E.select_tiles(d, E.gpu_params_b200(), split_pct=101)
    assert e.value.status == _abi.EATSS_E_INVALID
    with pytest.raises(E.EatssError) as e:
        E.plan(d, (16, 0, 16))
    assert e.value.status == _abi.EATSS_E_INVALID
    lib = E._lib
    assert lib.eatss_select_tiles(None, None, None, None, None) == _abi.EATSS_E_INVALID
    assert lib.eatss_run(None, None, None, None) == _abi.EATSS_E_INVALID
    with pytest.raises(ValueError):
        E.run(d, (16, 16, 16), [1, 2])  # wrong number of buffers


def test_run_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    d = E.desc_builtin("gemm", (64, 64, 64))
    with pytest.raises(E.EatssError) as e:
        E.run(d, (16, 16, 16), [256, 512, 768], stream=0)
    assert e.value.status == _abi.EATSS_E_CUDA


def test_flops_and_bytes_accounting():
    d = E.desc_builtin("gemm", (4000, 4000, 4000))
    assert d.flops == 2 * 4000 ** 3
    assert d.bytes == 4 * 4 * 4000 ** 2  # A, B read; C read + written
    assert E.desc_builtin("ccsd_t_d1", (48,)).flops == 2 * 48 ** 7
    assert E.desc_builtin("jacobi-2d", (4000,), tsteps=500).flops == 5 * 3998 ** 2 * 500
    assert E.desc_builtin("heat-3d", (120,), tsteps=500).flops == 15 * 118 ** 3 * 1000
    assert E.launches_per_run(E.desc_builtin("jacobi-2d", (64,), tsteps=7), (16, 16)) == 8


@pytest.mark.parametrize("tiles", [(16, 1024, 16), (32, 32, 32), (4, 4, 4), (1024, 1024, 1024), (24, 768, 48), (7, 13, 5)])
def test_contraction_plan_invariants(tiles):
    M_, N_, K_ = 4000, 4000, 4000
    d = E.desc_builtin("gemm", (M_, N_, K_))
    (p,) = E.plan(d, tiles)
    Ti, Tj, Tk = (min(t, n) for t, n in zip(tiles, (M_, N_, K_)))
    assert (p.tile[0], p.tile[1], p.tile[2]) == (Ti, Tj, Tk)
    assert p.grid_x == -(-N_ // Tj) and p.grid_y == -(-M_ // Ti)       # Fig. 4: tj -> x, ti -> y
    assert 1 <= p.block_x * p.block_y <= 1024                         # tile != block (Q1)
    # a pass covers (by*rm) x (bx*rn) outputs; passes cover the tile
    cover_i = p.block_y * p.rm
    cover_j = p.block_x * p.rn
    assert p.passes >= 1
    assert p.passes == (-(-Ti // cover_i)) * (-(-Tj // cover_j))
    assert p.smem_bytes <= 232448
    if p.a_in_smem:
        assert p.smem_bytes >= Ti * Tk * 4


def test_eatss_pick_is_register_resident():
    d = E.desc_builtin("gemm", (4000, 4000, 4000))
    tiles, _ = E.select_tiles(d, E.gpu_params_b200(), 50, 16)
    (p,) = E.plan(d, tiles)
    assert tiles == (16, 1024, 16) and p.passes == 1 and p.a_in_smem and p.vec == 4


# ------------------------------------------------------------------ 4-D builtins (readings R-N8, R-N9)
def test_fourd_descriptors_and_accounting():
    d = E.desc_builtin("mttkrp", (512, 32, 512, 512))
    assert d.num_loops == 4 and d.num_nests == 1 and d.num_buffers == 4
    assert [d.buffer_elems(i) for i in range(4)] == [512 * 32, 512 ** 3, 512 * 32, 512 * 32]
    assert d.flops == 2 * 512 * 32 * 512 * 512
    assert d.bytes == 4 * (2 * 512 * 32 + 512 ** 3 + 2 * 512 * 32)
    c = E.desc_builtin("conv-2d", (8192, 5))
    assert c.num_loops == 4 and c.num_buffers == 3
    assert [c.buffer_elems(i) for i in range(3)] == [8188 ** 2, 8192 ** 2, 25]
    assert c.flops == 2 * 25 * 8188 ** 2
    assert c.bytes == 4 * (8192 ** 2 + 25 + 8188 ** 2)
    with pytest.raises(E.EatssError):
        E.desc_builtin("conv-2d", (4, 5))  # filter larger than the image
    # model view (rules 2-8, tests/test_oracle_model.py::test_mttkrp_conv2d_derivation)
    assert d.model_info(0, 16) == (1, 4, [0, 48, 0, 0])
    assert c.model_info(0, 16) == (1, 3, [0, 32, 0, 0])


def test_mttkrp_plan_split_and_launches():
    d = E.desc_builtin("mttkrp", (512, 32, 512, 512))
    (p,) = E.plan(d, (128, 32, 16, 16))
    assert (p.grid_x, p.grid_y) == (1, 4)
    assert p.block_x * p.block_y == 128 and p.rm == 8 and p.vec == 4
    # (k-tile, l-tile) pairs split until ~2 CTAs per SM: 32 x 32 pairs over 4 blocks
    assert p.grid_z == p.passes and 1 < p.grid_z <= 32 * 32
    assert E.launches_per_run(d, (128, 32, 16, 16)) == 2          # kernel + split-order reduction
    (q,) = E.plan(d, (7, 12, 5, 9))                                # Tl % 4 != 0: general path
    assert q.vec == 1 and q.grid_z == 1
    d.set_exec(split_pct=50, engine=2)
    # D lo, tcgen05 kernel, reduction (-1 only without a CUDA driver: no TMA descriptor encoder)
    import torch
    assert E.launches_per_run(d, (1, 32, 128, 32)) == (3 if torch.cuda.is_available() else -1)
    assert E.launches_per_run(d, (128, 32, 16, 16)) == -1          # not MMA-legal on the tensor engine


@pytest.mark.parametrize("tiles", [(16, 64, 5, 5), (8, 152, 5, 5), (1024, 1024, 5, 5), (7, 13, 3, 3)])
def test_conv2d_plan_invariants(tiles):
    n, f = 8192, 5
    m = n - f + 1
    d = E.desc_builtin("conv-2d", (n, f))
    (p,) = E.plan(d, tiles)
    Ti, Tj = min(tiles[0], m), min(tiles[1], m)
    assert p.grid_x == -(-m // Tj) and p.grid_y == -(-m // Ti)
    assert 1 <= p.block_x <= 256
    assert (p.tile[2], p.tile[3]) == (min(tiles[2], f), min(tiles[3], f))
    if Tj % 4 == 0:  # fast path: the (row chunk + halo) x window fits the per-CTA budget
        assert p.vec == 4 and 0 < p.smem_bytes <= 2 * 64 * 1024 and p.rm >= 1
    else:
        assert p.vec == 1
    assert E.launches_per_run(d, tiles) == 1


def test_syrk_simt_layout_pass_counted():
    d = E.desc_builtin("syrk", (4000, 4000))
    d.set_exec(split_pct=50, engine=1)
    g = E.desc_builtin("gemm", (4000, 4000, 4000))
    g.set_exec(split_pct=50, engine=1)
    # syrk = the gemm-shaped SIMT kernel(s) + the A -> A^T layout pass
    assert E.launches_per_run(d, (16, 1024, 16)) == E.launches_per_run(g, (16, 1024, 16)) + 1
    (ps,) = E.plan(d, (16, 1024, 16))
    (pg,) = E.plan(g, (16, 1024, 16))
    assert (ps.block_x, ps.block_y, ps.rm, ps.rn, ps.vec) == (pg.block_x, pg.block_y, pg.rm, pg.rn, pg.vec)


# ------------------------------------------------------------------ warp alignment in the executor
@pytest.mark.parametrize("waf", [4, 8, 16, 32])
@pytest.mark.parametrize("tiles", [(16, 1024, 16), (32, 512, 48), (64, 64, 64), (4, 4, 4), (7, 13, 5),
                                   (1024, 1024, 16)])
def test_contraction_plan_honours_warp_alignment(waf, tiles):
    """exec.warp_align = WAF lays WAF lanes of every warp along l_s1 = j: the plan reports
    simt_x == WAF, the thread grid is whole warps of WAF x 32/WAF slots, and the tile is still
    covered (passes x micro-tile >= tile)."""
    d = E.desc_builtin("gemm", (4000, 4000, 4000))
    d.set_exec(split_pct=50, engine=1, warp_align=waf)
    (p,) = E.plan(d, tiles)
    assert p.simt_x == waf
    assert p.block_x % waf == 0 and p.block_y % (32 // waf) == 0
    assert (p.block_x * p.block_y) % 32 == 0 and p.block_x * p.block_y <= 1024
    Ti, Tj = min(tiles[0], 4000), min(tiles[1], 4000)
    cover_i, cover_j = p.block_y * p.rm, p.block_x * p.rn
    assert p.passes == (-(-Ti // cover_i)) * (-(-Tj // cover_j))


def test_default_layout_simt_x():
    d = E.desc_builtin("gemm", (4000, 4000, 4000))
    (p,) = E.plan(d, (16, 1024, 16))
    assert p.block_x % 32 == 0 and p.simt_x == 32
    (q,) = E.plan(d, (32, 32, 32))  # 8 lanes along j, rows below
    assert q.simt_x == q.block_x < 32


def test_exec_opts_validation():
    d = E.desc_builtin("gemm", (64, 64, 64))
    for bad in (3, 12, 64, -4):
        with pytest.raises(E.EatssError) as e:
            d.set_exec(warp_align=bad)
        assert e.value.status == _abi.EATSS_E_INVALID
    with pytest.raises(E.EatssError):
        d.set_exec(carveout_exact=2)
    d.set_exec(split_pct=0, warp_align=8, carveout_exact=1)
    assert E.last_carveout(d) == []  # no run yet


@pytest.mark.parametrize("waf", [4, 8, 16, 32])
def test_stencil_plan_reports_warp_alignment(waf):
    d = E.desc_builtin("jacobi-2d", (4000,), tsteps=10)
    d.set_exec(split_pct=50, engine=1, warp_align=waf)
    for p in E.plan(d, (16, 1024)):
        assert p.simt_x == waf  # staged path: WAF lanes of each warp along j
    d.set_exec(split_pct=50, engine=1)
    assert all(p.simt_x == 32 for p in E.plan(d, (16, 1024)))
