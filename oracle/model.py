"""EATSS tile-selection model, brute force -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may import it.
The product enumerator (csrc/model.cpp) is written independently and shares no
code with this file.

This is the *model oracle*: the non-linear integer formulation of PAPER.md §IV
(lines 86-181) written out rule by rule under "reading R" (the
same reading as SURVEY.md §8(c-2)), and maximised by evaluating EVERY point of
the tile domain -- no pruning, no search heuristics -- instead of Z3's iterative
"OBJ_{n+1} > OBJ_n" loop.  Both reach the exact maximum; Z3
returns an arbitrary optimum, we add a deterministic tie-break (rule 13).

Rules (PAPER.md citation for each):
  1  dedupe references per nest; compound R/W counts once
  2  cache-line groups -> nrefs ("references accessing distinct cache lines")
  3  cnt(l) = #groups whose stride-1 (last) subscript uses l    ("H_i ... stride-1")
  4  l_s1 = parallel loop stride-1 in most groups, ties innermost
  5  L1_set = refs stride-1 in l_s1, SH_set = the rest           (Eq. 1)
  6  V(f) = prod of T over iterators used by f
  7  B_size = prod of T over up to the first three parallel loops
  8  H(l) = cnt(l) * (WAF if l == l_s1); 0 for serial loops in >=3-D nests;
     0 for parallel loops in 2-D nests
  9  OBJ = B_size + sum H(l)*T_l, summed over nests              (Eq. 2; multi-nest sum Q15)
 10  domain: multiples of WAF in [WAF, min(T_P_B, N)]
 11  REG_SM = B_size * nrefs * FP_factor <= R_P_S
 12  M_SH <= SPLIT*L1_SH, M_L1 <= (1-SPLIT)*L1_SH, M_L2 <= L2, element units
     (P:167); SPLIT=1 swaps the L1 bound for L2/#SM; SPLIT=0 puts
     everything in the combined L1; B200 mode clamps M_SH to the opt-in
     shared memory per block (reading Q18).
 13  tie-break: max OBJ, then min sum of T on objective-free positions,
     then max T_{l_s1}, then lexicographically smallest T (reading Q16).

Pin status (tests/test_oracle_model.py):
  pinned    the worked example (unique optimum), Table II / l_s1 / nrefs,
            heat-3d 9/12 and mttkrp / conv-2d 11/12 feasible configurations (conv-2d's filter
            size 5 or 6 is the only one reading R agrees with, reading R-N9), Z3 driven as in P:179-181,
            a hand-solved space, the infeasible spaces, the tensor-mode optima derived by hand; the
            alternatives Q2 units, Q4 literal sigma, Q7 WARP scale, Q10 array / reference counts and Q11
            halo-inclusive footprints each break one of P:121 / P:153 / P:282 (Reading switch below).
  parity unpinned (our readings, held bit-exact against the C++ enumerator; their alternatives keep every
            printed fact and are measured on B200 instead, harness/readings.py): H weights (Q6), the 2-D
            H rule (Q7), the B-set order beyond three parallel loops (Q12), the tie-break (Q16); the
            split levels (Q17), the sweep sizes (Q19); the tensor-core mode (reading T) beyond Eq. 2.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

# --------------------------------------------------------------- descriptors


@dataclass(frozen=True)
class Ref:
    array: str
    # one entry per array dimension: (sorted tuple of iterator names, constant offset)
    subs: Tuple[Tuple[Tuple[str, ...], int], ...]
    write: bool = False

    def key(self):
        return (self.array, self.subs)

    def iters(self):
        s = set()
        for its, _ in self.subs:
            s.update(its)
        return frozenset(s)

    def last_iters(self):
        return frozenset(self.subs[-1][0])


@dataclass
class Loop:
    name: str
    extent: int
    parallel: bool


@dataclass
class Nest:
    loops: List[Loop]
    refs: List[Ref]


@dataclass
class Program:
    name: str
    nests: List[Nest]
    dtype_bytes: int = 4  # 4 = fp32, 8 = fp64

    @property
    def L(self) -> int:
        return max(len(n.loops) for n in self.nests)


def ref(array: str, *subs, write: bool = False) -> Ref:
    """ref('A', 'i', 'k') or ref('A', ('i', 1), 'j') -> A[i+1][j]."""
    out = []
    for s in subs:
        if isinstance(s, tuple):
            name, off = s
        else:
            name, off = s, 0
        its = tuple(sorted(name.split("+"))) if name else tuple()
        out.append((its, int(off)))
    return Ref(array, tuple(out), write)


# ------------------------------------------------------------- GPU params


@dataclass
class Gpu:
    T_P_B: int
    T_P_W: int
    R_P_S: int
    R_P_B: int
    R_P_T: int
    L1_SH: int  # bytes
    L2: int  # bytes
    n_SM: int
    max_smem_per_block: int  # bytes


# GA100 as printed in Table I + SM count from Table III.
# KB/MB read as KiB/MiB (reading Q2, pinned by the worked example).
GA100 = Gpu(T_P_B=1024, T_P_W=32, R_P_S=65536, R_P_B=65536, R_P_T=255,
            L1_SH=192 * 1024, L2=40 * 1024 * 1024, n_SM=108, max_smem_per_block=48 * 1024)

# B200 nominal values: L1+SMEM 256 KiB per SM, L2 126 MiB,
# 148 SMs, 227 KiB opt-in shared memory per block.
B200 = Gpu(T_P_B=1024, T_P_W=32, R_P_S=65536, R_P_B=65536, R_P_T=255,
           L1_SH=256 * 1024, L2=126 * 1024 * 1024, n_SM=148, max_smem_per_block=232448)


@dataclass
class Opts:
    split_pct: int = 50
    waf: int = 16
    mode: int = 1  # 0 = paper mode, 1 = B200 mode (SMEM clamp)


@dataclass(frozen=True)
class Reading:
    """Alternative readings of the ambiguous model text.

    Reading R (every default) is the library's; each field names the passage it reads and its
    alternatives, so tests can show which alternatives the paper's own numbers exclude (P:121,
    P:153) and the harness can measure what the rest would pick.
      h_count   Q6  "number of times each loop iterator appears in the stride-1 dimension":
                'group' (distinct cache-line groups, R), 'array' (arrays), 'ref' (deduped references)
      nrefs     Q10 "references accessing distinct cache lines": 'group' (R), 'array', 'ref'
      rule2d    Q7  2-D sub-case: 'R' (parallel loops 0, the serial loop unscaled),
                'none' (no 2-D rule: the >=3-D rule applies), 'scaled' (as R, the serial loop x WAF)
      waf_scale Q7  CMA scaling: 'waf' (R; "2 x 16") or 'warp' (T_P_W = 32)
      footprint Q11 data tile of a reference: 'nohalo' (R: product of T over its iterators)
                or 'halo' (per array dimension sum of T over its iterators - (n-1) + offset span)
      bset      Q12 "up to the first three outer parallel loop dimensions":
                'ls1_outer' (R: l_s1, then outermost others), 'outer' (the three outermost),
                'ls1_inner' (l_s1, then innermost others)
      split     Q4  sigma = 0 / 1: 'R' (0: one combined L1; 1: L1 bound by L2/#SM)
                or 'literal' (the printed inequalities at every sigma)
      units     Q2  KB / MB: 'KiB' (R) or 'KB' (powers of 1000)
      tiebreak  Q16 Z3's arbitrary optimum: 'R' (rule 13), 'lexmin', 'lexmax'
    """
    h_count: str = "group"
    nrefs: str = "group"
    rule2d: str = "R"
    waf_scale: str = "waf"
    footprint: str = "nohalo"
    bset: str = "ls1_outer"
    split: str = "R"
    units: str = "KiB"
    tiebreak: str = "R"


R = Reading()


# ------------------------------------------------------------- derivation


@dataclass
class Derived:
    loops: List[Loop]
    refs: List[Ref]  # deduped
    nrefs: int
    cnt: Dict[str, int]
    ls1: str
    l1_refs: List[Ref]
    sh_refs: List[Ref]
    l1_fp: List[frozenset]  # footprints (iterator sets)
    sh_fp: List[frozenset]
    all_fp: List[frozenset]
    bset: List[str]
    H: Dict[str, int]
    # per footprint (parallel to l1_fp / sh_fp): array dimensions as (iterator names, offset span)
    l1_dims: List[tuple] = field(default_factory=list)
    sh_dims: List[tuple] = field(default_factory=list)


def derive(nest: Nest, waf: int, rd: Reading = R) -> Derived:
    loops = nest.loops
    depth = len(loops)
    # rule 1: dedupe
    seen, refs = set(), []
    for r in nest.refs:
        if r.key() not in seen:
            seen.add(r.key())
            refs.append(r)
    # rule 2: cache-line groups
    groups = set()
    for r in refs:
        groups.add((r.array, r.subs[:-1], r.last_iters()))
    arrays = {r.array for r in refs}
    nrefs = {"group": len(groups), "array": len(arrays), "ref": len(refs)}[rd.nrefs]
    # rule 3: counts (Q6: over groups, arrays or references)
    if rd.h_count == "group":
        cnt = {l.name: sum(1 for g in groups if l.name in g[2]) for l in loops}
    elif rd.h_count == "array":
        cnt = {l.name: sum(1 for a in arrays if any(r.array == a and l.name in r.last_iters() for r in refs))
               for l in loops}
    else:
        cnt = {l.name: sum(1 for r in refs if l.name in r.last_iters()) for l in loops}
    # rule 4: CMA loop
    cands = [(cnt[l.name], d, l.name) for d, l in enumerate(loops) if l.parallel and cnt[l.name] > 0]
    if not cands:
        cands = [(cnt[l.name], d, l.name) for d, l in enumerate(loops)]
    ls1 = max(cands)[2]
    # rule 5: sets
    l1_refs = [r for r in refs if ls1 in r.last_iters()]
    sh_refs = [r for r in refs if ls1 not in r.last_iters()]

    def fps(rs):
        out, dims = [], []
        for r in rs:
            f = (r.array, r.iters())
            per_dim = [(its, off, off) for its, off in r.subs]
            if f not in out:
                out.append(f)
                dims.append(per_dim)
            else:  # widen the offset range of each dimension (halo reading, Q11)
                k = out.index(f)
                dims[k] = [(its, min(lo, off), max(hi, off)) for (its, lo, hi), (_, off) in zip(dims[k], r.subs)]
        return out, [tuple((its, hi - lo) for its, lo, hi in dd) for dd in dims]

    l1_fp, l1_dims = fps(l1_refs)
    sh_all, sh_dims_all = fps(sh_refs)
    keep = [k for k, f in enumerate(sh_all) if f not in l1_fp]
    sh_fp = [sh_all[k] for k in keep]
    sh_dims = [sh_dims_all[k] for k in keep]
    all_fp = l1_fp + sh_fp
    # rule 7: B-set (Q12)
    par = [l.name for l in loops if l.parallel]
    if rd.bset == "outer":
        bset = par[:3]
    elif rd.bset == "ls1_inner":
        bset = ([ls1] if ls1 in par else []) + [p for p in reversed(par) if p != ls1]
        bset = bset[:3]
    else:
        bset = ([ls1] if ls1 in par else []) + [p for p in par if p != ls1]
        bset = bset[:3]
    # rule 8: weights (Q7)
    scale = waf if rd.waf_scale == "waf" else 32
    H = {}
    for l in loops:
        h = cnt[l.name] * (scale if l.name == ls1 else 1)
        if depth >= 3 and not l.parallel:
            h = 0
        if depth == 2 and rd.rule2d != "none":
            if l.parallel:
                h = 0
            elif rd.rule2d == "scaled":
                h = cnt[l.name] * scale
        if depth == 2 and rd.rule2d == "none" and not l.parallel:
            h = 0
        H[l.name] = h
    return Derived(loops, refs, nrefs, cnt, ls1, l1_refs, sh_refs,
                   [f[1] for f in l1_fp], [f[1] for f in sh_fp], [f[1] for f in all_fp], bset, H,
                   l1_dims, sh_dims)


def table2(nest: Nest, waf: int = 16):
    """Per-reference Table II row: (ref, memory, cma, T-reuse loops, S-reuse loops)."""
    d = derive(nest, waf)
    rows = []
    for r in d.refs:
        mem = "L1" if r in d.l1_refs else "SH"
        cma = d.ls1 in r.last_iters()
        t_reuse = [l.name for l in d.loops if l.name not in r.iters()]
        s_reuse = [l.name for l in d.loops if l.name in r.last_iters()]
        rows.append((r, mem, cma, t_reuse, s_reuse))
    return rows


# ------------------------------------------------------------- capacities


def caps(gpu: Gpu, opts: Opts, e: int, rd: Reading = R):
    """Element-unit capacities (rule 12). Returns dict with possibly-None entries."""
    pct = opts.split_pct
    L1_SH, L2 = gpu.L1_SH, gpu.L2
    if rd.units == "KB":  # Q2: the printed KB / MB as powers of 1000
        L1_SH, L2 = L1_SH // 1024 * 1000, L2 // (1024 * 1024) * 1000 * 1000
    c = {}
    if rd.split == "literal":
        c["all_l1"] = None
        c["l1"] = ((100 - pct) * L1_SH) // (100 * e)
        c["sh"] = (pct * L1_SH) // (100 * e)
    elif pct == 0:
        c["all_l1"] = (L1_SH) // e  # L1 u SH footprints share the whole L1
        c["l1"] = None
        c["sh"] = None
    elif pct == 100:
        c["all_l1"] = None
        c["l1"] = L2 // (gpu.n_SM * e)
        c["sh"] = L1_SH // e
    else:
        c["all_l1"] = None
        c["l1"] = ((100 - pct) * L1_SH) // (100 * e)
        c["sh"] = (pct * L1_SH) // (100 * e)
    c["l2"] = L2 // e
    if opts.mode == 1:
        clamp = gpu.max_smem_per_block // e
        c["sh"] = clamp if c["sh"] is None else min(c["sh"], clamp)
        if pct == 0 and rd.split != "literal":
            c["sh"] = None  # SH set lives in L1 when no shared memory is carved out
    return c


def domain(extent: int, gpu: Gpu, waf: int) -> List[int]:
    hi = min(gpu.T_P_B, extent)
    d = list(range(waf, hi + 1, waf))
    if not d:
        d = [extent]  # reading Q13
    return d


# ------------------------------------------------------------- evaluation


@dataclass
class Result:
    tiles: Optional[Tuple[int, ...]]
    obj: int
    n_feasible: int
    n_ties: int
    ties: List[Tuple[int, ...]] = field(default_factory=list)


def _prod(T, names, pos):
    v = np.ones_like(T[0])
    for n in names:
        v = v * T[pos[n]]
    return v


def _volume(T, pos, f, dims, rd: Reading):
    """V^f: reading R -- product of T over the reference's iterators; halo reading (Q11) --
    per array dimension the extent sum(T) - (n - 1) + offset span."""
    if rd.footprint == "nohalo":
        return _prod(T, f, pos)
    v = np.ones_like(T[0])
    for its, span in dims:
        if not its:
            continue
        ext = sum(T[pos[n]] for n in its) - (len(its) - 1) + span
        v = v * ext
    return v


def evaluate(prog: Program, gpu: Gpu, opts: Opts, T: Sequence[np.ndarray], rd: Reading = R):
    """Vectorised rules 6-12 over arrays of tile values T[p] (one array per position).

    Returns (feasible bool array, OBJ int64 array)."""
    e = prog.dtype_bytes
    fpf = 1 if e == 4 else 2
    c = caps(gpu, opts, e, rd)
    feas = np.ones(T[0].shape, dtype=bool)
    obj = np.zeros(T[0].shape, dtype=np.int64)
    for nest in prog.nests:
        d = derive(nest, opts.waf, rd)
        pos = {l.name: p for p, l in enumerate(nest.loops)}
        Bn = _prod(T, d.bset, pos)
        # rule 11
        feas &= Bn * d.nrefs * fpf <= gpu.R_P_S
        # rule 12
        ml1 = sum((_volume(T, pos, f, dd, rd) for f, dd in zip(d.l1_fp, d.l1_dims)), np.zeros_like(Bn))
        msh = sum((_volume(T, pos, f, dd, rd) for f, dd in zip(d.sh_fp, d.sh_dims)), np.zeros_like(Bn))
        mall = ml1 + msh
        if c["all_l1"] is not None:
            feas &= mall <= c["all_l1"]
        if c["l1"] is not None:
            feas &= ml1 <= c["l1"]
        if c["sh"] is not None:
            feas &= msh <= c["sh"]
        feas &= mall <= c["l2"]
        # rules 8-9
        obj = obj + Bn
        for l in nest.loops:
            if d.H[l.name]:
                obj = obj + d.H[l.name] * T[pos[l.name]]
    return feas, obj


def objective_free_positions(prog: Program, waf: int, rd: Reading = R) -> List[int]:
    free = []
    for p in range(prog.L):
        ok = True
        for nest in prog.nests:
            if p >= len(nest.loops):
                continue
            d = derive(nest, waf, rd)
            name = nest.loops[p].name
            if d.H[name] != 0 or name in d.bset:
                ok = False
        if ok:
            free.append(p)
    return free


def extents(prog: Program) -> List[int]:
    L = prog.L
    ex = [0] * L
    for nest in prog.nests:
        for p, l in enumerate(nest.loops):
            ex[p] = max(ex[p], l.extent)
    return ex


# ------------------------------------------------------------- tensor-core mode (mode 2)
# Reading T: the same objective (Eq. 2) and tie-break,
# over MMA-legal tiles of the tcgen05 executor, with the register / L1 / SH capacities
# replaced by the resources that executor actually uses:
#   T1  applies to nests of depth 3 with one serial (reduction) loop and l_s1 parallel;
#   T2  domain: l_s1 (UMMA N) in {16, 32, ..., min(256, roundup16(N))}; the other B-set loop
#       (UMMA M rows: one CTA or a CTA pair) in {128, 256}; the serial loop (k per pipeline stage,
#       whole 128-byte swizzle atoms of fp32) in {32, 64};
#   T4  the 6-D contraction pattern (ccsd_t_d1: one serial loop, three M-side and three N-side loops,
#       _evaluate_tensor_6d): the executor's rows / columns / shared-memory budget instead of T2-T3.
#   T3  per nest, CG = T_M / 128 CTAs per tile:
#       legality: T_{l_s1} / CG a multiple of 16 (UMMA N per CTA half);
#       TMEM: two fp32 accumulator buffers of T_{l_s1} columns, 2*T_{l_s1} <= 512;
#       SMEM: 2 stages x {hi, lo} x e x (sum of the per-CTA input footprints) <= max_smem_per_block
#       - 2048, a footprint taken per CTA (T_M -> 128, T_{l_s1} -> T_{l_s1} / CG) and, for an
#       operand whose last subscript is l_s1 (MN-major on the tensor core), its l_s1 extent
#       rounded up to the 32-column swizzle atom.

TMEM_COLS = 512
SMEM_RESERVE = 2048  # barriers + 1024-byte alignment of the stage ring


def _contraction_sets(nest: Nest):
    """Depth >= 4 with one serial loop k and two read-only inputs X, Y sharing only k (T4): returns
    (M-set loops of the input whose iterators contain l_s1, in loop order; N-set loops; k), else None."""
    serial = [l.name for l in nest.loops if not l.parallel]
    if len(nest.loops) < 4 or len(serial) != 1:
        return None
    k = serial[0]
    d = derive(nest, 16)
    written = {r.array for r in nest.refs if r.write}
    ins = []
    for r in d.refs:
        if r.array not in written and r.iters() not in [x.iters() for x in ins]:
            ins.append(r)
    if len(ins) != 2:
        return None
    a, b = ins
    if a.iters() & b.iters() != {k} or (a.iters() | b.iters()) != {l.name for l in nest.loops}:
        return None
    x, y = (a, b) if d.ls1 in a.iters() else (b, a)
    if d.ls1 not in x.iters():
        return None
    order = [l.name for l in nest.loops]
    mset = [n for n in order if n in x.iters() and n != k]
    nset = [n for n in order if n in y.iters() and n != k]
    return mset, nset, k


def tensor_applicable(prog: Program):
    """'3d' (T1: depth-3 nests, one serial loop, l_s1 parallel), '6d' (T4: the 6-D contraction pattern
    of the ccsd executor: three M-side and three N-side loops), or False."""
    if all(len(n.loops) == 3 for n in prog.nests):
        for nest in prog.nests:
            if sum(1 for l in nest.loops if not l.parallel) != 1:
                return False
            d = derive(nest, 16)
            if not nest.loops[[l.name for l in nest.loops].index(d.ls1)].parallel:
                return False
        return "3d"
    if len(prog.nests) == 1:
        cs = _contraction_sets(prog.nests[0])
        if cs and len(cs[0]) == 3 and len(cs[1]) == 3:
            return "6d"
    return False


def tensor_domains(prog: Program, mode: int = 2):
    n0 = prog.nests[0]
    d = derive(n0, 16)
    doms = []
    ex = extents(prog)
    if tensor_applicable(prog) == "6d":
        mset, nset, k = _contraction_sets(n0)
        for p, l in enumerate(n0.loops):
            if l.name == k:
                doms.append([ex[p]])                                  # whole reduction in TMEM
            elif l.name == d.ls1:
                doms.append(list(range(4, ex[p] + 1, 4)))             # 16-byte TMA rows of the output
            elif l.name == nset[0]:
                doms.append([1])                                      # one outer N-side index per unit
            elif l.name == nset[-1]:
                doms.append(list(range(16, min(256, ex[p]) + 1, 16)) or [16])  # UMMA N granules
            else:
                doms.append(list(range(1, ex[p] + 1)))
        return doms
    for p, l in enumerate(n0.loops):
        if l.name == d.ls1:
            hi = min(256, -(-ex[p] // 16) * 16)
            doms.append(list(range(16, hi + 1, 16)))
        elif l.parallel:
            doms.append([128, 256])
        else:
            doms.append([32, 64] if mode == 2 else [64, 128])  # whole 128-byte atoms of fp32 / fp16
    return doms


def _evaluate_tensor_6d(prog: Program, gpu: Gpu, opts: Opts, T):
    """T4 (reading T for the 6-D contraction): MMA rows M = product of the M-side tiles
    <= 128 TMEM lanes; columns N = product of the N-side tiles, a multiple of 16, <= 256; a middle N-side
    tile > 1 needs whole innermost N-side and l_s1 tiles (one TMA box per unit); TMEM: an accumulator
    buffer (N rounded up to a power of two >= 32) next to the 128 columns of the A operand; shared memory:
    three epilogue groups' output tiles (M*N*e rounded to 1 KB) + two stages of the N-side operand (hi, lo;
    k in 32-element atoms) <= max_smem_per_block - 1536.  B (the parallelism term) = M * N, the output
    tile of one CTA (on the tensor core every parallel loop maps into it; for depth 3 it equals Ti*Tj).
    T4-H: the H weights count only the references streamed per unit (see below)."""
    e = prog.dtype_bytes
    nest = prog.nests[0]
    d = derive(nest, opts.waf)
    mset, nset, k = _contraction_sets(nest)
    pos = {l.name: p for p, l in enumerate(nest.loops)}
    ex = {l.name: l.extent for l in nest.loops}
    M = _prod(T, mset, pos)
    N = _prod(T, nset, pos)
    feas = (M <= 128) & (N <= 256) & (N % 16 == 0) & (T[pos[nset[-1]]] <= ex[nset[-1]])
    feas &= ex[d.ls1] % 4 == 0  # 16-byte rows of the output tile
    feas &= ~((T[pos[nset[1]]] > 1) & ((T[pos[nset[-1]]] != ex[nset[-1]]) | (T[pos[d.ls1]] != ex[d.ls1])))
    bstride = np.maximum(32, 2 ** np.ceil(np.log2(np.maximum(N, 1))).astype(np.int64))
    feas &= bstride <= 384
    kext = ex[k]
    feas &= (kext <= 64) & (kext % 4 == 0)
    x_stage = -(-(M * N * e) // 1024) * 1024
    v_stage = 2 * (-(-kext // 32)) * N * 128
    feas &= 3 * x_stage + 2 * v_stage <= gpu.max_smem_per_block - 1536
    # T4-H: the M-side operand is resident in TMEM across every unit of its tile (read from HBM once
    # per A tile), so only the streamed references -- the output and the N-side operand -- earn the
    # stride-1 (CMA) weight of Eq. 2: H is derived on the nest without the M-side operand
    written = {r.array for r in nest.refs if r.write}
    x_arr = next(r.array for r in d.refs if r.array not in written and set(mset) <= set(r.iters()))
    Hs = derive(Nest(nest.loops, [r for r in nest.refs if r.array != x_arr]), opts.waf).H
    obj = M * N
    for l in nest.loops:
        if Hs[l.name]:
            obj = obj + Hs[l.name] * T[pos[l.name]]
    return feas, obj


def evaluate_tensor(prog: Program, gpu: Gpu, opts: Opts, T):
    """T1-T3 (mode 2: the 3xTF32 engine) or T5 (mode 3: the 3xFP16 engine -- 2-byte operands, B staged
    K-major by its transposing split, so no 32-column rounding and N per CTA half in multiples of 8)."""
    if tensor_applicable(prog) == "6d":
        return _evaluate_tensor_6d(prog, gpu, opts, T)
    f16 = opts.mode == 3
    e = 2 if f16 else prog.dtype_bytes
    feas = np.ones(T[0].shape, dtype=bool)
    obj = np.zeros(T[0].shape, dtype=np.int64)
    for nest in prog.nests:
        d = derive(nest, opts.waf)
        pos = {l.name: p for p, l in enumerate(nest.loops)}
        rows = [l.name for l in nest.loops if l.parallel and l.name != d.ls1][0]  # UMMA M loop
        cg = T[pos[rows]] // 128
        n_cta = T[pos[d.ls1]] // cg
        feas &= (T[pos[d.ls1]] % cg == 0) & (n_cta % (8 if f16 else 16) == 0)     # T3 legality
        feas &= 2 * T[pos[d.ls1]] <= TMEM_COLS                                      # T3 TMEM
        written = {r.array for r in nest.refs if r.write}
        inputs = []
        for r in d.refs:
            f = (r.array, r.iters())
            if r.array not in written and f not in [x[:2] for x in inputs]:
                inputs.append((r.array, r.iters(), d.ls1 in r.last_iters()))
        vin = np.zeros_like(T[0])
        for _, its, mn_major in inputs:
            v = np.ones_like(T[0])
            for it in its:
                if it == rows:
                    v = v * 128
                elif it == d.ls1:
                    v = v * (-(-n_cta // 32) * 32 if (mn_major and not f16) else n_cta)
                else:
                    v = v * T[pos[it]]
            vin = vin + v
        feas &= 2 * 2 * e * vin <= gpu.max_smem_per_block - SMEM_RESERVE           # T3 SMEM
        obj = obj + _prod(T, d.bset, pos)                                           # Eq. 2
        for l in nest.loops:
            if d.H[l.name]:
                obj = obj + d.H[l.name] * T[pos[l.name]]
    return feas, obj


def select_tiles(prog: Program, gpu: Gpu, opts: Opts, keep_ties: bool = True, rd: Reading = R) -> Result:
    """Exhaustive maximisation of OBJ over the whole domain (no pruning); `rd` selects the reading."""
    L = prog.L
    tensor = opts.mode in (2, 3)
    if tensor and not tensor_applicable(prog):
        return Result(None, 0, 0, 0, [])
    if opts.mode == 3 and tensor_applicable(prog) != "3d":
        return Result(None, 0, 0, 0, [])  # the 3xFP16 engine runs the depth-3 contractions only
    doms = ([np.array(v, dtype=np.int64) for v in tensor_domains(prog, opts.mode)] if tensor else
            [np.array(domain(n, gpu, opts.waf), dtype=np.int64) for n in extents(prog)])
    free = objective_free_positions(prog, opts.waf, rd)
    if tensor and tensor_applicable(prog) == "6d":  # T4: objective-free = outside the CTA tile (the reduction)
        k = _contraction_sets(prog.nests[0])[2]
        free = [p for p, l in enumerate(prog.nests[0].loops) if l.name == k and not derive(prog.nests[0], opts.waf).H[k]]
    ls1_pos = [l.name for l in prog.nests[0].loops].index(derive(prog.nests[0], opts.waf, rd).ls1)
    best_key, best, ties, n_feas = None, None, [], 0
    # iterate the first position in Python, the rest as one numpy meshgrid block
    rest = np.meshgrid(*doms[1:], indexing="ij") if L > 1 else []
    rest = [r.ravel() for r in rest]
    for t0 in doms[0]:
        T = [np.full(rest[0].shape if rest else (1,), t0, dtype=np.int64)] + rest
        feas, obj = evaluate_tensor(prog, gpu, opts, T) if tensor else evaluate(prog, gpu, opts, T, rd)
        n_feas += int(feas.sum())
        if not feas.any():
            continue
        idx = np.nonzero(feas)[0]
        o = obj[idx]
        omax = int(o.max())
        if best is not None and omax < best:
            continue
        sel = idx[o == omax]
        cand = [tuple(int(T[p][k]) for p in range(L)) for k in sel]
        if best is None or omax > best:
            best, ties = omax, cand
        else:
            ties.extend(cand)

    if best is None:
        return Result(None, 0, 0, 0, [])

    def key(t):
        return (sum(t[p] for p in free), -t[ls1_pos], t)

    if rd.tiebreak == "lexmin":
        ties.sort()
    elif rd.tiebreak == "lexmax":
        ties.sort(reverse=True)
    else:
        ties.sort(key=key)
    return Result(ties[0], best, n_feas, len(ties), ties if keep_ties else [])


# ------------------------------------------------------------- builtins


def P(name: str, nests: List[Nest], dtype_bytes: int = 4) -> Program:
    return Program(name, nests, dtype_bytes)


def matmul_paper(n: int = 1024, dtype_bytes: int = 8) -> Program:
    """Fig. 4 matmul Out[i][j] += In[i][k] * Ker[k][j]."""
    return P("matmul", [Nest(
        [Loop("i", n, True), Loop("j", n, True), Loop("k", n, False)],
        [ref("Out", "i", "j", write=True), ref("Out", "i", "j"), ref("In", "i", "k"), ref("Ker", "k", "j")],
    )], dtype_bytes)


def gemm(ni=4000, nj=4000, nk=4000, dtype_bytes=4) -> Program:
    return P("gemm", [Nest(
        [Loop("i", ni, True), Loop("j", nj, True), Loop("k", nk, False)],
        [ref("C", "i", "j", write=True), ref("C", "i", "j"), ref("A", "i", "k"), ref("B", "k", "j")],
    )], dtype_bytes)


def two_mm(ni=4000, nj=4000, nk=4000, nl=4000, dtype_bytes=4) -> Program:
    n1 = Nest([Loop("i", ni, True), Loop("j", nj, True), Loop("k", nk, False)],
              [ref("tmp", "i", "j", write=True), ref("A", "i", "k"), ref("B", "k", "j")])
    n2 = Nest([Loop("i", ni, True), Loop("j", nl, True), Loop("k", nj, False)],
              [ref("D", "i", "j", write=True), ref("tmp", "i", "k"), ref("C", "k", "j")])
    return P("2mm", [n1, n2], dtype_bytes)


def three_mm(ni=4000, nj=4000, nk=4000, nl=4000, nm=4000, dtype_bytes=4) -> Program:
    n1 = Nest([Loop("i", ni, True), Loop("j", nj, True), Loop("k", nk, False)],
              [ref("E", "i", "j", write=True), ref("A", "i", "k"), ref("B", "k", "j")])
    n2 = Nest([Loop("i", nj, True), Loop("j", nl, True), Loop("k", nm, False)],
              [ref("F", "i", "j", write=True), ref("C", "i", "k"), ref("D", "k", "j")])
    n3 = Nest([Loop("i", ni, True), Loop("j", nl, True), Loop("k", nj, False)],
              [ref("G", "i", "j", write=True), ref("E", "i", "k"), ref("F", "k", "j")])
    return P("3mm", [n1, n2, n3], dtype_bytes)


def syrk(ni=4000, nj=4000, dtype_bytes=4) -> Program:
    return P("syrk", [Nest(
        [Loop("i", ni, True), Loop("j", ni, True), Loop("k", nj, False)],
        [ref("C", "i", "j", write=True), ref("A", "i", "k"), ref("A", "j", "k")],
    )], dtype_bytes)


def jacobi2d(n=4000, dtype_bytes=4) -> Program:
    """jacobi-2d-imper: compute nest + copy nest; time loop excluded (Q14)."""
    m = n - 2  # interior extent
    c = Nest([Loop("i", m, True), Loop("j", m, True)],
             [ref("B", "i", "j", write=True), ref("A", "i", "j"), ref("A", "i", ("j", -1)),
              ref("A", "i", ("j", 1)), ref("A", ("i", 1), "j"), ref("A", ("i", -1), "j")])
    cp = Nest([Loop("i", m, True), Loop("j", m, True)],
              [ref("A", "i", "j", write=True), ref("B", "i", "j")])
    return P("jacobi-2d", [c, cp], dtype_bytes)


def heat3d(n=120, dtype_bytes=4) -> Program:
    """heat-3d: one sweep nest (B = f(A)); the A = f(B) nest is identical in shape."""
    m = n - 2
    loops = [Loop("i", m, True), Loop("j", m, True), Loop("k", m, True)]

    def sweep(dst, src):
        return Nest(list(loops), [
            ref(dst, "i", "j", "k", write=True),
            ref(src, ("i", 1), "j", "k"), ref(src, "i", "j", "k"), ref(src, ("i", -1), "j", "k"),
            ref(src, "i", ("j", 1), "k"), ref(src, "i", ("j", -1), "k"),
            ref(src, "i", "j", ("k", 1)), ref(src, "i", "j", ("k", -1)),
        ])

    return P("heat-3d", [sweep("B", "A"), sweep("A", "B")], dtype_bytes)


def ccsd_t_d1(d=48, dtype_bytes=4) -> Program:
    names = ["h3", "h2", "h1", "p6", "p5", "p4", "h7"]
    loops = [Loop(nm, d, nm != "h7") for nm in names]
    return P("ccsd_t_d1", [Nest(loops, [
        ref("t3", "h3", "h2", "h1", "p6", "p5", "p4", write=True),
        ref("t2", "h7", "p4", "p5", "h1"),
        ref("v2", "h3", "h2", "p6", "h7"),
    ])], dtype_bytes)


def fdtd2d(nx=1000, ny=1000, dtype_bytes=8) -> Program:
    """PolyBench fdtd-2d nests (for the nrefs = 4 pin)."""
    n1 = Nest([Loop("i", nx - 1, True), Loop("j", ny, True)],
              [ref("ey", "i", "j", write=True), ref("hz", "i", "j"), ref("hz", ("i", -1), "j")])
    n2 = Nest([Loop("i", nx, True), Loop("j", ny - 1, True)],
              [ref("ex", "i", "j", write=True), ref("hz", "i", "j"), ref("hz", "i", ("j", -1))])
    n3 = Nest([Loop("i", nx - 1, True), Loop("j", ny - 1, True)],
              [ref("hz", "i", "j", write=True), ref("ex", "i", ("j", 1)), ref("ex", "i", "j"),
               ref("ey", ("i", 1), "j"), ref("ey", "i", "j")])
    return P("fdtd-2d", [n1, n2, n3], dtype_bytes)


# Low-dimensional PolyBench 3.2 kernels (Fig. 7): 2-deep nests
# (i, j), the reduction loop not parallel (reading R-N7).
def mvt(n=4000, dtype_bytes=4) -> Program:
    loops = [Loop("i", n, True), Loop("j", n, False)]
    n1 = Nest(list(loops), [ref("x1", "i", write=True), ref("x1", "i"), ref("A", "i", "j"), ref("y_1", "j")])
    n2 = Nest(list(loops), [ref("x2", "i", write=True), ref("x2", "i"), ref("A", "j", "i"), ref("y_2", "j")])
    return P("mvt", [n1, n2], dtype_bytes)


def atax(nx=4000, ny=4000, dtype_bytes=4) -> Program:
    n1 = Nest([Loop("i", nx, True), Loop("j", ny, False)],
              [ref("tmp", "i", write=True), ref("tmp", "i"), ref("A", "i", "j"), ref("x", "j")])
    n2 = Nest([Loop("i", nx, False), Loop("j", ny, True)],
              [ref("y", "j", write=True), ref("y", "j"), ref("A", "i", "j"), ref("tmp", "i")])
    return P("atax", [n1, n2], dtype_bytes)


def bicg(nx=4000, ny=4000, dtype_bytes=4) -> Program:
    n1 = Nest([Loop("i", nx, False), Loop("j", ny, True)],
              [ref("s", "j", write=True), ref("s", "j"), ref("r", "i"), ref("A", "i", "j")])
    n2 = Nest([Loop("i", nx, True), Loop("j", ny, False)],
              [ref("q", "i", write=True), ref("q", "i"), ref("A", "i", "j"), ref("p", "j")])
    return P("bicg", [n1, n2], dtype_bytes)


def gemver(n=4000, dtype_bytes=4) -> Program:
    n1 = Nest([Loop("i", n, True), Loop("j", n, True)],
              [ref("A", "i", "j", write=True), ref("A", "i", "j"), ref("u1", "i"), ref("v1", "j"),
               ref("u2", "i"), ref("v2", "j")])
    n2 = Nest([Loop("i", n, True), Loop("j", n, False)],
              [ref("x", "i", write=True), ref("x", "i"), ref("A", "j", "i"), ref("y", "j")])
    n3 = Nest([Loop("i", n, True)], [ref("x", "i", write=True), ref("x", "i"), ref("z", "i")])
    n4 = Nest([Loop("i", n, True), Loop("j", n, False)],
              [ref("w", "i", write=True), ref("w", "i"), ref("A", "i", "j"), ref("x", "j")])
    return P("gemver", [n1, n2, n3, n4], dtype_bytes)


# Non-PolyBench 4-D kernels (Figs. 10-11): our restatement
# (reading R-N8, R-N9).  Reduction loops are not parallel.
def mttkrp(ni=512, nj=32, nk=512, nl=512, dtype_bytes=4) -> Program:
    """A[i][j] += B[i][k][l] * C[k][j] * D[l][j]  (mode-1 MTTKRP, loops i, j, k, l)."""
    return P("mttkrp", [Nest(
        [Loop("i", ni, True), Loop("j", nj, True), Loop("k", nk, False), Loop("l", nl, False)],
        [ref("A", "i", "j", write=True), ref("A", "i", "j"), ref("B", "i", "k", "l"),
         ref("C", "k", "j"), ref("D", "l", "j")],
    )], dtype_bytes)


def conv2d(n=8192, f=5, dtype_bytes=4) -> Program:
    """out[i][j] += inp[i+p][j+q] * W[p][q]  (valid 2-D cross-correlation, loops i, j, p, q)."""
    m = n - f + 1
    return P("conv-2d", [Nest(
        [Loop("i", m, True), Loop("j", m, True), Loop("p", f, False), Loop("q", f, False)],
        [ref("out", "i", "j", write=True), ref("out", "i", "j"), ref("inp", "i+p", "j+q"), ref("W", "p", "q")],
    )], dtype_bytes)


BUILTINS = {
    "gemm": gemm, "2mm": two_mm, "3mm": three_mm, "syrk": syrk,
    "jacobi-2d": jacobi2d, "heat-3d": heat3d, "ccsd_t_d1": ccsd_t_d1,
    "mvt": mvt, "atax": atax, "bicg": bicg, "gemver": gemver,
    "mttkrp": mttkrp, "conv-2d": conv2d,
}
