// model.cpp -- the EATSS non-linear integer tile model (§IV),
// re-evaluated for B200 limits and maximised by exhaustive enumeration with
// monotone pruning instead of Z3's iterative search.
//
// Reading R rule by rule; each function cites the passage:
//   derive_nest   rules 1-8   (Table II)
//   capacities    rule 12
//   enumerate     rules 9-13  (Eq. 2, tie-break Q16)
// Every constraint left-hand side is a sum of products of tile sizes, hence
// monotone non-decreasing in every T_p: with unassigned positions set to their
// smallest domain value, a violated constraint stays violated for every larger
// value, so the DFS stops the loop at that depth (exact, no approximation).
#include <algorithm>
#include <chrono>
#include <cstring>
#include <set>
#include <tuple>

#include "desc.hpp"

namespace eatss {

static int popcount32(uint32_t x) { return __builtin_popcount(x); }

// Rules 1-8 for one nest.
NestModel derive_nest(const Nest &n, int waf) {
    const int depth = (int)n.loops.size();
    NestModel m;
    // rule 1 -- dedupe: (array, subscripts) identical => one reference
    std::vector<const Ref *> refs;
    auto same = [](const Ref &a, const Ref &b) {
        if (a.array != b.array || a.subs.size() != b.subs.size()) return false;
        for (size_t i = 0; i < a.subs.size(); i++)
            if (a.subs[i].iters != b.subs[i].iters || a.subs[i].off != b.subs[i].off) return false;
        return true;
    };
    for (const Ref &r : n.refs) {
        bool dup = false;
        for (const Ref *q : refs) dup = dup || same(*q, r);
        if (!dup) refs.push_back(&r);
    }
    // rule 2 -- cache-line groups: (array, all-but-last subscripts with offsets,
    // iterator set of the last subscript) ("distinct cache lines")
    std::set<std::vector<int64_t>> groups;
    for (const Ref *r : refs) {
        std::vector<int64_t> key{r->array};
        for (size_t i = 0; i + 1 < r->subs.size(); i++) {
            key.push_back(r->subs[i].iters);
            key.push_back(r->subs[i].off);
        }
        key.push_back(-1);
        key.push_back(r->subs.back().iters);
        groups.insert(key);
    }
    m.nrefs = (int)groups.size();
    // rule 3 -- cnt(l): groups whose stride-1 subscript uses loop l
    m.cnt.assign(depth, 0);
    for (const auto &g : groups) {
        uint32_t last = (uint32_t)g.back();
        for (int p = 0; p < depth; p++)
            if (last & (1u << p)) m.cnt[p]++;
    }
    // rule 4 -- l_s1: parallel loop with the largest count, ties -> innermost
    int best = -1;
    for (int p = 0; p < depth; p++) {
        if (!n.loops[p].parallel || m.cnt[p] == 0) continue;
        if (best < 0 || m.cnt[p] > m.cnt[best] || (m.cnt[p] == m.cnt[best] && p > best)) best = p;
    }
    if (best < 0) {
        for (int p = 0; p < depth; p++)
            if (best < 0 || m.cnt[p] > m.cnt[best] || (m.cnt[p] == m.cnt[best] && p > best)) best = p;
    }
    m.ls1 = best;
    // rule 5 -- L1_set / SH_set (Eq. 1); footprints deduped per (array, iterators)
    std::vector<std::pair<int, uint32_t>> l1, sh;
    auto all_iters = [](const Ref *r) {
        uint32_t s = 0;
        for (const Sub &x : r->subs) s |= x.iters;
        return s;
    };
    for (const Ref *r : refs) {
        std::pair<int, uint32_t> f{r->array, all_iters(r)};
        bool in_l1 = (r->subs.back().iters >> m.ls1) & 1u;
        auto &dst = in_l1 ? l1 : sh;
        if (std::find(dst.begin(), dst.end(), f) == dst.end()) dst.push_back(f);
    }
    for (auto &f : l1) m.l1_fp.push_back(f.second);
    for (auto &f : sh)
        if (std::find(l1.begin(), l1.end(), f) == l1.end()) m.sh_fp.push_back(f.second);
    // rule 7 -- B-set: l_s1 (if parallel) then the outermost other parallel loops, <= 3
    int nb = 0;
    if (n.loops[m.ls1].parallel) {
        m.bset |= 1u << m.ls1;
        nb++;
    }
    for (int p = 0; p < depth && nb < 3; p++) {
        if (p == m.ls1 || !n.loops[p].parallel) continue;
        m.bset |= 1u << p;
        nb++;
    }
    // rule 8 -- H weights
    m.H.assign(depth, 0);
    for (int p = 0; p < depth; p++) {
        int64_t h = (int64_t)m.cnt[p] * (p == m.ls1 ? waf : 1);
        if (depth >= 3 && !n.loops[p].parallel) h = 0;
        if (depth == 2 && n.loops[p].parallel) h = 0;
        m.H[p] = h;
    }
    return m;
}

std::vector<int64_t> program_extents(const eatss_kernel_desc &d) {
    size_t L = 0;
    for (const Nest &n : d.nests) L = std::max(L, n.loops.size());
    std::vector<int64_t> ex(L, 0);
    for (const Nest &n : d.nests)
        for (size_t p = 0; p < n.loops.size(); p++) ex[p] = std::max(ex[p], n.loops[p].extent);
    return ex;
}

namespace {

struct Caps {
    int64_t all_l1 = -1, l1 = -1, sh = -1, l2 = -1;  // -1 = no such constraint
};

// rule 12: capacities in element units, integer floors
Caps capacities(const eatss_gpu_params &g, const eatss_model_opts &o, int e) {
    Caps c;
    const int64_t pct = o.split_pct;
    if (pct == 0) {
        c.all_l1 = g.l1_shared_bytes / e;
    } else if (pct == 100) {
        c.l1 = g.l2_bytes / (g.num_sms * e);  // L2 per SM replaces L1
        c.sh = g.l1_shared_bytes / e;
    } else {
        c.l1 = ((100 - pct) * g.l1_shared_bytes) / (100 * e);
        c.sh = (pct * g.l1_shared_bytes) / (100 * e);
    }
    c.l2 = g.l2_bytes / e;
    if (o.mode == 1 && pct != 0) {
        int64_t clamp = g.max_smem_per_block / e;
        c.sh = std::min(c.sh, clamp);
    }
    return c;
}

struct NestEval {
    const Nest *nest;
    NestModel m;
    std::vector<uint32_t> in_fp;  // tensor mode: footprints of the arrays the nest only reads
    std::vector<char> in_mn;      // ... whose last subscript uses l_s1 (MN-major tensor-core operand)
    int rows_pos = -1;            // tensor mode: the parallel loop that is not l_s1 (UMMA M)
};

// Tensor-core mode (reading T): the executor stages every input footprint in
// shared memory (2 stages x {hi, lo}) and keeps two fp32 accumulators of T_{l_s1} TMEM columns.
void input_footprints(NestEval &ne) {
    const Nest &n = *ne.nest;
    std::vector<int> written;
    for (const Ref &r : n.refs)
        if (r.write) written.push_back(r.array);
    std::vector<std::pair<int, uint32_t>> seen;
    for (const Ref &r : n.refs) {
        if (std::find(written.begin(), written.end(), r.array) != written.end()) continue;
        uint32_t it = 0;
        for (const Sub &s : r.subs) it |= s.iters;
        std::pair<int, uint32_t> f{r.array, it};
        if (std::find(seen.begin(), seen.end(), f) != seen.end()) continue;
        seen.push_back(f);
        ne.in_fp.push_back(it);
        ne.in_mn.push_back((r.subs.back().iters >> ne.m.ls1) & 1u ? 1 : 0);
    }
    for (int p = 0; p < (int)n.loops.size(); p++)
        if (n.loops[p].parallel && p != ne.m.ls1) {
            ne.rows_pos = p;
            break;
        }
}
// T4 (reading T for the 6-D contraction pattern): one serial loop k, two read-only
// inputs sharing only k; M-side = the loops of the input that uses l_s1, N-side = the other input's.
struct Sets6 {
    bool ok = false;
    std::vector<int> m, n;  // loop positions, outermost first
    int k = -1;
    std::vector<int64_t> H;  // T4-H: Eq. 2 weights without the M-side (TMEM-resident) operand
};
Sets6 contraction_sets(const NestEval &ne, int waf) {
    Sets6 r;
    const Nest &n = *ne.nest;
    const int L = (int)n.loops.size();
    int serial = 0;
    for (int p = 0; p < L; p++)
        if (!n.loops[p].parallel) { serial++; r.k = p; }
    if (L < 4 || serial != 1 || ne.in_fp.size() != 2) return r;
    const uint32_t a = ne.in_fp[0], b = ne.in_fp[1], kb = 1u << r.k, all = (1u << L) - 1u;
    if ((a & b) != kb || (a | b) != all) return r;
    const uint32_t x = ((a >> ne.m.ls1) & 1u) ? a : b, y = x == a ? b : a;
    if (!((x >> ne.m.ls1) & 1u)) return r;
    for (int p = 0; p < L; p++) {
        if (p == r.k) continue;
        if ((x >> p) & 1u) r.m.push_back(p);
        if ((y >> p) & 1u) r.n.push_back(p);
    }
    r.ok = r.m.size() == 3 && r.n.size() == 3;
    // T4-H: the M-side operand stays in TMEM across all units of its tile (read once per A tile), so only
    // the streamed references (output, N-side operand) earn the stride-1 weight: H of the nest without it
    int x_array = -1;
    for (const Ref &rf : n.refs) {
        uint32_t it = 0;
        for (const Sub &sb : rf.subs) it |= sb.iters;
        if (!rf.write && it == x) x_array = rf.array;
    }
    Nest reduced;
    reduced.loops = n.loops;
    for (const Ref &rf : n.refs)
        if (rf.array != x_array) reduced.refs.push_back(rf);
    r.H = derive_nest(reduced, waf).H;
    return r;
}
constexpr int64_t kTmemCols = 512;

struct Search {
    int L = 0;
    std::vector<std::vector<int64_t>> dom;
    std::vector<NestEval> nests;
    Caps caps;
    int64_t regs = 0;
    int fpf = 1;
    uint32_t free_mask = 0;
    int ls1_pos = 0;
    // result
    std::vector<int64_t> T, best;
    int64_t best_obj = -1, best_free = 0, n_feasible = 0, n_ties = 0;
    bool found = false;

    static int64_t prod(const std::vector<int64_t> &T, uint32_t mask) {
        int64_t v = 1;
        for (int p = 0; mask; p++, mask >>= 1)
            if (mask & 1u) v *= T[p];
        return v;
    }

    bool tensor = false, tensor6 = false, f16 = false;  // f16: mode 3 (the 3xFP16 engine)
    Sets6 s6;                        // tensor6: M-side / N-side / reduction positions
    std::vector<int64_t> ext;        // loop extents
    int64_t smem_cap = 0;
    int esz = 4;

    bool feasible(const std::vector<int64_t> &T) const {
        if (tensor6) {  // reading T4: the ccsd executor's rows, columns and shared memory
            int64_t M = 1, N = 1;
            for (int p : s6.m) M *= T[p];
            for (int p : s6.n) N *= T[p];
            const int ls1 = nests[0].m.ls1, inner = s6.n.back(), mid = s6.n[1];
            if (M > 128 || N > 256 || N % 16 || T[inner] > ext[inner] || ext[ls1] % 4) return false;
            if (T[mid] > 1 && (T[inner] != ext[inner] || T[ls1] != ext[ls1])) return false;
            int64_t bstride = 32;
            while (bstride < N) bstride *= 2;
            if (bstride > 384) return false;  // one accumulator buffer next to the 128 A columns
            const int64_t kx = ext[s6.k];
            if (kx > 64 || kx % 4) return false;
            const int64_t x_stage = (M * N * esz + 1023) / 1024 * 1024, v_stage = 2 * ((kx + 31) / 32) * N * 128;
            return 3 * x_stage + 2 * v_stage <= smem_cap - 1536;
        }
        if (tensor) {  // reading T3
            for (const NestEval &ne : nests) {
                const int64_t tn = T[ne.m.ls1], cg = T[ne.rows_pos] / 128;
                if (cg < 1 || tn % cg || (tn / cg) % (f16 ? 8 : 16)) return false;  // UMMA N per CTA half
                if (2 * tn > kTmemCols) return false;                   // two fp32 accumulator buffers
                const int64_t n_cta = tn / cg;
                int64_t vin = 0;
                for (size_t f = 0; f < ne.in_fp.size(); f++) {
                    int64_t v = 1;
                    for (int p = 0; p < L; p++) {
                        if (!((ne.in_fp[f] >> p) & 1u)) continue;
                        if (p == ne.rows_pos) v *= 128;  // per-CTA rows
                        else if (p == ne.m.ls1) v *= (ne.in_mn[f] && !f16) ? (n_cta + 31) / 32 * 32 : n_cta;
                        else v *= T[p];
                    }
                    vin += v;
                }
                if (2 * 2 * esz * vin > smem_cap - 2048) return false;  // 2 stages x {hi, lo}
            }
            return true;
        }
        for (const NestEval &ne : nests) {
            const NestModel &m = ne.m;
            const int64_t B = prod(T, m.bset);
            if (B * m.nrefs * fpf > regs) return false;  // rule 11
            int64_t ml1 = 0, msh = 0;
            for (uint32_t f : m.l1_fp) ml1 += prod(T, f);
            for (uint32_t f : m.sh_fp) msh += prod(T, f);
            if (caps.all_l1 >= 0 && ml1 + msh > caps.all_l1) return false;
            if (caps.l1 >= 0 && ml1 > caps.l1) return false;
            if (caps.sh >= 0 && msh > caps.sh) return false;
            if (ml1 + msh > caps.l2) return false;
        }
        return true;
    }

    int64_t objective(const std::vector<int64_t> &T) const {  // Eq. 2, summed over nests
        int64_t obj = 0;
        for (const NestEval &ne : nests) {
            if (tensor6) {  // T4: the parallelism term is the CTA's output tile M x N
                int64_t M = 1, N = 1;
                for (int p : s6.m) M *= T[p];
                for (int p : s6.n) N *= T[p];
                obj += M * N;
                for (size_t p = 0; p < s6.H.size(); p++) obj += s6.H[p] * T[p];
                continue;
            }
            obj += prod(T, ne.m.bset);
            for (size_t p = 0; p < ne.m.H.size(); p++) obj += ne.m.H[p] * T[p];
        }
        return obj;
    }

    // rule 13: is candidate T better than the incumbent (both with OBJ == best_obj)?
    bool better_tie(const std::vector<int64_t> &T, int64_t fsum) const {
        if (fsum != best_free) return fsum < best_free;
        if (T[ls1_pos] != best[ls1_pos]) return T[ls1_pos] > best[ls1_pos];
        return T < best;  // lexicographically smallest
    }

    void leaf() {
        n_feasible++;
        const int64_t obj = objective(T);
        int64_t fsum = 0;
        for (int p = 0; p < L; p++)
            if ((free_mask >> p) & 1u) fsum += T[p];
        if (!found || obj > best_obj) {
            found = true;
            best_obj = obj;
            best = T;
            best_free = fsum;
            n_ties = 1;
        } else if (obj == best_obj) {
            n_ties++;
            if (better_tie(T, fsum)) {
                best = T;
                best_free = fsum;
            }
        }
    }

    void dfs(int p) {
        if (p == L) {
            leaf();
            return;
        }
        for (int64_t v : dom[p]) {
            T[p] = v;
            if (tensor) {  // reading T's legality is not monotone: enumerate the (small) space whole
                if (p + 1 == L) {
                    if (feasible(T)) leaf();
                } else {
                    dfs(p + 1);
                }
                continue;
            }
            // positions > p sit at their minimum; monotone constraints => break
            if (!feasible(T)) break;
            dfs(p + 1);
        }
        T[p] = dom[p].front();
    }
};

}  // namespace
}  // namespace eatss

using namespace eatss;

extern "C" eatss_status eatss_select_tiles(const eatss_kernel_desc *d, const eatss_gpu_params *g,
                                           const eatss_model_opts *o, int64_t *tiles,
                                           eatss_model_report *rep) {
    if (!d || !g || !o || !tiles) return fail(EATSS_E_INVALID, "eatss_select_tiles: null argument");
    if (o->split_pct < 0 || o->split_pct > 100)
        return fail(EATSS_E_INVALID, "eatss_select_tiles: split_pct must be in 0..100");
    if (o->warp_align <= 0 || o->warp_align > 1024)
        return fail(EATSS_E_INVALID, "eatss_select_tiles: warp_align must be in 1..1024");
    if (g->num_sms <= 0 || g->l1_shared_bytes <= 0 || g->l2_bytes <= 0 || g->regs_per_sm <= 0 ||
        g->threads_per_block <= 0)
        return fail(EATSS_E_INVALID, "eatss_select_tiles: bad gpu params");
    auto t0 = std::chrono::steady_clock::now();
    Search s;
    const std::vector<int64_t> ext = program_extents(*d);
    s.L = (int)ext.size();
    const int e = dtype_bytes(d->dtype);
    s.fpf = (e == 8) ? 2 : 1;  // FP_factor
    s.regs = g->regs_per_sm;
    s.caps = capacities(*g, *o, e);
    for (const Nest &n : d->nests) {
        NestEval ne;
        ne.nest = &n;
        ne.m = derive_nest(n, o->warp_align);
        input_footprints(ne);
        s.nests.push_back(ne);
    }
    s.ext = ext;
    if (o->mode == 3 && !(s.nests.size() >= 1 && s.nests[0].nest->loops.size() == 3))
        return fail(EATSS_E_UNSUPPORTED, "eatss_select_tiles: mode 3 (3xFP16 engine) needs depth-3 contraction nests");
    if (o->mode == 2 && s.nests.size() == 1 && s.nests[0].nest->loops.size() >= 4) {
        // tensor-core mode T4: the 6-D contraction pattern of the ccsd executor
        s.s6 = contraction_sets(s.nests[0], o->warp_align);
        if (!s.s6.ok)
            return fail(EATSS_E_UNSUPPORTED, "eatss_select_tiles: tensor mode needs a depth-3 contraction or the "
                                             "6-D contraction pattern (one reduction loop, 3 + 3 output loops)");
        s.tensor = s.tensor6 = true;
        s.esz = e;
        s.smem_cap = g->max_smem_per_block;
        const int ls1 = s.nests[0].m.ls1;
        for (int p = 0; p < s.L; p++) {
            std::vector<int64_t> dm;
            if (p == s.s6.k) {
                dm = {ext[p]};  // the whole reduction stays in TMEM
            } else if (p == ls1) {
                for (int64_t v = 4; v <= ext[p]; v += 4) dm.push_back(v);  // 16-byte output rows
            } else if (p == s.s6.n.front()) {
                dm = {1};  // one outer N-side index per unit
            } else if (p == s.s6.n.back()) {
                for (int64_t v = 16; v <= std::min<int64_t>(256, ext[p]); v += 16) dm.push_back(v);  // UMMA N granules
            } else {
                for (int64_t v = 1; v <= ext[p]; v++) dm.push_back(v);
            }
            if (dm.empty()) dm.push_back(16);
            s.dom.push_back(dm);
        }
    } else if (o->mode == 2 || o->mode == 3) {
        // tensor-core mode: depth-3 nests with one serial loop and a parallel l_s1 only
        for (const NestEval &ne : s.nests) {
            int serial = 0;
            for (const Loop &l : ne.nest->loops) serial += l.parallel ? 0 : 1;
            if (ne.nest->loops.size() != 3 || serial != 1 || !ne.nest->loops[ne.m.ls1].parallel)
                return fail(EATSS_E_UNSUPPORTED, "eatss_select_tiles: tensor mode needs depth-3 contraction nests");
        }
        s.tensor = true;
        s.f16 = o->mode == 3;
        s.esz = s.f16 ? 2 : e;
        s.smem_cap = g->max_smem_per_block;
        const Nest &n0 = d->nests[0];
        for (int p = 0; p < s.L; p++) {
            std::vector<int64_t> dm;
            if (p == s.nests[0].m.ls1) {  // UMMA N: multiples of 16 up to 256
                const int64_t hi = std::min<int64_t>(256, ((ext[p] + 15) / 16) * 16);
                for (int64_t v = 16; v <= hi; v += 16) dm.push_back(v);
            } else if (n0.loops[p].parallel) {
                dm = {128, 256};  // UMMA M rows: one CTA (cta_group::1) or a CTA pair (cta_group::2)
            } else {
                dm = s.f16 ? std::vector<int64_t>{64, 128} : std::vector<int64_t>{32, 64};  // whole 128-byte atoms
            }
            s.dom.push_back(dm);
        }
    } else {
        // rule 10 -- domain: multiples of WAF in [WAF, min(T_P_B, N)]; N < WAF -> {N}
        for (int p = 0; p < s.L; p++) {
            std::vector<int64_t> dm;
            const int64_t hi = std::min<int64_t>(g->threads_per_block, ext[p]);
            for (int64_t v = o->warp_align; v <= hi; v += o->warp_align) dm.push_back(v);
            if (dm.empty()) dm.push_back(ext[p]);
            s.dom.push_back(dm);
        }
    }
    // objective-free positions: H == 0 and outside the B-set in every nest; T4: outside
    // the CTA tile, i.e. the reduction loop
    for (int p = 0; p < s.L; p++) {
        bool fr = true;
        for (const NestEval &ne : s.nests) {
            if (p >= (int)ne.nest->loops.size()) continue;
            const bool in_b = s.tensor6 ? p != s.s6.k : ((ne.m.bset >> p) & 1u) != 0;
            const int64_t h = s.tensor6 ? s.s6.H[p] : ne.m.H[p];
            if (h != 0 || in_b) fr = false;
        }
        if (fr) s.free_mask |= 1u << p;
    }
    s.ls1_pos = s.nests[0].m.ls1;
    s.T.resize(s.L);
    for (int p = 0; p < s.L; p++) s.T[p] = s.dom[p].front();
    s.dfs(0);
    double secs = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    if (rep) {
        std::memset(rep, 0, sizeof(*rep));
        rep->ls1_loop = s.ls1_pos;
        for (const NestEval &ne : s.nests) rep->nrefs = std::max(rep->nrefs, ne.m.nrefs);
        rep->n_feasible = s.n_feasible;
        rep->n_ties = s.n_ties;
        rep->solve_seconds = secs;
        if (s.found) {
            rep->obj = s.best_obj;
            for (const NestEval &ne : s.nests) {
                int64_t ml1 = 0, msh = 0;
                for (uint32_t f : ne.m.l1_fp) ml1 += Search::prod(s.best, f);
                for (uint32_t f : ne.m.sh_fp) msh += Search::prod(s.best, f);
                const int64_t B = Search::prod(s.best, ne.m.bset);
                rep->m_l1 = std::max(rep->m_l1, ml1);
                rep->m_sh = std::max(rep->m_sh, msh);
                rep->b_size = std::max(rep->b_size, B);
                rep->reg_sm = std::max(rep->reg_sm, B * ne.m.nrefs * s.fpf);
            }
        }
    }
    if (!s.found)
        return fail(EATSS_E_INFEASIBLE, "eatss_select_tiles: no tile vector satisfies the constraints");
    for (int p = 0; p < s.L; p++) tiles[p] = s.best[p];
    return EATSS_OK;
}

extern "C" eatss_status eatss_desc_model_info(const eatss_kernel_desc *d, int nest, int waf,
                                              int32_t *ls1, int32_t *nrefs, int64_t *H) {
    if (!d || nest < 0 || nest >= (int)d->nests.size() || waf <= 0)
        return fail(EATSS_E_INVALID, "eatss_desc_model_info: bad nest or waf");
    NestModel m = derive_nest(d->nests[nest], waf);
    if (ls1) *ls1 = m.ls1;
    if (nrefs) *nrefs = m.nrefs;
    if (H)
        for (size_t p = 0; p < m.H.size(); p++) H[p] = m.H[p];
    return EATSS_OK;
}
