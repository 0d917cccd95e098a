// ccsd.cu -- tiled 6-D tensor contraction executor (CCSD(T) d1, BASELINE config 5).
//
//   t3[h3][h2][h1][p6][p5][p4] -= sum_h7 t2[h7][p4][p5][h1] * v2[h3][h2][p6][h7]
//
// Tile vector (Th3, Th2, Th1, Tp6, Tp5, Tp4, Th7) over the 7-deep nest (P:125:
// one tile variable per loop dimension).  Model split for this nest (DESIGN.md
// §2.2, rules 4-5): l_s1 = p4 (stride-1 of t3), so t3 is the L1_set reference
// (read/written through L1, coalesced along p4), while t2 (stride-1 h1) and v2
// (stride-1 h7) are the SH_set: their tiles are staged in shared memory per
// h7-tile.  The nest is a contraction over h7 of a "row" index set
// R = (h3, h2, p6) with a "column" set C = (h1, p5, p4); one CTA owns a
// Th3*Th2*Tp6 x Th1*Tp5*Tp4 output tile, each thread a register micro-tile
// (rm rows x rn columns, cyclic), t3 loaded once, updated over all h7, stored
// once when the tile fits in registers (otherwise RMW per h7-tile).
// 64-bit offsets throughout: 48^6 = 1.2e10 elements.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include "contract.cuh"
#include "devsw.hpp"

namespace eatss {

struct CcsdArgs {
    float *__restrict__ t3;
    const float *__restrict__ t2;
    const float *__restrict__ v2;
    int64_t H3, H2, H1, P6, P5, P4, H7;
    int T[7];  // h3 h2 h1 p6 p5 p4 h7
    int nt_h1, nt_p5, nt_p4, nt_h2, nt_p6;  // tile counts for decoding blockIdx
    int Rt, Ct;  // tile rows / cols
    int tkp, ctp;
    int passes_i, passes_j;
    int64_t h3_off;  // first h3 of this launch (multi-GPU shard)
    int32_t *counts;
};

__device__ __forceinline__ void cpa4(void *smem, const void *gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(gmem));
}

template <int RM, int RN, int MODE>  // MODE 0 resident, 1 stream, 2 coverage
__global__ void __launch_bounds__(RM * RN >= 32 ? 512 : 1024) ccsd_d1_kernel(const CcsdArgs p) {
    extern __shared__ __align__(16) float sm[];
    float *Vs = sm;                       // [Rt][tkp]   v2 tile (rows x h7)
    float *Ts = sm + p.Rt * p.tkp;        // [Th7][ctp]  t2 tile (h7 x cols)
    // t3 offset tables of the tile: row part (h3,h2,p6) and column part (h1,p5,p4); -1 = outside
    int64_t *rowoff = reinterpret_cast<int64_t *>(Ts + p.T[6] * p.ctp + ((p.T[6] * p.ctp) & 1));
    int32_t *coloff = reinterpret_cast<int32_t *>(rowoff + p.Rt);
    const int tx = threadIdx.x, ty = threadIdx.y, BX = blockDim.x, BY = blockDim.y;
    const int tid = ty * BX + tx, nthr = BX * BY;
    const int Th3 = p.T[0], Th2 = p.T[1], Th1 = p.T[2], Tp6 = p.T[3], Tp5 = p.T[4], Tp4 = p.T[5],
              Th7 = p.T[6];
    // decode tile origin
    int bx = blockIdx.x;
    const int64_t p4_0 = (int64_t)(bx % p.nt_p4) * Tp4; bx /= p.nt_p4;
    const int64_t p5_0 = (int64_t)(bx % p.nt_p5) * Tp5; bx /= p.nt_p5;
    const int64_t h1_0 = (int64_t)bx * Th1;
    int by = blockIdx.y;
    const int64_t p6_0 = (int64_t)(by % p.nt_p6) * Tp6; by /= p.nt_p6;
    const int64_t h2_0 = (int64_t)(by % p.nt_h2) * Th2; by /= p.nt_h2;
    const int64_t h3_0 = p.h3_off + (int64_t)by * Th3;
    // strides of t3
    const int64_t s_p5 = p.P4, s_p6 = p.P5 * p.P4, s_h1 = p.P6 * s_p6, s_h2 = p.H1 * s_h1,
                  s_h3 = p.H2 * s_h2;

    // decode a local row index -> (h3, h2, p6) global; returns false if out of range
    auto row = [&](int rl, int64_t &h3, int64_t &h2, int64_t &p6) {
        const int a = rl % Tp6, b = (rl / Tp6) % Th2, c = rl / (Tp6 * Th2);
        h3 = h3_0 + c; h2 = h2_0 + b; p6 = p6_0 + a;
        return rl < p.Rt && h3 < p.H3 && h2 < p.H2 && p6 < p.P6;
    };
    auto col = [&](int cl, int64_t &h1, int64_t &p5, int64_t &p4) {
        const int a = cl % Tp4, b = (cl / Tp4) % Tp5, c = cl / (Tp4 * Tp5);
        h1 = h1_0 + c; p5 = p5_0 + b; p4 = p4_0 + a;
        return cl < p.Ct && h1 < p.H1 && p5 < p.P5 && p4 < p.P4;
    };

    const int nk = (int)((p.H7 + Th7 - 1) / Th7);
    auto stage = [&](int t) {
        const int64_t k0 = (int64_t)t * Th7;
        const int kt = (int)min((int64_t)Th7, p.H7 - k0);
        for (int e = tid; e < p.Rt * kt; e += nthr) {
            const int rl = e / kt, kk = e - rl * kt;
            int64_t h3, h2, p6;
            if (row(rl, h3, h2, p6)) cpa4(Vs + rl * p.tkp + kk, p.v2 + ((h3 * p.H2 + h2) * p.P6 + p6) * p.H7 + k0 + kk);
        }
        for (int e = tid; e < p.Ct * kt; e += nthr) {
            const int kk = e / p.Ct, cl = e - kk * p.Ct;
            int64_t h1, p5, p4;
            if (col(cl, h1, p5, p4)) cpa4(Ts + kk * p.ctp + cl, p.t2 + (((k0 + kk) * p.P4 + p4) * p.P5 + p5) * p.H1 + h1);
        }
        asm volatile("cp.async.commit_group;\n" ::);
    };

    float acc[RM][RN];
    // thread's rows / columns for pass (pi, pj)
    for (int e = tid; e < p.Rt; e += nthr) {
        int64_t h3, h2, p6;
        rowoff[e] = row(e, h3, h2, p6) ? h3 * s_h3 + h2 * s_h2 + p6 * s_p6 : -1;
    }
    for (int e = tid; e < p.Ct; e += nthr) {
        int64_t h1, p5, p4;
        coloff[e] = col(e, h1, p5, p4) ? (int32_t)(h1 * s_h1 + p5 * s_p5 + p4) : -1;
    }
    __syncthreads();

    auto run_pass = [&](int ri0, int cj0, bool load_first, bool store_last, int t_begin, int t_end) {
        // shared-memory row / column of each micro-tile entry, clamped inside the staged tile
        auto srow = [&](int r) { return min(ri0 + ty + r * BY, p.Rt - 1); };
        auto scol = [&](int c) { return min(cj0 + tx + c * BX, p.Ct - 1); };
        auto t3_off = [&](int r, int c, bool &ok) -> int64_t {
            const int rl = ri0 + ty + r * BY, cl = cj0 + tx + c * BX;
            if (rl >= p.Rt || cl >= p.Ct) { ok = false; return 0; }
            const int64_t ro = rowoff[rl];
            const int32_t co = coloff[cl];
            ok = (ro >= 0) & (co >= 0);
            return ro + co;
        };
        if constexpr (MODE != 2) {
            if (load_first) {
#pragma unroll
                for (int r = 0; r < RM; r++)
#pragma unroll
                    for (int c = 0; c < RN; c++) {
                        bool ok;
                        const int64_t o = t3_off(r, c, ok);
                        acc[r][c] = ok ? p.t3[o] : 0.f;
                    }
            }
        }
        for (int t = t_begin; t < t_end; t++) {
            const int64_t k0 = (int64_t)t * Th7;
            const int kt = (int)min((int64_t)Th7, p.H7 - k0);
            if (MODE == 0) {  // resident: stage here with a single buffer
                __syncthreads();
                stage(t);
                asm volatile("cp.async.wait_group 0;\n" ::);
                __syncthreads();
            }
            for (int kk = 0; kk < kt; kk++) {
                float a[RM], b[RN];
#pragma unroll
                for (int r = 0; r < RM; r++) a[r] = Vs[srow(r) * p.tkp + kk];
#pragma unroll
                for (int c = 0; c < RN; c++) b[c] = Ts[kk * p.ctp + scol(c)];
                if constexpr (MODE == 2) {
#pragma unroll
                    for (int r = 0; r < RM; r++)
#pragma unroll
                        for (int c = 0; c < RN; c++) {
                            bool ok;
                            // point index over the 7-D nest, row-major (h3,h2,h1,p6,p5,p4,h7)
                            const int64_t o6 = t3_off(r, c, ok);
                            if (ok) atomicAdd(p.counts + o6 * p.H7 + k0 + kk, 1);
                        }
                } else {
#pragma unroll
                    for (int r = 0; r < RM; r++)
#pragma unroll
                        for (int c = 0; c < RN; c++) acc[r][c] = fmaf(-a[r], b[c], acc[r][c]);
                }
            }
        }
        if constexpr (MODE != 2) {
            if (store_last) {
                __syncthreads();  // keeps the offset-table reads below from being hoisted
#pragma unroll
                for (int r = 0; r < RM; r++)
#pragma unroll
                    for (int c = 0; c < RN; c++) {
                        bool ok;
                        const int64_t o = t3_off(r, c, ok);
                        if (ok) p.t3[o] = acc[r][c];
                    }
            }
        }
    };

    if constexpr (MODE == 1) {
        // streaming: per h7-tile, every pass loads, updates and stores its t3 block
        for (int t = 0; t < nk; t++) {
            __syncthreads();
            stage(t);
            asm volatile("cp.async.wait_group 0;\n" ::);
            __syncthreads();
            for (int pi = 0; pi < p.passes_i; pi++)
                for (int pj = 0; pj < p.passes_j; pj++)
                    run_pass(pi * BY * RM, pj * BX * RN, true, true, t, t + 1);
        }
    } else {
        run_pass(0, 0, true, true, 0, nk);
    }
}

#include "ccsd_fast.cuh"

// ------------------------------------------------------------------ planning / launch
static inline int64_t cdiv6(int64_t a, int64_t b) { return (a + b - 1) / b; }

struct CcsdFastPlan {
    bool ok = false;
    int rm, rn, vec, bx, by, rtp, ctp, S, smem, kst, t3s_off;
};

static CcsdFastPlan plan_ccsd_fast(const int64_t *dims, const int *T, int Rt, int Ct) {
    CcsdFastPlan f;
    f.vec = (dims[5] % 4 == 0 && T[5] % 4 == 0) ? 4 : 1;
    struct MT { int rm, rn; };
    const MT c4[] = {{1, 4}, {2, 4}, {4, 4}, {4, 8}, {8, 8}};
    const MT c1[] = {{1, 1}, {1, 2}, {2, 2}, {2, 4}, {4, 4}, {4, 8}, {8, 8}};
    const MT *cand = f.vec == 4 ? c4 : c1;
    const int nc = f.vec == 4 ? 5 : 7;
    const int64_t want = cdiv6((int64_t)Rt * Ct, 512);
    int pick = 0;
    for (int c = 0; c < nc; c++) {
        if (c > 0 && (cand[c].rm > Rt || cand[c].rn > ((Ct + f.vec - 1) / f.vec) * f.vec)) continue;
        pick = c;
        if (cand[c].rm * cand[c].rn >= want) break;
    }
    f.rm = cand[pick].rm;
    f.rn = cand[pick].rn;
    const int maxt = f.rm * f.rn >= 32 ? 512 : 1024;
    const int64_t by = cdiv6(Rt, f.rm), bx = cdiv6(Ct, f.rn);
    if (by * bx > maxt) return f;
    f.by = (int)by;
    f.bx = (int)bx;
    f.rtp = ((Rt + 3) / 4) * 4 + (f.rm < 4 ? 0 : 0);
    f.ctp = ((Ct + 3) / 4) * 4;
    f.S = 3;
    int group = std::max(1, (16 + T[6] - 1) / T[6]);
    if (devsw("EATSS_CCSD_GROUP", 0) > 0) group = devsw("EATSS_CCSD_GROUP", 0);
    const bool want_prefetch = devsw("EATSS_CCSD_NOPREFETCH", 0) == 0;
    auto layout = [&](int kst, bool pre, int64_t *bytes, int *t3s_off) {
        const int64_t ring = (int64_t)f.S * kst * (f.rtp + f.ctp);
        const int64_t tab = ((ring + 1) & ~1LL);
        const int64_t t3s = ((tab + (int64_t)Rt * 4 + (int64_t)Ct * 3 + 3) & ~3LL);
        *t3s_off = pre ? (int)t3s : -1;
        *bytes = (pre ? t3s + (int64_t)Rt * Ct : t3s) * 4;
    };
    f.t3s_off = -1;
    for (int g = group; g >= 1 && want_prefetch; g--) {
        const int kst = (int)std::min<int64_t>((int64_t)T[6] * g, dims[6]);
        int64_t bytes;
        int off;
        layout(kst, true, &bytes, &off);
        if (bytes <= 227 * 1024) {
            f.kst = kst;
            f.t3s_off = off;
            f.smem = (int)bytes;
            f.ok = true;
            return f;
        }
    }
    f.kst = (int)std::min<int64_t>((int64_t)T[6] * group, dims[6]);
    int64_t bytes;
    int off;
    layout(f.kst, false, &bytes, &off);
    if (bytes > 227 * 1024) return f;
    f.smem = (int)bytes;
    f.ok = true;
    return f;
}

template <int RM, int RN, int V>
static cudaError_t ccsd_fast_launch(const CcsdFastArgs &a, const CcsdFastPlan &f, int64_t gx, int64_t gy,
                                    int carveout, cudaStream_t s) {
    auto k = ccsd_fast_kernel<RM, RN, V>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, f.smem);
    if (e != cudaSuccess) return e;
    const int cvr = cv_resolve(carveout, 50);
    cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, cvr);
    note_carveout(cvr);
    k<<<dim3((unsigned)gx, (unsigned)gy), dim3(f.bx, f.by), f.smem, s>>>(a);
    return cudaGetLastError();
}

static cudaError_t ccsd_fast_dispatch(const CcsdFastArgs &a, const CcsdFastPlan &f, int64_t gx, int64_t gy,
                                      int cv, cudaStream_t s) {
    const int key = f.vec * 10000 + f.rm * 100 + f.rn;
    switch (key) {
        case 40104: return ccsd_fast_launch<1, 4, 4>(a, f, gx, gy, cv, s);
        case 40204: return ccsd_fast_launch<2, 4, 4>(a, f, gx, gy, cv, s);
        case 40404: return ccsd_fast_launch<4, 4, 4>(a, f, gx, gy, cv, s);
        case 40408: return ccsd_fast_launch<4, 8, 4>(a, f, gx, gy, cv, s);
        case 40808: return ccsd_fast_launch<8, 8, 4>(a, f, gx, gy, cv, s);
        case 10101: return ccsd_fast_launch<1, 1, 1>(a, f, gx, gy, cv, s);
        case 10102: return ccsd_fast_launch<1, 2, 1>(a, f, gx, gy, cv, s);
        case 10202: return ccsd_fast_launch<2, 2, 1>(a, f, gx, gy, cv, s);
        case 10204: return ccsd_fast_launch<2, 4, 1>(a, f, gx, gy, cv, s);
        case 10404: return ccsd_fast_launch<4, 4, 1>(a, f, gx, gy, cv, s);
        case 10408: return ccsd_fast_launch<4, 8, 1>(a, f, gx, gy, cv, s);
        case 10808: return ccsd_fast_launch<8, 8, 1>(a, f, gx, gy, cv, s);
    }
    return cudaErrorInvalidConfiguration;
}

struct CcsdPlan {
    int T[7];
    int Rt, Ct, rm, rn, bx, by, passes_i, passes_j, tkp, ctp, smem;
    bool stream;
    int64_t gx, gy;
};

CcsdPlan plan_ccsd(const int64_t *dims, const int64_t *tiles) {
    CcsdPlan p;
    for (int d = 0; d < 7; d++) p.T[d] = (int)std::max<int64_t>(1, std::min(tiles[d], dims[d]));
    p.Rt = p.T[0] * p.T[1] * p.T[3];
    p.Ct = p.T[2] * p.T[4] * p.T[5];
    const int64_t outputs = (int64_t)p.Rt * p.Ct;
    struct MT { int rm, rn, maxt; };
    const MT cand[] = {{1, 1, 1024}, {1, 2, 1024}, {2, 2, 1024}, {2, 4, 1024}, {4, 4, 1024}, {4, 8, 512}, {8, 8, 512}};
    const int64_t want = cdiv6(outputs, 512);
    int pick = 0;
    for (int c = 0; c < 7; c++) {
        if (c > 0 && (cand[c].rm > p.Rt || cand[c].rn > p.Ct)) continue;
        pick = c;
        if (cand[c].rm * cand[c].rn >= want) break;
    }
    p.rm = cand[pick].rm;
    p.rn = cand[pick].rn;
    int64_t by = cdiv6(p.Rt, p.rm), bx = cdiv6(p.Ct, p.rn);
    if (by * bx <= cand[pick].maxt) {
        p.stream = false;
        p.bx = (int)bx; p.by = (int)by; p.passes_i = p.passes_j = 1;
    } else {
        p.stream = true;
        p.rm = 8; p.rn = 8;
        p.bx = (int)std::min<int64_t>(cdiv6(p.Ct, 8), 512);
        p.by = (int)std::max<int64_t>(1, std::min<int64_t>(cdiv6(p.Rt, 8), 512 / p.bx));
        p.passes_i = (int)cdiv6(p.Rt, (int64_t)p.by * 8);
        p.passes_j = (int)cdiv6(p.Ct, (int64_t)p.bx * 8);
    }
    p.tkp = p.T[6] + 1;
    p.ctp = p.Ct + ((p.Ct % 2 == 0) ? 1 : 0);
    p.smem = (p.Rt * p.tkp + p.T[6] * p.ctp + 1) * 4 + p.Rt * 8 + p.Ct * 4;
    p.gx = cdiv6(dims[2], p.T[2]) * cdiv6(dims[4], p.T[4]) * cdiv6(dims[5], p.T[5]);
    p.gy = cdiv6(dims[0], p.T[0]) * cdiv6(dims[1], p.T[1]) * cdiv6(dims[3], p.T[3]);
    return p;
}

template <int RM, int RN, int MODE>
static cudaError_t ccsd_launch(const CcsdArgs &a, const CcsdPlan &p, int carveout, cudaStream_t s) {
    auto k = ccsd_d1_kernel<RM, RN, MODE>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem);
    if (e != cudaSuccess) return e;
    cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, cv_resolve(carveout, 0));
    note_carveout(cv_resolve(carveout, 0));
    k<<<dim3((unsigned)p.gx, (unsigned)p.gy), dim3(p.bx, p.by), p.smem, s>>>(a);
    return cudaGetLastError();
}

template <int MODE>
static cudaError_t ccsd_mt(const CcsdArgs &a, const CcsdPlan &p, int cv, cudaStream_t s) {
    switch (p.rm * 100 + p.rn) {
        case 101: return ccsd_launch<1, 1, MODE>(a, p, cv, s);
        case 102: return ccsd_launch<1, 2, MODE>(a, p, cv, s);
        case 202: return ccsd_launch<2, 2, MODE>(a, p, cv, s);
        case 204: return ccsd_launch<2, 4, MODE>(a, p, cv, s);
        case 404: return ccsd_launch<4, 4, MODE>(a, p, cv, s);
        case 408: return ccsd_launch<4, 8, MODE>(a, p, cv, s);
        case 808: return ccsd_launch<8, 8, MODE>(a, p, cv, s);
    }
    return cudaErrorInvalidConfiguration;
}

// dims: full (H3..H7); h3_begin/h3_count select a slab of h3 (multi-GPU shard) --
// pointers are the full tensors.
cudaError_t launch_ccsd_d1(float *t3, const float *t2, const float *v2, const int64_t *dims,
                           const int64_t *tiles, int64_t h3_begin, int64_t h3_count, int carveout,
                           int32_t *counts, cudaStream_t s) {
    int64_t d2[7];
    for (int i = 0; i < 7; i++) d2[i] = dims[i];
    d2[0] = h3_count;
    CcsdPlan p = plan_ccsd(d2, tiles);
    if (p.gy > 65535 || p.gx > 2147483647LL) return cudaErrorInvalidConfiguration;
    if (!counts && devsw("EATSS_CCSD_SLOW", 0) == 0) {
        CcsdFastPlan f = plan_ccsd_fast(d2, p.T, p.Rt, p.Ct);
        if (f.ok) {
            CcsdFastArgs a;
            a.t3 = t3; a.t2 = t2; a.v2 = v2;
            a.H3 = h3_begin + h3_count; a.H2 = dims[1]; a.H1 = dims[2]; a.P6 = dims[3]; a.P5 = dims[4];
            a.P4 = dims[5]; a.H7 = dims[6];
            for (int i = 0; i < 7; i++) a.T[i] = p.T[i];
            a.nt_h1 = (int)cdiv6(dims[2], p.T[2]); a.nt_p5 = (int)cdiv6(dims[4], p.T[4]);
            a.nt_p4 = (int)cdiv6(dims[5], p.T[5]); a.nt_h2 = (int)cdiv6(dims[1], p.T[1]);
            a.nt_p6 = (int)cdiv6(dims[3], p.T[3]);
            a.Rt = p.Rt; a.Ct = p.Ct; a.rtp = f.rtp; a.ctp = f.ctp; a.S = f.S; a.kst = f.kst; a.t3s_off = f.t3s_off;
            a.h3_off = h3_begin;
            return ccsd_fast_dispatch(a, f, p.gx, p.gy, carveout, s);
        }
    }
    if (p.smem > 227 * 1024) return cudaErrorInvalidConfiguration;
    CcsdArgs a;
    a.t3 = t3; a.t2 = t2; a.v2 = v2;
    a.H3 = h3_begin + h3_count; a.H2 = dims[1]; a.H1 = dims[2]; a.P6 = dims[3]; a.P5 = dims[4];
    a.P4 = dims[5]; a.H7 = dims[6];
    for (int i = 0; i < 7; i++) a.T[i] = p.T[i];
    a.nt_h1 = (int)cdiv6(dims[2], p.T[2]); a.nt_p5 = (int)cdiv6(dims[4], p.T[4]);
    a.nt_p4 = (int)cdiv6(dims[5], p.T[5]); a.nt_h2 = (int)cdiv6(dims[1], p.T[1]);
    a.nt_p6 = (int)cdiv6(dims[3], p.T[3]);
    a.Rt = p.Rt; a.Ct = p.Ct; a.tkp = p.tkp; a.ctp = p.ctp;
    a.passes_i = p.passes_i; a.passes_j = p.passes_j;
    a.h3_off = h3_begin;
    a.counts = counts;
    if (counts) return ccsd_mt<2>(a, p, carveout, s);
    if (p.stream) return ccsd_mt<1>(a, p, carveout, s);
    return ccsd_mt<0>(a, p, carveout, s);
}

void ccsd_plan_dims(const int64_t *dims, const int64_t *tiles, int64_t *gx, int64_t *gy, int *bx,
                    int *by, int *rm, int *rn, int *passes, int *smem) {
    CcsdPlan p = plan_ccsd(dims, tiles);
    *gx = p.gx; *gy = p.gy; *bx = p.bx; *by = p.by; *rm = p.rm; *rn = p.rn;
    *passes = p.passes_i * p.passes_j; *smem = p.smem;
}

}  // namespace eatss
