// ccsd_fast.cuh -- register-resident fast path of the 6-D contraction (included by ccsd.cu).
//
// Per CTA tile (rows R = (h3,h2,p6), cols C = (h1,p5,p4), reduction h7):
//   * per-CTA offset tables in shared memory replace all div/mod index decoding:
//     t3 row / column parts, the v2 row part, the t2 column part, and a permutation of
//     the columns into h1-fastest order so that t2 (stride-1 in h1) is gathered with
//     consecutive lanes on consecutive addresses, and v2 (stride-1 in h7) likewise;
//   * the SH_set tiles v2(R x h7) -- stored transposed -- and t2(h7 x C) go through an
//     S-stage cp.async ring, so the gather of h7-tile t+S-1 overlaps the FMAs of t;
//   * a thread owns rm contiguous rows x rn columns (16-byte column vectors when
//     p4 is 4-aligned): shared-memory reads are broadcasts / conflict-free vectors;
//   * acc accumulates -sum_h7 v2*t2 from 0; the epilogue adds it to t3 with 16-byte
//     loads and stores (t3, the L1_set reference, is read and written exactly once).
#pragma once

struct CcsdFastArgs {
    float *__restrict__ t3;
    const float *__restrict__ t2;
    const float *__restrict__ v2;
    int64_t H3, H2, H1, P6, P5, P4, H7;
    int T[7];
    int nt_h1, nt_p5, nt_p4, nt_h2, nt_p6;
    int Rt, Ct, rtp, ctp, S;
    int kst;  // h7 per pipeline stage (multiple of the tile's Th7)
    int t3s_off;  // float offset of the t3 tile prefetch buffer in smem, -1 = none
    int64_t h3_off;
};

__device__ __forceinline__ void cpa4f(void *smem, const void *gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(gmem));
}

template <int RM, int RN, int V>
__global__ void __launch_bounds__(RM * RN >= 32 ? 512 : 1024) ccsd_fast_kernel(const CcsdFastArgs p) {
    extern __shared__ __align__(16) float smf[];
    constexpr int VN = RN / V;
    const int tx = threadIdx.x, ty = threadIdx.y, BX = blockDim.x;
    const int tid = ty * BX + tx, nthr = BX * blockDim.y;
    // Th7 here is the pipeline stage extent: kst = a whole number of the tile's h7-tiles
    // (T[6]) grouped so a stage covers >= 16 h7 -- numerically identical (register-resident
    // accumulators, h7 ascending), fewer barriers for the small EATSS h7 tile.
    const int Th3 = p.T[0], Th2 = p.T[1], Th1 = p.T[2], Tp6 = p.T[3], Tp5 = p.T[4], Tp4 = p.T[5], Th7 = p.kst;
    (void)Th3;
    const int stage_elems = Th7 * (p.rtp + p.ctp);
    float *ring = smf;
    int64_t *t3row = reinterpret_cast<int64_t *>(smf + ((p.S * stage_elems + 1) & ~1));
    int64_t *v2row = t3row + p.Rt;
    int32_t *t3col = reinterpret_cast<int32_t *>(v2row + p.Rt);
    int32_t *t2col = t3col + p.Ct;
    int32_t *perm = t2col + p.Ct;

    // tile origin
    int bx = blockIdx.x;
    const int64_t p4_0 = (int64_t)(bx % p.nt_p4) * Tp4; bx /= p.nt_p4;
    const int64_t p5_0 = (int64_t)(bx % p.nt_p5) * Tp5; bx /= p.nt_p5;
    const int64_t h1_0 = (int64_t)bx * Th1;
    int by = blockIdx.y;
    const int64_t p6_0 = (int64_t)(by % p.nt_p6) * Tp6; by /= p.nt_p6;
    const int64_t h2_0 = (int64_t)(by % p.nt_h2) * Th2; by /= p.nt_h2;
    const int64_t h3_0 = p.h3_off + (int64_t)by * Th3;
    const int64_t s_p5 = p.P4, s_p6 = p.P5 * p.P4, s_h1 = p.P6 * s_p6, s_h2 = p.H1 * s_h1, s_h3 = p.H2 * s_h2;
    const int64_t t2_k = p.P4 * p.P5 * p.H1;  // t2 stride of h7

    for (int rl = tid; rl < p.Rt; rl += nthr) {
        const int a = rl % Tp6, b = (rl / Tp6) % Th2, c = rl / (Tp6 * Th2);
        const int64_t h3 = h3_0 + c, h2 = h2_0 + b, p6 = p6_0 + a;
        const bool ok = h3 < p.H3 && h2 < p.H2 && p6 < p.P6;
        t3row[rl] = ok ? h3 * s_h3 + h2 * s_h2 + p6 * s_p6 : -1;
        v2row[rl] = ok ? ((h3 * p.H2 + h2) * p.P6 + p6) * p.H7 : -1;
    }
    for (int cl = tid; cl < p.Ct; cl += nthr) {
        const int a = cl % Tp4, b = (cl / Tp4) % Tp5, c = cl / (Tp4 * Tp5);
        const int64_t h1 = h1_0 + c, p5 = p5_0 + b, p4 = p4_0 + a;
        const bool ok = h1 < p.H1 && p5 < p.P5 && p4 < p.P4;
        t3col[cl] = ok ? (int32_t)(h1 * s_h1 + p5 * s_p5 + p4) : -1;
        t2col[cl] = ok ? (int32_t)((p4 * p.P5 + p5) * p.H1 + h1) : -1;
        // gather order: s = ((p4l * Tp5) + p5l) * Th1 + h1l  (h1 fastest = t2's stride-1)
        const int s = (a * Tp5 + b) * Th1 + c;
        perm[s] = cl;
    }
    __syncthreads();

    const int nk = (int)((p.H7 + Th7 - 1) / Th7);
    const int wv_o = tid / Th7, wv_i = tid - (tid / Th7) * Th7, wv_do = nthr / Th7, wv_di = nthr - (nthr / Th7) * Th7;
    const int wt_o = tid / p.Ct, wt_i = tid - (tid / p.Ct) * p.Ct, wt_do = nthr / p.Ct,
              wt_di = nthr - (nthr / p.Ct) * p.Ct;
    // Per-thread staging assignments, fixed across stages (registers, no table lookups in the
    // loop): t2 columns s = tid + j*nthr (all kk of a stage), v2 elements (rl, kk) = tid + j*nthr.
    constexpr int MAXP = 4;
    const bool fixed = (p.Ct <= MAXP * nthr) && (p.Rt * Th7 <= MAXP * nthr);
    int t2cl[MAXP], t2tc[MAXP], v2rl[MAXP], v2kk[MAXP];
    int64_t v2vr[MAXP];
#pragma unroll
    for (int j = 0; j < MAXP; j++) {
        const int s = tid + j * nthr;
        t2cl[j] = -1; t2tc[j] = -1;
        if (fixed && s < p.Ct) { t2cl[j] = perm[s]; t2tc[j] = t2col[t2cl[j]]; }
        const int e = tid + j * nthr;
        v2rl[j] = -1; v2kk[j] = 0; v2vr[j] = -1;
        if (fixed && e < p.Rt * Th7) { v2rl[j] = e / Th7; v2kk[j] = e - v2rl[j] * Th7; v2vr[j] = v2row[v2rl[j]]; }
    }

    auto stage = [&](int t) {
        if (t < nk && fixed) {
            float *VsT = ring + (t % p.S) * stage_elems;
            float *Ts = VsT + Th7 * p.rtp;
            const int64_t k0 = (int64_t)t * Th7;
            const int kt = (int)min((int64_t)Th7, p.H7 - k0);
#pragma unroll
            for (int j = 0; j < MAXP; j++) {
                if (v2rl[j] >= 0) {
                    float *dst = VsT + v2kk[j] * p.rtp + v2rl[j];
                    if (v2vr[j] >= 0 && v2kk[j] < kt) cpa4f(dst, p.v2 + v2vr[j] + k0 + v2kk[j]);
                    else *dst = 0.f;
                }
                if (t2cl[j] >= 0) {
                    const float *src = p.t2 + k0 * t2_k + t2tc[j];
                    for (int kk = 0; kk < Th7; kk++) {
                        float *dst = Ts + kk * p.ctp + t2cl[j];
                        if (t2tc[j] >= 0 && kk < kt) cpa4f(dst, src + kk * t2_k);
                        else *dst = 0.f;
                    }
                }
            }
        } else if (t < nk) {
            float *VsT = ring + (t % p.S) * stage_elems;
            float *Ts = VsT + Th7 * p.rtp;
            const int64_t k0 = (int64_t)t * Th7;
            const int kt = (int)min((int64_t)Th7, p.H7 - k0);
            // division-free walks: (outer, inner) advanced by (nthr / inner, nthr % inner)
            for (int rl = wv_o, kk = wv_i; rl < p.Rt;) {  // (rl, kk), kk fastest: v2 stride-1 in h7
                const int64_t vr = v2row[rl];
                if (vr >= 0 && kk < kt) cpa4f(VsT + kk * p.rtp + rl, p.v2 + vr + k0 + kk);
                else VsT[kk * p.rtp + rl] = 0.f;
                rl += wv_do; kk += wv_di;
                if (kk >= Th7) { kk -= Th7; rl++; }
            }
            for (int kk = wt_o, s = wt_i; kk < Th7;) {  // (kk, s), s fastest: t2 stride-1 in h1
                const int cl = perm[s];
                const int32_t tc = t2col[cl];
                if (tc >= 0 && kk < kt) cpa4f(Ts + kk * p.ctp + cl, p.t2 + (k0 + kk) * t2_k + tc);
                else Ts[kk * p.ctp + cl] = 0.f;
                kk += wt_do; s += wt_di;
                if (s >= p.Ct) { s -= p.Ct; kk++; }
            }
        }
        asm volatile("cp.async.commit_group;\n" ::);
    };

    float acc[RM][RN];
#pragma unroll
    for (int r = 0; r < RM; r++)
#pragma unroll
        for (int c = 0; c < RN; c++) acc[r][c] = 0.f;
    const int r0 = min(ty * RM, p.rtp - RM);
    int cc[VN];
#pragma unroll
    for (int c = 0; c < VN; c++) cc[c] = min((tx + c * BX) * V, p.ctp - V);

    // t3 tile prefetch into shared memory, issued with the last stage so the HBM read of
    // the L1_set reference overlaps the final FMAs (epilogue reads it from smem).
    float *t3s = p.t3s_off >= 0 ? smf + p.t3s_off : nullptr;
    auto prefetch_t3 = [&]() {
        if (!t3s) return;
        const int cg = p.Ct / V;  // column groups per row
        const int o0 = tid / cg, i0 = tid - o0 * cg, dO = nthr / cg, dI = nthr - dO * cg;
        for (int rl = o0, g = i0; rl < p.Rt;) {
            const int64_t ro = t3row[rl];
            const int cl = g * V;
            const int32_t co = t3col[cl];
            if (ro >= 0 && co >= 0) {
                if constexpr (V == 4) {
                    unsigned sa = (unsigned)__cvta_generic_to_shared(t3s + rl * p.Ct + cl);
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(p.t3 + ro + co));
                } else {
                    cpa4f(t3s + rl * p.Ct + cl, p.t3 + ro + co);
                }
            }
            rl += dO; g += dI;
            if (g >= cg) { g -= cg; rl++; }
        }
    };

    for (int s = 0; s < p.S - 1; s++) {
        if (s == nk - 1) prefetch_t3();
        stage(s);
    }
    for (int t = 0; t < nk; t++) {
        if (t + p.S - 1 == nk - 1) prefetch_t3();
        stage(t + p.S - 1);
        if (p.S == 2) asm volatile("cp.async.wait_group 1;\n" ::);
        else asm volatile("cp.async.wait_group 2;\n" ::);
        __syncthreads();
        const float *VsT = ring + (t % p.S) * stage_elems;
        const float *Ts = VsT + Th7 * p.rtp;
        const int kt = (int)min((int64_t)Th7, p.H7 - (int64_t)t * Th7);
        for (int kk = 0; kk < kt; kk++) {
            float a[RM], b[RN];
            if constexpr (RM % 4 == 0) {
#pragma unroll
                for (int r = 0; r < RM; r += 4) {
                    const float4 v = *reinterpret_cast<const float4 *>(VsT + kk * p.rtp + r0 + r);
                    a[r] = v.x; a[r + 1] = v.y; a[r + 2] = v.z; a[r + 3] = v.w;
                }
            } else {
#pragma unroll
                for (int r = 0; r < RM; r++) a[r] = VsT[kk * p.rtp + r0 + r];
            }
#pragma unroll
            for (int c = 0; c < VN; c++) {
                if constexpr (V == 4) {
                    const float4 v = *reinterpret_cast<const float4 *>(Ts + kk * p.ctp + cc[c]);
                    b[4 * c] = v.x; b[4 * c + 1] = v.y; b[4 * c + 2] = v.z; b[4 * c + 3] = v.w;
                } else {
                    b[c] = Ts[kk * p.ctp + cc[c]];
                }
            }
#pragma unroll
            for (int r = 0; r < RM; r++)
#pragma unroll
                for (int c = 0; c < RN; c++) acc[r][c] = fmaf(-a[r], b[c], acc[r][c]);
        }
        __syncthreads();
    }
    asm volatile("cp.async.wait_group 0;\n" ::);
    if (t3s) __syncthreads();

    // epilogue: t3 += acc (t3 read and written once)
#pragma unroll
    for (int r = 0; r < RM; r++) {
        const int rl = ty * RM + r;
        if (rl >= p.Rt) continue;
        const int64_t ro = t3row[rl];
        if (ro < 0) continue;
#pragma unroll
        for (int c = 0; c < VN; c++) {
            const int cl = (tx + c * BX) * V;
            if (cl >= p.Ct) continue;
            const int32_t co = t3col[cl];
            if (co < 0) continue;
            if constexpr (V == 4) {
                float4 *q = reinterpret_cast<float4 *>(p.t3 + ro + co);
                float4 o = t3s ? *reinterpret_cast<const float4 *>(t3s + rl * p.Ct + cl) : *q;
                o.x += acc[r][4 * c]; o.y += acc[r][4 * c + 1]; o.z += acc[r][4 * c + 2]; o.w += acc[r][4 * c + 3];
                *q = o;
            } else {
                const float o = t3s ? t3s[rl * p.Ct + cl] : p.t3[ro + co];
                p.t3[ro + co] = o + acc[r][c];
            }
        }
    }
}
