// staged.cuh -- register-resident fast path of the contraction executor (included by contract.cu).
//
// Per k-tile both operand slices of the tile are brought into shared memory through
// an S-stage ring so the copy of k-tile t+S-1 overlaps the FMAs of k-tile t:
//   * the SH_set tile A(i0..i0+Ti, k0..k0+Tk) (Eq. 1) with cp.async,
//     stored transposed (A^T[k][i]) so a thread's rm rows are one 16-byte broadcast;
//   * the L1_set slice B(k0..k0+Tk, j0..j0+Tj) (stride-1 in l_s1 = j) with one
//     cp.async.bulk row copy per k (the Blackwell bulk-copy engine, completion on an
//     mbarrier with an expected transaction count) -- no thread spends instructions
//     on it -- or, for unaligned / transposed operands, with cp.async.
// A thread owns rm contiguous rows x rn columns (16-byte column vectors cyclic over
// the warp, so every B read is a conflict-free 16-byte vector); accumulators stay
// in registers across all k-tiles; the epilogue is C = beta*C + alpha*acc.
#pragma once

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

template <typename T, int RM, int RN, int V, bool TRANSB>
__global__ void __launch_bounds__((16384 / (RM * RN)) < 1024 ? (16384 / (RM * RN)) : 1024,
                                  (RM * RN == 64 && sizeof(T) == 4) ? 2 : 1)  // 8x8 fp32: two CTAs per SM (<= 128 registers)
    contract_staged_kernel(const CArgs<T> p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    constexpr int VN = RN / V;
    constexpr bool BULK = (V == 4) && !TRANSB && sizeof(T) == 4;
    T *const sm = reinterpret_cast<T *>(smem_raw);
    const int aip = p.tkp;  // A^T pitch (>= Ti, multiple of 4)
    const int bjp = p.tjp;  // B pitch (>= Tj, multiple of 4)
    // B slice: [k][j] (pitch bjp), or for a transposed operand with p.bkp > 0 untransposed [j][k]
    // rows (pitch bkp, 16-byte aligned) filled by 16-byte copies and read 4 k at a time
    const bool BT4 = TRANSB && sizeof(T) == 4 && p.bkp > 0;
    const int stage_elems = p.Tk * aip + (BT4 ? bjp * p.bkp : p.Tk * bjp);
    const int S = p.nbuf;
    uint64_t *bars = reinterpret_cast<uint64_t *>(sm + S * stage_elems);  // 8-byte aligned (elems % 2 == 0)

    const int BX = blockDim.x;
    const int tid = threadIdx.y * BX + threadIdx.x, nthr = BX * blockDim.y;
    int tx = threadIdx.x, ty = threadIdx.y;
    if (p.waf) warp_layout(tid, BX, p.waf, tx, ty);  // WAF lanes per warp along j
    // tile of this CTA (Fig. 4 mapping); with a split wave tail (p.sp > 1, 1-D grid) the last
    // tiles are cut along k into sp parts whose partial sums are added to C atomically
    const int nk = (int)((p.K + p.Tk - 1) / p.Tk);
    int64_t tile_i, tile_j;
    int ks0 = 0, nloc = nk;
    bool split = false;
    if (p.sp > 1) {
        int64_t t = blockIdx.x;
        if (t >= p.nfull) {
            const int64_t v = t - p.nfull;
            const int part = (int)(v % p.sp);
            t = p.nfull + v / p.sp;
            ks0 = (int)((int64_t)part * nk / p.sp);
            nloc = (int)((int64_t)(part + 1) * nk / p.sp) - ks0;
            split = true;
        }
        tile_i = t / p.gx;
        tile_j = t - tile_i * p.gx;
    } else {
        tile_i = blockIdx.y;
        tile_j = blockIdx.x;
    }
    const int64_t i0 = tile_i * p.Ti, j0 = tile_j * p.Tj;
    const int rows = (int)imin64(p.Ti, p.M - i0);
    const int cols = (int)imin64(p.Tj, p.N - j0);

    if constexpr (BULK) {
        if (tid == 0)
            for (int s = 0; s < S; s++) mbar_init(bars + s, 1);
        __syncthreads();
    }

    // Division-free staging walks: element e = tid + n*nthr of an (outer x inner) box is
    // tracked as (o, i) and advanced by (nthr / inner, nthr % inner).
    struct Walk {
        int o0, i0, dO, dI, inner;
    };
    auto mkwalk = [&](int inner) {
        Walk w;
        w.inner = max(inner, 1);
        w.o0 = tid / w.inner;
        w.i0 = tid - w.o0 * w.inner;
        w.dO = nthr / w.inner;
        w.dI = nthr - w.dO * w.inner;
        return w;
    };
    const Walk wa = mkwalk(p.Tk);  // A: (row, k), k fastest -> coalesced reads
    const Walk wb = TRANSB ? mkwalk(BT4 ? p.Tk >> 2 : p.Tk) : mkwalk(V == 4 ? cols >> 2 : cols);

    auto stage = [&](int t) {  // local stage t = global k-stage ks0 + t, ring slot t % S
        if (t < nloc) {
            const int s = t % S;
            T *As = sm + s * stage_elems;
            T *Bs = As + p.Tk * aip;
            const int64_t k0 = (int64_t)(ks0 + t) * p.Tk;
            const int kt = (int)imin64(p.Tk, p.K - k0);
            if constexpr (BULK) {
                // one bulk copy per B row; spread over lane 0 of every warp, so no warp falls a whole
                // k-tile of copy issue behind the others (the trailing barrier would wait for it).  A copy
                // may complete before thread 0's expect_tx: the transaction count goes transiently
                // negative, and the phase cannot complete before thread 0's arrival.
                const T *src = p.B + k0 * p.ldb + j0;
                if (tid == 0) mbar_arrive_expect_tx(bars + s, (unsigned)(kt * cols * 4));
                if (p.bulk_spread) {
                    if ((tid & 31) == 0)
                        for (int kk = tid >> 5; kk < kt; kk += (nthr + 31) >> 5)
                            bulk_g2s(Bs + kk * bjp, src + kk * p.ldb, cols * 4, bars + s);
                } else if (tid == 0) {
                    for (int kk = 0; kk < kt; kk++) bulk_g2s(Bs + kk * bjp, src + kk * p.ldb, cols * 4, bars + s);
                }
            }
            for (int r = wa.o0, kk = wa.i0; r < rows;) {
                if (kk < kt) cp_elem(As + kk * aip + r, p.A + (i0 + r) * p.lda + k0 + kk);
                r += wa.dO;
                kk += wa.dI;
                if (kk >= wa.inner) { kk -= wa.inner; r++; }
            }
            if (BT4) {  // row jj of B^T: k0 .. k0 + kt, 16-byte chunks (scalar tail chunk)
                for (int jj = wb.o0, c = wb.i0; jj < cols;) {
                    const T *src = p.B + (j0 + jj) * p.ldb + k0 + 4 * c;
                    T *dst = Bs + jj * p.bkp + 4 * c;
                    if (4 * c + 4 <= kt) cp_async16(dst, src);
                    else
                        for (int e = 0; e < 4; e++)
                            if (4 * c + e < kt) cp_elem(dst + e, src + e);
                    jj += wb.dO;
                    c += wb.dI;
                    if (c >= wb.inner) { c -= wb.inner; jj++; }
                }
            } else if constexpr (TRANSB) {
                for (int jj = wb.o0, kk = wb.i0; jj < cols;) {
                    if (kk < kt) cp_elem(Bs + kk * bjp + jj, p.B + (j0 + jj) * p.ldb + k0 + kk);
                    jj += wb.dO;
                    kk += wb.dI;
                    if (kk >= wb.inner) { kk -= wb.inner; jj++; }
                }
            } else if constexpr (!BULK) {
                for (int kk = wb.o0, c = wb.i0; kk < kt;) {
                    if constexpr (V == 4) cp_async16(Bs + kk * bjp + 4 * c, p.B + (k0 + kk) * p.ldb + j0 + 4 * c);
                    else cp_elem(Bs + kk * bjp + c, p.B + (k0 + kk) * p.ldb + j0 + c);
                    kk += wb.dO;
                    c += wb.dI;
                    if (c >= wb.inner) { c -= wb.inner; kk++; }
                }
            }
        }
        cp_async_commit();  // empty groups keep the wait_group count uniform
    };

    T acc[RM][RN];
#pragma unroll
    for (int r = 0; r < RM; r++)
#pragma unroll
        for (int c = 0; c < RN; c++) acc[r][c] = T(0);

    const int r0 = min(ty * RM, max(0, aip - RM));  // contiguous rows, clamped inside the pitch
    int cc[VN];
#pragma unroll
    for (int c = 0; c < VN; c++) cc[c] = min((tx + c * BX) * V, bjp - V);

    auto body = [&](const T *As, const T *Bs, int kk) {
        T a[RM], b[RN];
        if constexpr (sizeof(T) == 4 && RM % 4 == 0) {
#pragma unroll
            for (int r = 0; r < RM; r += 4) {
                const float4 v = *reinterpret_cast<const float4 *>(As + kk * aip + r0 + r);
                a[r] = v.x; a[r + 1] = v.y; a[r + 2] = v.z; a[r + 3] = v.w;
            }
        } else {
#pragma unroll
            for (int r = 0; r < RM; r++) a[r] = As[kk * aip + r0 + r];
        }
#pragma unroll
        for (int c = 0; c < VN; c++) {
            if constexpr (V == 4) {
                const float4 v = *reinterpret_cast<const float4 *>(Bs + kk * bjp + cc[c]);
                b[4 * c] = v.x; b[4 * c + 1] = v.y; b[4 * c + 2] = v.z; b[4 * c + 3] = v.w;
            } else {
                b[c] = Bs[kk * bjp + cc[c]];
            }
        }
#pragma unroll
        for (int r = 0; r < RM; r++)
#pragma unroll
            for (int c = 0; c < RN; c++) acc[r][c] = fma(a[r], b[c], acc[r][c]);
    };

    // transposed operand in [j][k] rows: four k per pass, one 16-byte read per owned column
    auto loada = [&](const T *As, int kk, T (&a)[RM]) {
        if constexpr (sizeof(T) == 4 && RM % 4 == 0) {
#pragma unroll
            for (int r = 0; r < RM; r += 4) {
                const float4 v = *reinterpret_cast<const float4 *>(As + kk * aip + r0 + r);
                a[r] = v.x; a[r + 1] = v.y; a[r + 2] = v.z; a[r + 3] = v.w;
            }
        } else {
#pragma unroll
            for (int r = 0; r < RM; r++) a[r] = As[kk * aip + r0 + r];
        }
    };
    auto body4t = [&](const T *As, const T *Bs, int kk) {
        if constexpr (TRANSB && sizeof(T) == 4 && V == 1) {
            float b[RN][4];
#pragma unroll
            for (int c = 0; c < RN; c++) {
                const float4 v = *reinterpret_cast<const float4 *>(Bs + cc[c] * p.bkp + kk);
                b[c][0] = v.x; b[c][1] = v.y; b[c][2] = v.z; b[c][3] = v.w;
            }
#pragma unroll
            for (int q = 0; q < 4; q++) {
                T a[RM];
                loada(As, kk + q, a);
#pragma unroll
                for (int r = 0; r < RM; r++)
#pragma unroll
                    for (int c = 0; c < RN; c++) acc[r][c] = fma(a[r], b[c][q], acc[r][c]);
            }
        }
    };
    auto body1t = [&](const T *As, const T *Bs, int kk) {
        if constexpr (TRANSB && V == 1) {
            T a[RM], b[RN];
            loada(As, kk, a);
#pragma unroll
            for (int c = 0; c < RN; c++) b[c] = Bs[cc[c] * p.bkp + kk];
#pragma unroll
            for (int r = 0; r < RM; r++)
#pragma unroll
                for (int c = 0; c < RN; c++) acc[r][c] = fma(a[r], b[c], acc[r][c]);
        }
    };

    for (int s = 0; s < S - 1; s++) stage(s);
    for (int t = 0; t < nloc; t++) {
        stage(t + S - 1);
        if (S == 1) cp_async_wait<0>();
        else if (S == 2) cp_async_wait<1>();
        else cp_async_wait<2>();
        if constexpr (BULK) mbar_wait(bars + (t % S), (unsigned)((t / S) & 1));
        __syncthreads();
        const T *As = sm + (t % S) * stage_elems;
        const T *Bs = As + p.Tk * aip;
        const int kt = (int)imin64(p.Tk, p.K - (int64_t)(ks0 + t) * p.Tk);
        int kk = 0;
        if (BT4) {
            for (; kk + 4 <= kt; kk += 4) body4t(As, Bs, kk);
            for (; kk < kt; kk++) body1t(As, Bs, kk);
        } else {
            for (; kk + 4 <= kt; kk += 4) {
#pragma unroll
                for (int q = 0; q < 4; q++) body(As, Bs, kk + q);
            }
            for (; kk < kt; kk++) body(As, Bs, kk);
        }
        __syncthreads();
    }
    cp_async_wait<0>();

    // epilogue: C = (init_zero ? 0 : beta*C) + alpha*acc; a k-part of a split tile adds alpha*acc to
    // C, which staged_tail_prepass has already set to (init_zero ? 0 : beta*C)
    if (split) {
#pragma unroll
        for (int r = 0; r < RM; r++) {
            const int rl = ty * RM + r;
            if (rl >= rows) continue;
            T *crow = p.C + (i0 + rl) * p.ldc + j0;
#pragma unroll
            for (int c = 0; c < VN; c++) {
#pragma unroll
                for (int e = 0; e < V; e++) {
                    const int cl = (tx + c * BX) * V + e;
                    if (cl < cols) atomicAdd(crow + cl, p.alpha * acc[r][c * V + e]);
                }
            }
        }
        return;
    }
#pragma unroll
    for (int r = 0; r < RM; r++) {
        const int rl = ty * RM + r;
        if (rl >= rows) continue;
        T *crow = p.C + (i0 + rl) * p.ldc + j0;
#pragma unroll
        for (int c = 0; c < VN; c++) {
            const int cl = (tx + c * BX) * V;
            if (cl >= cols) continue;
            if constexpr (V == 4) {
                float4 *cp = reinterpret_cast<float4 *>(crow + cl);
                float4 o = p.init_zero ? make_float4(0.f, 0.f, 0.f, 0.f) : *cp;
                if (!p.init_zero) { o.x *= p.beta; o.y *= p.beta; o.z *= p.beta; o.w *= p.beta; }
                o.x = fma(p.alpha, acc[r][4 * c + 0], o.x);
                o.y = fma(p.alpha, acc[r][4 * c + 1], o.y);
                o.z = fma(p.alpha, acc[r][4 * c + 2], o.z);
                o.w = fma(p.alpha, acc[r][4 * c + 3], o.w);
                *cp = o;
            } else {
                T o = p.init_zero ? T(0) : crow[cl] * p.beta;
                crow[cl] = fma(p.alpha, acc[r][c], o);
            }
        }
    }
}

// C := init_zero ? 0 : beta*C on the tiles t >= nfull (the split wave tail); one CTA per tile row.
template <typename T>
__global__ void staged_tail_prepass(const CArgs<T> p) {
    const int64_t t = p.nfull + (int64_t)blockIdx.x / p.Ti, r = (int64_t)blockIdx.x % p.Ti;
    const int64_t ti = t / p.gx, tj = t - ti * p.gx;
    const int64_t i = ti * p.Ti + r, j0 = tj * p.Tj;
    if (i >= p.M) return;
    T *c = p.C + i * p.ldc + j0;
    const int64_t w = p.N - j0 < p.Tj ? p.N - j0 : p.Tj;
    for (int64_t x = threadIdx.x; x < w; x += blockDim.x) c[x] = p.init_zero ? T(0) : p.beta * c[x];
}
