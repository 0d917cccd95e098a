// contract.cu -- SIMT tiled contraction executor for the gemm family (sm_100a).
//
// Executes Fig. 4's tiled nest for ANY tile vector (Ti, Tj, Tk):
//   ti -> blockIdx.y, tj -> blockIdx.x (PPCG mapping), tk sequential,
//   intra-tile points i, j -> threads, k intra-thread ("intra-thread reuse").
// Memory types follow the model's split (Eq. 1, Table II):
//   * SH_set operand (A(i,k), non-CMA) is staged tile by tile into shared memory
//     with cp.async double buffering (the Ti x Tk footprint V^{In});
//   * L1_set operands (B(k,j) and C(i,j), stride-1 in l_s1 = j) are read through
//     L1 with coalesced 16-byte vector loads along j; the carve-out between L1 and
//     shared memory is set from the split factor;
//   * syrk's second operand A(j,k) is not stride-1 in j (SH_set), so it
//     is staged transposed into shared memory.
// Tile != thread block (reading Q1): a CTA of bx*by threads covers the Ti x Tj
// output tile with a register micro-tile (rm x rn per thread, rows cyclic with
// stride by, column vectors cyclic with stride bx*vec).  When the whole tile fits
// in registers the accumulators stay resident across all k-tiles; otherwise the
// output tile is read-modify-written per k-tile through L1 ("Out: T-reuse(k)",
// Table II) -- exactly the liveness trade-off the model prices.
// Partial tiles are predicated (Fig. 4 min() guards, reading Q25).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include "contract.cuh"
#include "devsw.hpp"

namespace eatss {

template <typename T>
struct CArgs {
    int64_t M, N, K;
    const T *__restrict__ A;
    int64_t lda;
    const T *__restrict__ B;
    int64_t ldb;
    T *__restrict__ C;
    int64_t ldc;
    T alpha, beta;
    int init_zero;
    int Ti, Tj, Tk;
    int a_smem, b_smem, nbuf;
    int tkp, tjp;
    int bkp;  // staged transposed operand: B slice kept as [j][k] with this k-pitch (0 = [k][j] layout)
    int64_t gx;      // staged: j-tiles of the grid (tile index t = ti * gx + tj)
    int64_t nfull;   // staged: tiles run whole; tiles >= nfull are split along k into sp parts
    int sp;          // staged: 1 = 2-D grid, no split
    int passes_i, passes_j;
    int waf;          // lanes of each warp along j (0: linear layout, tx fastest)
    int bulk_spread;  // staged bulk path: the per-row B copies are issued by lane 0 of every warp (else thread 0)
    int32_t *counts;  // coverage mode
};

// Thread layout with WAF lanes of every warp along the CMA loop j (the SIMT length as a fraction of
// the warp size): lane l of warp w owns column slot (w % wx)*WAF + l % WAF and row slot
// (w / wx)*(32/WAF) + l / WAF, wx = BX / WAF.  The planner makes BX a multiple of WAF and BY a
// multiple of 32/WAF, so this is a permutation of the (tx, ty) slots.
__device__ __forceinline__ void warp_layout(int tid, int BX, int waf, int &tx, int &ty) {
    const int w = tid >> 5, l = tid & 31, wx = BX / waf;
    tx = (w % wx) * waf + (l % waf);
    ty = (w / wx) * (32 / waf) + l / waf;
}

enum { MODE_RESIDENT = 0, MODE_STREAM = 1, MODE_COVER = 2 };

__device__ __forceinline__ int64_t imin64(int64_t a, int64_t b) { return a < b ? a : b; }

__device__ __forceinline__ void cp_async4(void *smem, const void *gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void cp_async8(void *smem, const void *gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void cp_async16(void *smem, const void *gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N));
}

template <typename T>
__device__ __forceinline__ void cp_elem(T *s, const T *g) {
    if constexpr (sizeof(T) == 4) cp_async4(s, g);
    else cp_async8(s, g);
}

// Stage A(i0.., k0..k0+kt) -> As[row * tkp + kk]
template <typename T>
__device__ __forceinline__ void stage_a(const CArgs<T> &p, T *As, int64_t i0, int rows, int64_t k0,
                                        int kt, int tid, int nthr) {
    const bool v16 = (sizeof(T) == 4) && ((p.lda & 3) == 0) && ((k0 & 3) == 0) && ((kt & 3) == 0) &&
                     ((reinterpret_cast<uintptr_t>(p.A) & 15) == 0);
    if (v16) {
        const int cpr = kt >> 2;  // 16-byte chunks per row
        const int total = rows * cpr;
        for (int e = tid; e < total; e += nthr) {
            const int r = e / cpr, c = e - r * cpr;
            cp_async16(As + r * p.tkp + 4 * c, p.A + (i0 + r) * p.lda + k0 + 4 * c);
        }
    } else {
        const int total = rows * kt;
        for (int e = tid; e < total; e += nthr) {
            const int r = e / kt, c = e - r * kt;
            cp_elem(As + r * p.tkp + c, p.A + (i0 + r) * p.lda + k0 + c);
        }
    }
}

// Stage the transposed operand: Bs[kk * tjp + jj] = B[(j0 + jj) * ldb + k0 + kk]
template <typename T>
__device__ __forceinline__ void stage_bt(const CArgs<T> &p, T *Bs, int64_t j0, int cols, int64_t k0,
                                         int kt, int tid, int nthr) {
    const int total = cols * kt;
    for (int e = tid; e < total; e += nthr) {
        const int jj = e / kt, kk = e - jj * kt;  // lanes run along k: coalesced global reads
        cp_elem(Bs + kk * p.tjp + jj, p.B + (j0 + jj) * p.ldb + k0 + kk);
    }
}

template <typename T, int V>
struct VecT;
template <>
struct VecT<float, 4> {
    using type = float4;
};
template <>
struct VecT<float, 1> {
    using type = float;
};
template <>
struct VecT<double, 1> {
    using type = double;
};

template <typename T, int V>
__device__ __forceinline__ void load_vec(T (&dst)[V], const T *src) {
    if constexpr (V == 4) {
        float4 v = __ldg(reinterpret_cast<const float4 *>(src));
        dst[0] = v.x; dst[1] = v.y; dst[2] = v.z; dst[3] = v.w;
    } else {
        dst[0] = __ldg(src);
    }
}

template <typename T, int RM, int RN, int V, bool TRANSB, int MODE>
__global__ void __launch_bounds__((16384 / (RM * RN)) < 1024 ? (16384 / (RM * RN)) : 1024)
    contract_kernel(const CArgs<T> p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    constexpr int VN = RN / V;
    T *As = reinterpret_cast<T *>(smem_raw);
    T *Bs = As + (p.a_smem ? p.nbuf * p.Ti * p.tkp : 0);

    const int BX = blockDim.x, BY = blockDim.y;
    const int tid = threadIdx.y * BX + threadIdx.x, nthr = BX * BY;
    int tx = threadIdx.x, ty = threadIdx.y;
    if (p.waf) warp_layout(tid, BX, p.waf, tx, ty);
    const int64_t i0 = (int64_t)blockIdx.y * p.Ti, j0 = (int64_t)blockIdx.x * p.Tj;
    const int rows = (int)imin64(p.Ti, p.M - i0);
    const int cols = (int)imin64(p.Tj, p.N - j0);
    const int nk = (int)((p.K + p.Tk - 1) / p.Tk);

    T acc[RM][RN];

    auto stage = [&](int t, int buf) {
        const int64_t k0 = (int64_t)t * p.Tk;
        const int kt = (int)imin64(p.Tk, p.K - k0);
        if (p.a_smem) stage_a(p, As + buf * p.Ti * p.tkp, i0, rows, k0, kt, tid, nthr);
        if (TRANSB && p.b_smem) stage_bt(p, Bs + buf * p.Tk * p.tjp, j0, cols, k0, kt, tid, nthr);
        cp_async_commit();
    };

    // accumulate k in [k0, k0+kt) into acc for the pass (pi, pj)
    auto compute = [&](int64_t k0, int kt, int buf, int ri0, int cj0) {
        const T *Ab = As + buf * p.Ti * p.tkp;
        const T *Bb = Bs + buf * p.Tk * p.tjp;
        int rr[RM];
        bool rv[RM];
#pragma unroll
        for (int r = 0; r < RM; r++) {
            rr[r] = ri0 + ty + r * BY;
            rv[r] = rr[r] < rows;
            if (!rv[r]) rr[r] = 0;  // keep shared-memory reads inside the staged tile
        }
        int cc[VN];
        bool cv[VN];
#pragma unroll
        for (int c = 0; c < VN; c++) {
            cc[c] = cj0 + (tx + c * BX) * V;
            cv[c] = cc[c] < cols;
            if (!cv[c]) cc[c] = 0;
        }
        for (int kk = 0; kk < kt; kk++) {
            const int64_t k = k0 + kk;
            T a[RM];
            T b[RN];
            if constexpr (MODE != MODE_COVER) {
#pragma unroll
            for (int r = 0; r < RM; r++) {
                if (p.a_smem) a[r] = Ab[rr[r] * p.tkp + kk];
                else a[r] = rv[r] ? __ldg(p.A + (i0 + rr[r]) * p.lda + k) : T(0);
            }
#pragma unroll
            for (int c = 0; c < VN; c++) {
                T v[V];
                if constexpr (TRANSB) {
                    if (p.b_smem) v[0] = Bb[kk * p.tjp + cc[c]];
                    else v[0] = cv[c] ? __ldg(p.B + (j0 + cc[c]) * p.ldb + k) : T(0);
                } else {
                    if (cv[c]) load_vec<T, V>(v, p.B + k * p.ldb + j0 + cc[c]);
                    else {
#pragma unroll
                        for (int q = 0; q < V; q++) v[q] = T(0);
                    }
                }
#pragma unroll
                for (int q = 0; q < V; q++) b[c * V + q] = v[q];
            }
            }
            if constexpr (MODE == MODE_COVER) {
#pragma unroll
                for (int r = 0; r < RM; r++)
#pragma unroll
                    for (int c = 0; c < VN; c++)
#pragma unroll
                        for (int q = 0; q < V; q++)
                            if (rv[r] && cv[c] && cc[c] + q < cols)
                                atomicAdd(p.counts + ((i0 + rr[r]) * p.N + (j0 + cc[c] + q)) * p.K + k, 1);
            } else {
#pragma unroll
                for (int r = 0; r < RM; r++)
#pragma unroll
                    for (int c = 0; c < RN; c++) acc[r][c] = fma(a[r], b[c], acc[r][c]);
            }
        }
    };

    // C(i,j) = first ? (init_zero ? 0 : beta*C) + alpha*acc : C + alpha*acc
    auto epilogue = [&](bool first, int ri0, int cj0) {
        if constexpr (MODE == MODE_COVER) return;
#pragma unroll
        for (int r = 0; r < RM; r++) {
            const int rl = ri0 + ty + r * BY;
            if (rl >= rows) continue;
            T *crow = p.C + (i0 + rl) * p.ldc + j0;
#pragma unroll
            for (int c = 0; c < VN; c++) {
                const int cl = cj0 + (tx + c * BX) * V;
                if (cl >= cols) continue;
                if constexpr (V == 4) {
                    float4 *cp = reinterpret_cast<float4 *>(crow + cl);
                    float4 o;
                    if (first && p.init_zero) o = make_float4(0.f, 0.f, 0.f, 0.f);
                    else {
                        o = *cp;
                        if (first) { o.x *= p.beta; o.y *= p.beta; o.z *= p.beta; o.w *= p.beta; }
                    }
                    o.x = fma(p.alpha, acc[r][c * 4 + 0], o.x);
                    o.y = fma(p.alpha, acc[r][c * 4 + 1], o.y);
                    o.z = fma(p.alpha, acc[r][c * 4 + 2], o.z);
                    o.w = fma(p.alpha, acc[r][c * 4 + 3], o.w);
                    *cp = o;
                } else {
                    T o = (first && p.init_zero) ? T(0) : crow[cl];
                    if (first && !p.init_zero) o *= p.beta;
                    crow[cl] = fma(p.alpha, acc[r][c], o);
                }
            }
        }
    };

    auto zero_acc = [&]() {
#pragma unroll
        for (int r = 0; r < RM; r++)
#pragma unroll
            for (int c = 0; c < RN; c++) acc[r][c] = T(0);
    };

    const bool use_smem = p.a_smem || (TRANSB && p.b_smem);
    if (use_smem) stage(0, 0);
    if constexpr (MODE != MODE_STREAM) zero_acc();
    for (int t = 0; t < nk; t++) {
        const int64_t k0 = (int64_t)t * p.Tk;
        const int kt = (int)imin64(p.Tk, p.K - k0);
        const int buf = (p.nbuf == 2) ? (t & 1) : 0;
        if (use_smem) {
            if (p.nbuf == 2 && t + 1 < nk) {
                stage(t + 1, (t + 1) & 1);
                cp_async_wait<1>();
            } else {
                cp_async_wait<0>();
            }
            __syncthreads();
        }
        if constexpr (MODE == MODE_STREAM || MODE == MODE_COVER) {
            for (int pi = 0; pi < p.passes_i; pi++)
                for (int pj = 0; pj < p.passes_j; pj++) {
                    const int ri0 = pi * BY * RM, cj0 = pj * BX * RN;
                    zero_acc();
                    compute(k0, kt, buf, ri0, cj0);
                    epilogue(t == 0, ri0, cj0);
                }
        } else {
            compute(k0, kt, buf, 0, 0);
        }
        if (use_smem) {
            __syncthreads();
            if (p.nbuf == 1 && t + 1 < nk) stage(t + 1, 0);
        }
    }
    if constexpr (MODE == MODE_RESIDENT) epilogue(true, 0, 0);
}

#include "staged.cuh"

#if 0  // superseded by staged.cuh (kept out of the build)
// ------------------------------------------------------------------ staged resident kernel
// The register-resident fast path: per k-tile both operand slices -- the SH_set
// tile A(i0.., k0..k0+Tk) (stored transposed so a thread's rows are contiguous)
// and the L1_set slice B(k0..k0+Tk, j0..) -- are brought into shared memory with
// cp.async through an S-stage ring, so the load of k-tile t+S-1 overlaps the FMAs
// of k-tile t.  A thread owns rm contiguous rows x rn columns (16-byte vectors,
// cyclic over the warp) -- every shared-memory read is a broadcast (A) or a
// conflict-free 16-byte vector (B).
template <typename T, int RM, int RN, int V, bool TRANSB>
__global__ void __launch_bounds__((16384 / (RM * RN)) < 1024 ? (16384 / (RM * RN)) : 1024)
    contract_staged_kernel(const CArgs<T> p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    constexpr int VN = RN / V;
    T *const sm = reinterpret_cast<T *>(smem_raw);
    const int aip = p.tkp;  // A^T pitch (>= Ti, multiple of 4)
    const int bjp = p.tjp;  // B pitch (>= Tj, multiple of 4)
    const int stage_elems = p.Tk * (aip + bjp);
    const int S = p.nbuf;

    const int tx = threadIdx.x, ty = threadIdx.y, BX = blockDim.x;
    const int tid = ty * BX + tx, nthr = BX * blockDim.y;
    const int64_t i0 = (int64_t)blockIdx.y * p.Ti, j0 = (int64_t)blockIdx.x * p.Tj;
    const int rows = (int)imin64(p.Ti, p.M - i0);
    const int cols = (int)imin64(p.Tj, p.N - j0);
    const int nk = (int)((p.K + p.Tk - 1) / p.Tk);

    // Division-free staging walks: element e = tid + n*nthr of an (outer x inner) box is
    // tracked as (o, i) and advanced by (nthr / inner, nthr % inner) -- one division per CTA.
    struct Walk {
        int o0, i0, dO, dI, inner;
    };
    auto mkwalk = [&](int inner) {
        Walk w;
        w.inner = max(inner, 1);
        w.o0 = tid / w.inner; w.i0 = tid - w.o0 * w.inner;
        w.dO = nthr / w.inner; w.dI = nthr - w.dO * w.inner;
        return w;
    };
    const Walk wa = mkwalk(p.Tk);                                      // A: (row, k), k fastest
    const Walk wb = TRANSB ? mkwalk(p.Tk) : mkwalk(V == 4 ? cols >> 2 : cols);  // B: (k, col) / (col, k)

    auto stage = [&](int t) {
        if (t < nk) {
            T *As = sm + (t % S) * stage_elems;
            T *Bs = As + p.Tk * aip;
            const int64_t k0 = (int64_t)t * p.Tk;
            const int kt = (int)imin64(p.Tk, p.K - k0);
            for (int r = wa.o0, kk = wa.i0; r < rows;) {  // lanes along k: coalesced reads
                if (kk < kt) cp_elem(As + kk * aip + r, p.A + (i0 + r) * p.lda + k0 + kk);
                r += wa.dO; kk += wa.dI;
                if (kk >= wa.inner) { kk -= wa.inner; r++; }
            }
            if constexpr (TRANSB) {
                for (int jj = wb.o0, kk = wb.i0; jj < cols;) {
                    if (kk < kt) cp_elem(Bs + kk * bjp + jj, p.B + (j0 + jj) * p.ldb + k0 + kk);
                    jj += wb.dO; kk += wb.dI;
                    if (kk >= wb.inner) { kk -= wb.inner; jj++; }
                }
            } else {
                for (int kk = wb.o0, c = wb.i0; kk < kt;) {
                    if constexpr (V == 4) cp_async16(Bs + kk * bjp + 4 * c, p.B + (k0 + kk) * p.ldb + j0 + 4 * c);
                    else cp_elem(Bs + kk * bjp + c, p.B + (k0 + kk) * p.ldb + j0 + c);
                    kk += wb.dO; c += wb.dI;
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

    const int r0 = min(ty * RM, max(0, p.tkp - RM));  // contiguous rows (clamped inside the pitch)
    int cc[VN];
#pragma unroll
    for (int c = 0; c < VN; c++) cc[c] = min((tx + c * BX) * V, bjp - V);

    for (int s = 0; s < S - 1; s++) stage(s);
    for (int t = 0; t < nk; t++) {
        stage(t + S - 1);
        if (S == 1) cp_async_wait<0>();
        else if (S == 2) cp_async_wait<1>();
        else cp_async_wait<2>();
        __syncthreads();
        const T *As = sm + (t % S) * stage_elems;
        const T *Bs = As + p.Tk * aip;
        const int kt = (int)imin64(p.Tk, p.K - (int64_t)t * p.Tk);
#pragma unroll 2
        for (int kk = 0; kk < kt; kk++) {
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
        }
        __syncthreads();
    }
    cp_async_wait<0>();

    // epilogue: C = (init_zero ? 0 : beta*C) + alpha*acc
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

#endif

// ------------------------------------------------------------------ planning

namespace {
struct MT {
    int rm, rn;
};
const MT kV4[] = {{1, 4}, {2, 4}, {4, 4}, {4, 8}, {8, 8}};
const MT kV1[] = {{1, 1}, {1, 2}, {2, 2}, {2, 4}, {4, 4}, {4, 8}, {8, 8}};
inline int maxthreads(int rm, int rn) { return std::min(1024, 16384 / (rm * rn)); }
inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
}  // namespace

ContractPlan plan_contraction(const ContractNest &n, const int64_t *tiles, int smem_limit, int waf_req) {
    ContractPlan p;
    p.rTi = tiles[0]; p.rTj = tiles[1]; p.rTk = tiles[2];
    p.Ti = std::max<int64_t>(1, std::min(tiles[0], n.M));
    p.Tj = std::max<int64_t>(1, std::min(tiles[1], n.N));
    p.Tk = std::max<int64_t>(1, std::min(tiles[2], n.K));
    const int esz = n.f64 ? 8 : 4;
    const uintptr_t ab = reinterpret_cast<uintptr_t>(n.B), ac = reinterpret_cast<uintptr_t>(n.C);
    const bool v4 = !n.f64 && !n.transB && (n.N % 4 == 0) && (n.ldb % 4 == 0) && (n.ldc % 4 == 0) &&
                    (p.Tj % 4 == 0) && (ab % 16 == 0) && (ac % 16 == 0);
    p.vec = v4 ? 4 : 1;
    const MT *cand = v4 ? kV4 : kV1;
    const int ncand = v4 ? 5 : 7;
    const int64_t rows = p.Ti, cols = p.Tj;
    const int64_t outputs = rows * cols;
    int target_threads = 256;
    if (devsw("EATSS_THREADS", 0) > 0) target_threads = std::max(32, devsw("EATSS_THREADS", 0));
    const int64_t want = cdiv(outputs, target_threads);
    const int waf = (waf_req == 4 || waf_req == 8 || waf_req == 16 || waf_req == 32) ? waf_req : 0;
    const int yq = waf ? 32 / waf : 1;  // rows of one warp
    p.waf = waf;
    auto rup = [](int64_t v, int64_t m) { return ((v + m - 1) / m) * m; };
    // smallest micro-tile reaching `want` outputs/thread that does not exceed the tile; with a warp
    // alignment the thread grid is rounded to whole warps of WAF x 32/WAF (idle slots predicated) and
    // the first candidate that keeps >= 3/4 of the slots busy is taken (else the busiest one)
    int pick = -1, best = -1;
    double best_u = -1.0;
    for (int c = 0; c < ncand; c++) {
        if (cand[c].rm > std::max<int64_t>(rows, 1) && c > 0) continue;
        if (cand[c].rn > ((cols + p.vec - 1) / p.vec) * p.vec && c > 0) continue;
        if (!waf) {
            pick = c;
            if (cand[c].rm * cand[c].rn >= want) break;
            continue;
        }
        const int64_t by0 = cdiv(rows, cand[c].rm), bx0 = cdiv(cols, cand[c].rn);
        const int64_t byr = rup(by0, yq), bxr = rup(bx0, waf);
        if (bxr * byr > maxthreads(cand[c].rm, cand[c].rn)) continue;
        const double u = (double)(by0 * bx0) / (double)(byr * bxr);
        if (u > best_u) { best_u = u; best = c; }
        if (cand[c].rm * cand[c].rn >= want && u >= 0.75) { pick = c; break; }
    }
    if (waf && pick < 0) pick = best;
    if (pick < 0) pick = 0;
    p.rm = cand[pick].rm;
    p.rn = cand[pick].rn;
    int64_t by = cdiv(rows, p.rm), bx = cdiv(cols, p.rn);
    if (waf) {
        by = rup(by, yq);
        bx = rup(bx, waf);
    }
    const int mt = maxthreads(p.rm, p.rn);
    if (by * bx <= mt) {
        p.stream = false;
        p.bx = (int)bx;
        p.by = (int)by;
    } else {
        // output tile exceeds the register budget: largest micro-tile, RMW passes through L1
        p.rm = 8;
        p.rn = 8;
        const int lim = maxthreads(8, 8);
        p.bx = (int)std::min<int64_t>(cdiv(cols, p.rn), lim / yq);
        if (waf) p.bx = std::max(waf, p.bx / waf * waf);
        p.by = (int)std::max<int64_t>(1, std::min<int64_t>(cdiv(rows, p.rm), lim / p.bx));
        if (waf) p.by = std::max(yq, p.by / yq * yq);
        p.stream = true;
        p.passes_i = (int)cdiv(rows, (int64_t)p.by * p.rm);
        p.passes_j = (int)cdiv(cols, (int64_t)p.bx * p.rn);
    }
    // shared memory: SH_set tiles, double buffered when two fit
    p.tkp = (int)(((p.Tk + 3) / 4) * 4 + (esz == 4 ? 4 : 2));
    p.tjp = (int)((p.Tj % 2 == 0) ? p.Tj + 1 : p.Tj + 2);
    const int64_t a_bytes = p.Ti * p.tkp * esz;
    const int64_t b_bytes = n.transB ? p.Tk * p.tjp * esz : 0;
    auto fits = [&](int nb, bool a, bool b) {
        return nb * ((a ? a_bytes : 0) + (b ? b_bytes : 0)) <= smem_limit;
    };
    p.a_smem = true;
    p.b_smem = n.transB;
    p.nbuf = 2;
    if (!fits(2, p.a_smem, p.b_smem)) p.nbuf = 1;
    if (!fits(p.nbuf, p.a_smem, p.b_smem) && p.b_smem) {
        p.b_smem = false;  // transposed operand too large: read through L1
        p.nbuf = fits(2, true, false) ? 2 : 1;
    }
    if (!fits(p.nbuf, p.a_smem, p.b_smem)) {
        p.a_smem = false;  // SH tile too large for shared memory: read through L1 (PPCG does the same)
        p.nbuf = (p.b_smem && fits(2, false, true)) ? 2 : 1;
    }
    p.smem_bytes = (int)(p.nbuf * ((p.a_smem ? a_bytes : 0) + (p.b_smem ? b_bytes : 0)));
    if (!p.stream) {
        // register-resident: stage both operand slices per k-tile through an S-stage cp.async ring
        // The ring holds S stages of kst k-rows each; a k-tile of Tk rows is staged as
        // ceil(Tk/kst) sub-stages (numerically identical: accumulators are resident and k
        // stays ascending).  Default (measured, profiles/): one stage per whole k-tile
        // (S = 1) so two CTAs share an SM and overlap each other's copies; kst is halved only
        // when a k-tile does not fit.  EATSS_STAGES / EATSS_KSUB override for experiments.
        const int64_t aip = ((p.Ti + 3) / 4) * 4, bjp = ((p.Tj + 3) / 4) * 4;
        // transposed operand (syrk: B(k, j) = A(j, k)), fp32: stage it untransposed as [j][k] rows
        // with 16-byte copies (k-pitch kst + 4: conflict-free 16-byte reads along k)
        const uintptr_t bb = reinterpret_cast<uintptr_t>(n.B);
        const bool bt4 = n.transB && !n.f64 && n.ldb % 4 == 0 && bb % 16 == 0 &&
                         devsw("EATSS_TRANSB_LEGACY", 0) == 0;
        auto stage_of = [&](int64_t ks) {
            const int64_t b = bt4 ? bjp * (ks + 4) : ks * bjp;
            return (ks * aip + b) * esz;
        };
        int64_t kst = bt4 ? ((p.Tk + 3) / 4) * 4 : p.Tk, S = 1;
        const int64_t kmin = bt4 ? 4 : 1;
        while (kst > kmin && S * (stage_of(kst) + 16) > smem_limit)
            kst = bt4 ? std::max<int64_t>(4, ((kst / 2 + 3) / 4) * 4) : (kst + 1) / 2;
        if (devsw("EATSS_STAGES", 0) > 0) S = devsw("EATSS_STAGES", 0);
        if (const int ksub = devsw("EATSS_KSUB", 0)) kst = std::max<int64_t>(1, (p.Tk + ksub - 1) / std::max(1, ksub));
        if (bt4) kst = ((kst + 3) / 4) * 4;
        const int64_t stage_bytes = stage_of(kst);
        if (S * (stage_bytes + 16) > smem_limit) S = std::max<int64_t>(1, smem_limit / (stage_bytes + 16));
        if (S * (stage_bytes + 16) <= smem_limit && devsw("EATSS_NO_STAGED", 0) == 0) {
            p.staged = true;
            p.nbuf = (int)S;
            p.kst = (int)kst;
            p.tkp = (int)aip;
            p.tjp = (int)bjp;
            p.bkp = bt4 ? (int)(kst + 4) : 0;
            p.a_smem = true;
            p.b_smem = true;
            p.smem_bytes = (int)(S * stage_bytes + 16 * S);  // + one mbarrier per stage
        }
    }
    p.grid_x = cdiv(n.N, p.Tj);
    p.grid_y = cdiv(n.M, p.Ti);
    return p;
}

int plan_simt_x(const ContractPlan &p) {
    if (p.waf) return p.waf;
    // linear layout (tx fastest): a warp spans min(32, bx) consecutive column slots when bx divides 32
    // or is a multiple of it; otherwise its lanes wrap over rows and the run along j is bx % 32
    if (p.bx >= 32) return p.bx % 32 == 0 ? 32 : p.bx % 32;
    return p.bx;
}

namespace {
thread_local int g_last_cv = -1;
}
void note_carveout(int pct) { g_last_cv = pct; }
int take_carveout() {
    const int v = g_last_cv;
    g_last_cv = -1;
    return v;
}

// ------------------------------------------------------------------ dispatch

template <typename T, int RM, int RN, int V, bool TB, int MODE>
static cudaError_t launch_one(const CArgs<T> &a, const ContractPlan &p, int carveout,
                              cudaStream_t s) {
    auto k = contract_kernel<T, RM, RN, V, TB, MODE>;
    cudaError_t e;
    if (p.smem_bytes > 48 * 1024) {
        e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
        if (e != cudaSuccess) return e;
    }
    const int cv = cv_resolve(carveout, 0);
    e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, cv);
    if (e != cudaSuccess) return e;
    note_carveout(cv);
    dim3 grid((unsigned)p.grid_x, (unsigned)p.grid_y, 1), block(p.bx, p.by, 1);
    k<<<grid, block, p.smem_bytes, s>>>(a);
    return cudaGetLastError();
}

// contraction_launches(): set while counting the kernels a launch would issue (no launch happens)
static thread_local int *g_dry_launches = nullptr;

template <typename T, int RM, int RN, int V, bool TB>
static cudaError_t launch_staged(const CArgs<T> &a, const ContractPlan &p, int carveout, cudaStream_t s) {
    auto k = contract_staged_kernel<T, RM, RN, V, TB>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
    if (e != cudaSuccess) return e;
    // The staged path keeps its operand slices in shared memory: the split's carve-out is
    // honoured unless it would cut the co-resident CTAs below what registers allow
    // (the sigma -> carve-out mapping); exec.carveout_exact keeps sigma as is.
    int need = 0;
    cudaFuncAttributes fa;
    if (cudaFuncGetAttributes(&fa, k) == cudaSuccess && fa.numRegs > 0) {
        const int threads = ((p.bx * p.by + 31) / 32) * 32;
        const int nb_regs = 65536 / (((fa.numRegs + 7) / 8) * 8 * threads);
        const int per_cta = p.smem_bytes + 1024;  // + per-CTA reservation
        const int nb = std::max(1, std::min(nb_regs, 233472 / per_cta));
        need = (int)std::min<int64_t>(100, (100LL * nb * per_cta + 233471) / 233472);
    }
    const int cv = cv_resolve(carveout, need);
    e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, cv);
    if (e != cudaSuccess) return e;
    if (!g_dry_launches) note_carveout(cv);
    dim3 block(p.bx, p.by, 1);
    // wave-quantisation tail: when the last wave would leave at least half of the resident-CTA
    // slots idle, its tiles are split along k (EATSS_SIMT_SPLITK=0 disables)
    CArgs<T> b = a;
    b.sp = 1;
    b.gx = p.grid_x;
    const int64_t T_ = p.grid_x * p.grid_y;
    static const bool splitk = devsw("EATSS_SIMT_SPLITK", 1) != 0;
    int nb = 0, dev = 0, nsm = 148;
    if (splitk && cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k, p.bx * p.by, p.smem_bytes) == cudaSuccess &&
        nb > 0) {
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        const int64_t slots = (int64_t)nb * nsm, rem = T_ % slots;
        const int64_t nk = (a.K + a.Tk - 1) / a.Tk;
        if (T_ > slots && rem > 0 && 2 * rem <= slots) {
            b.sp = (int)std::min<int64_t>(std::min<int64_t>(4, slots / rem), nk);
            b.nfull = T_ - rem;
        }
    }
    cudaGetLastError();
    if (g_dry_launches) {
        *g_dry_launches += b.sp > 1 ? 2 : 1;
        return cudaSuccess;
    }
    if (b.sp > 1) {
        const int64_t ntail = T_ - b.nfull;
        staged_tail_prepass<T><<<(unsigned)(ntail * b.Ti), 256, 0, s>>>(b);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        k<<<(unsigned)(b.nfull + ntail * b.sp), block, p.smem_bytes, s>>>(b);
    } else {
        dim3 grid((unsigned)p.grid_x, (unsigned)p.grid_y, 1);
        k<<<grid, block, p.smem_bytes, s>>>(b);
    }
    return cudaGetLastError();
}

template <typename T, int V, bool TB>
static cudaError_t by_mt_staged(const CArgs<T> &a, const ContractPlan &p, int cv, cudaStream_t s) {
    const int key = p.rm * 100 + p.rn;
    if constexpr (V == 4) {
        switch (key) {
            case 104: return launch_staged<T, 1, 4, 4, TB>(a, p, cv, s);
            case 204: return launch_staged<T, 2, 4, 4, TB>(a, p, cv, s);
            case 404: return launch_staged<T, 4, 4, 4, TB>(a, p, cv, s);
            case 408: return launch_staged<T, 4, 8, 4, TB>(a, p, cv, s);
            case 808: return launch_staged<T, 8, 8, 4, TB>(a, p, cv, s);
        }
    } else {
        switch (key) {
            case 101: return launch_staged<T, 1, 1, 1, TB>(a, p, cv, s);
            case 102: return launch_staged<T, 1, 2, 1, TB>(a, p, cv, s);
            case 202: return launch_staged<T, 2, 2, 1, TB>(a, p, cv, s);
            case 204: return launch_staged<T, 2, 4, 1, TB>(a, p, cv, s);
            case 404: return launch_staged<T, 4, 4, 1, TB>(a, p, cv, s);
            case 408: return launch_staged<T, 4, 8, 1, TB>(a, p, cv, s);
            case 808: return launch_staged<T, 8, 8, 1, TB>(a, p, cv, s);
        }
    }
    return cudaErrorInvalidConfiguration;
}

template <typename T, int V, bool TB, int MODE>
static cudaError_t by_mt(const CArgs<T> &a, const ContractPlan &p, int cv, cudaStream_t s) {
    const int key = p.rm * 100 + p.rn;
    if constexpr (V == 4) {
        switch (key) {
            case 104: return launch_one<T, 1, 4, 4, TB, MODE>(a, p, cv, s);
            case 204: return launch_one<T, 2, 4, 4, TB, MODE>(a, p, cv, s);
            case 404: return launch_one<T, 4, 4, 4, TB, MODE>(a, p, cv, s);
            case 408: return launch_one<T, 4, 8, 4, TB, MODE>(a, p, cv, s);
            case 808: return launch_one<T, 8, 8, 4, TB, MODE>(a, p, cv, s);
        }
    } else {
        switch (key) {
            case 101: return launch_one<T, 1, 1, 1, TB, MODE>(a, p, cv, s);
            case 102: return launch_one<T, 1, 2, 1, TB, MODE>(a, p, cv, s);
            case 202: return launch_one<T, 2, 2, 1, TB, MODE>(a, p, cv, s);
            case 204: return launch_one<T, 2, 4, 1, TB, MODE>(a, p, cv, s);
            case 404: return launch_one<T, 4, 4, 1, TB, MODE>(a, p, cv, s);
            case 408: return launch_one<T, 4, 8, 1, TB, MODE>(a, p, cv, s);
            case 808: return launch_one<T, 8, 8, 1, TB, MODE>(a, p, cv, s);
        }
    }
    return cudaErrorInvalidConfiguration;
}

template <typename T, int MODE>
static cudaError_t by_variant(const CArgs<T> &a, const ContractPlan &p, bool transB, int cv,
                              cudaStream_t s) {
    if constexpr (sizeof(T) == 4) {
        if (p.vec == 4) return by_mt<T, 4, false, MODE>(a, p, cv, s);
    }
    if (transB) return by_mt<T, 1, true, MODE>(a, p, cv, s);
    return by_mt<T, 1, false, MODE>(a, p, cv, s);
}

template <typename T>
static cudaError_t launch_typed(const ContractNest &n, const ContractPlan &p, int carveout,
                               int32_t *counts, cudaStream_t s) {
    CArgs<T> a;
    a.M = n.M; a.N = n.N; a.K = n.K;
    a.A = static_cast<const T *>(n.A); a.lda = n.lda;
    a.B = static_cast<const T *>(n.B); a.ldb = n.ldb;
    a.C = static_cast<T *>(n.C); a.ldc = n.ldc;
    a.alpha = (T)n.alpha; a.beta = (T)n.beta;
    a.init_zero = n.init_zero ? 1 : 0;
    a.Ti = (int)p.Ti; a.Tj = (int)p.Tj;
    a.Tk = p.staged ? p.kst : (int)p.Tk;  // the staged kernel walks k in ring stages of kst rows
    a.a_smem = p.a_smem; a.b_smem = p.b_smem; a.nbuf = p.nbuf;
    a.tkp = p.tkp; a.tjp = p.tjp; a.bkp = p.bkp;
    a.gx = p.grid_x; a.nfull = 0; a.sp = 1;
    a.passes_i = p.passes_i; a.passes_j = p.passes_j;
    a.waf = p.waf;
    static const int spread = devsw("EATSS_SIMT_BULK_SPREAD", 1);  // development A/B
    a.bulk_spread = spread;
    a.counts = counts;
    if (counts) return by_variant<T, MODE_COVER>(a, p, n.transB, carveout, s);
    if (p.staged) {
        if constexpr (sizeof(T) == 4) {
            if (p.vec == 4) return by_mt_staged<T, 4, false>(a, p, carveout, s);
        }
        if (n.transB) return by_mt_staged<T, 1, true>(a, p, carveout, s);
        return by_mt_staged<T, 1, false>(a, p, carveout, s);
    }
    if (p.stream) return by_variant<T, MODE_STREAM>(a, p, n.transB, carveout, s);
    return by_variant<T, MODE_RESIDENT>(a, p, n.transB, carveout, s);
}

cudaError_t launch_contraction(const ContractNest &n, const ContractPlan &p, int carveout_pct,
                               int32_t *coverage_counts, cudaStream_t s) {
    if (n.M <= 0 || n.N <= 0) return cudaSuccess;
    if (p.grid_y > 65535) return cudaErrorInvalidConfiguration;
    if (n.f64) return launch_typed<double>(n, p, carveout_pct, coverage_counts, s);
    return launch_typed<float>(n, p, carveout_pct, coverage_counts, s);
}

// dst[c][r] = src[r][c] (rows x cols fp32, row pitch lds; dst pitch rows): 32 x 32 shared tiles,
// coalesced both ways.  The SIMT executor's layout pass for a transposed operand (syrk's A^T).
__global__ void transpose_kernel(const float *__restrict__ src, int64_t rows, int64_t cols, int64_t lds,
                                 float *__restrict__ dst) {
    __shared__ float t[32][33];
    const int64_t c0 = (int64_t)blockIdx.x * 32, r0 = (int64_t)blockIdx.y * 32;
    for (int y = threadIdx.y; y < 32; y += blockDim.y) {
        const int64_t r = r0 + y, c = c0 + threadIdx.x;
        if (r < rows && c < cols) t[y][threadIdx.x] = src[r * lds + c];
    }
    __syncthreads();
    for (int y = threadIdx.y; y < 32; y += blockDim.y) {
        const int64_t c = c0 + y, r = r0 + threadIdx.x;
        if (r < rows && c < cols) dst[c * rows + r] = t[threadIdx.x][y];
    }
}

cudaError_t launch_transpose(const float *src, int64_t rows, int64_t cols, int64_t lds, float *dst, cudaStream_t s) {
    if (rows <= 0 || cols <= 0) return cudaSuccess;
    if ((rows + 31) / 32 > 65535) return cudaErrorInvalidConfiguration;
    dim3 grid((unsigned)((cols + 31) / 32), (unsigned)((rows + 31) / 32)), block(32, 8);
    transpose_kernel<<<grid, block, 0, s>>>(src, rows, cols, lds, dst);
    return cudaGetLastError();
}

int contraction_launches(const ContractNest &n, const ContractPlan &p) {
    if (!p.staged || n.M <= 0 || n.N <= 0) return 1;
    int c = 0;
    g_dry_launches = &c;
    launch_contraction(n, p, 50, nullptr, nullptr);
    g_dry_launches = nullptr;
    return c > 0 ? c : 1;
}

}  // namespace eatss
