// lowdim.cu -- tiled executor of the paper's low-dimensional PolyBench kernels (SURVEY §8(f) row 4:
// mvt, atax, bicg, gemver; Fig. 7; mvt in Fig. 9).
//
// Every nest of these kernels is a matrix-vector product over a row-major matrix A[nx][ny], in
// one of two forms (reading R-N7):
//   row form   rowout[i] (+)= ar * sum_j A[i][j] * vr[j]   (i parallel, j reduction: stride-1 j)
//   col form   colout[j] (+)= ac * sum_i A[i][j] * vc[i]   (j parallel, i reduction)
// One tile (Ti, Tj) is one CTA (tj -> blockIdx.x, ti -> blockIdx.y), clipped with min()
// (reading Q25).  A CTA streams its Ti x Tj block of A once, with 16-byte loads along j (the CMA
// loop), and evaluates BOTH forms from that single read when both are requested: PolyBench's bicg
// loop computes s = A^T r and q = A p in one sweep, and mvt's two nests read the same matrix, so
// on B200 each becomes one pass over A instead of two (A is the only O(n^2) traffic: the kernels
// are HBM-bound, AI ~ 0.5 flop/B).  gemver's rank-2 update is fused into the pass that consumes
// the updated matrix (the A^T y product), which writes A' back once.
// Reductions: a row's partial over the CTA's j range is reduced across the warp with
// __shfl_xor_sync and added to rowout with one atomic per row and CTA; a column's partial over
// the CTA's rows is reduced across warps in shared memory and added with one atomic per column
// and CTA.  The summation order therefore differs from the literal loop (fp32 tolerance; exact on
// small-integer inputs); callers zero or pre-scale the outputs first.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

namespace eatss {

struct LowdimArgs {
    const float *A;  // [nx][ny] (read; written back as A' when upd)
    float *Aout;     // A' destination (upd), may alias A
    int64_t nx, ny;
    int Ti, Tj;
    // row form
    float *rowout;
    const float *vr;
    float ar;
    // col form
    float *colout;
    const float *vc;
    float ac;
    // fused rank-2 update A' = A + u1 v1^T + u2 v2^T (gemver nest 1)
    const float *u1, *v1, *u2, *v2;
};

constexpr int LD_THREADS = 256;
constexpr int LD_MAXG = 4;  // column groups per lane held in registers (sub-tiles of <= 512 columns)

template <bool ROW, bool COL, bool UPD, int V, int LPRC>  // LPRC: compile-time lanes per row (0 = runtime)
__global__ void __launch_bounds__(LD_THREADS) lowdim_kernel(const LowdimArgs p, int lpr_rt) {
    const int LPR = LPRC > 0 ? LPRC : lpr_rt;
    // Lane layout: LPR lanes share a row (16-byte groups along j), RPW = 32 / LPR rows per warp, so
    // narrow tiles (few columns) still keep every lane streaming.
    __shared__ float colred[LD_THREADS / 32][32 * V * LD_MAXG];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int lr = lane % LPR, rg = lane / LPR, RPW = 32 / LPR;
    // one CTA per tile (ti = blockIdx.y, tj = blockIdx.x); beyond 65535 row tiles a CTA executes
    // ti = blockIdx.y, + gridDim.y, ... one after the other (each tile whole)
    const int64_t j0 = (int64_t)blockIdx.x * p.Tj, j1 = min(j0 + (int64_t)p.Tj, p.ny);
    const int64_t ntile_i = (p.nx + p.Ti - 1) / p.Ti;
    if (j0 >= j1 || (int64_t)blockIdx.y >= ntile_i) return;
    const int ng = (int)((j1 - j0 + LPR * V - 1) / (LPR * V));  // column groups per lane (<= LD_MAXG)
    float vrr[LD_MAXG][V], v1r[LD_MAXG][V], v2r[LD_MAXG][V], cacc[LD_MAXG][V];
#pragma unroll
    for (int g = 0; g < LD_MAXG; g++)
#pragma unroll
        for (int e = 0; e < V; e++) {
            const int64_t j = j0 + (int64_t)(g * LPR + lr) * V + e;
            const bool ok = g < ng && j < j1;
            vrr[g][e] = (ROW && ok) ? __ldg(p.vr + j) : 0.f;
            v1r[g][e] = (UPD && ok) ? __ldg(p.v1 + j) : 0.f;
            v2r[g][e] = (UPD && ok) ? __ldg(p.v2 + j) : 0.f;
            cacc[g][e] = 0.f;
        }
    // rows in batches of RB per lane group: all loads of a batch are issued before any product
    constexpr int RB = 2;
    for (int64_t ti = blockIdx.y; ti < ntile_i; ti += gridDim.y) {
        const int64_t i0 = ti * p.Ti, i1 = min(i0 + (int64_t)p.Ti, p.nx);
        const int64_t step = (int64_t)nw * RPW;
        for (int64_t ib = i0 + (int64_t)warp * RPW + rg; ib - rg < i1; ib += step * RB) {
            float a[RB][LD_MAXG][V];
#pragma unroll
            for (int r = 0; r < RB; r++) {
                const int64_t i = ib + r * step;
                const bool rok = i < i1;
                const float *arow = p.A + i * p.ny;
#pragma unroll
                for (int g = 0; g < LD_MAXG; g++) {
                    const int64_t j = j0 + (int64_t)(g * LPR + lr) * V;
                    const bool gok = rok && g < ng;
                    if constexpr (V == 4) {
                        if (gok && j + 3 < j1) {
                            const float4 x = __ldcs(reinterpret_cast<const float4 *>(arow + j));
                            a[r][g][0] = x.x; a[r][g][1] = x.y; a[r][g][2] = x.z; a[r][g][3] = x.w;
                        } else {
#pragma unroll
                            for (int e = 0; e < 4; e++) a[r][g][e] = (gok && j + e < j1) ? arow[j + e] : 0.f;
                        }
                    } else {
                        a[r][g][0] = (gok && j < j1) ? __ldcs(arow + j) : 0.f;
                    }
                }
            }
#pragma unroll
            for (int r = 0; r < RB; r++) {
                const int64_t i = ib + r * step;
                const bool rok = i < i1;
                const float vci = (COL && rok) ? __ldg(p.vc + i) : 0.f;
                float racc = 0.f;
                if constexpr (UPD) {
                    const float u1i = rok ? __ldg(p.u1 + i) : 0.f, u2i = rok ? __ldg(p.u2 + i) : 0.f;
                    float *orow = p.Aout + i * p.ny;
#pragma unroll
                    for (int g = 0; g < LD_MAXG; g++) {
                        if (g >= ng) break;
                        const int64_t j = j0 + (int64_t)(g * LPR + lr) * V;
#pragma unroll
                        for (int e = 0; e < V; e++) a[r][g][e] = (a[r][g][e] + u1i * v1r[g][e]) + u2i * v2r[g][e];
                        if (!rok) continue;
                        if constexpr (V == 4) {
                            if (j + 3 < j1) {
                                __stcs(reinterpret_cast<float4 *>(orow + j),
                                       make_float4(a[r][g][0], a[r][g][1], a[r][g][2], a[r][g][3]));
                            } else {
#pragma unroll
                                for (int e = 0; e < 4; e++)
                                    if (j + e < j1) orow[j + e] = a[r][g][e];
                            }
                        } else if (j < j1) {
                            orow[j] = a[r][g][0];
                        }
                    }
                }
#pragma unroll
                for (int g = 0; g < LD_MAXG; g++)
#pragma unroll
                    for (int e = 0; e < V; e++) {
                        if constexpr (ROW) racc = fmaf(a[r][g][e], vrr[g][e], racc);
                        if constexpr (COL) cacc[g][e] = fmaf(a[r][g][e], vci, cacc[g][e]);
                    }
                if constexpr (ROW) {  // reduce across the LPR lanes of the row
                    for (int o = LPR >> 1; o > 0; o >>= 1) racc += __shfl_xor_sync(0xffffffffu, racc, o);
                    if (lr == 0 && rok) atomicAdd(p.rowout + i, p.ar * racc);
                }
            }
        }
    }
    if constexpr (COL) {  // reduce the column partials: across the warp's row groups, then the warps
#pragma unroll
        for (int g = 0; g < LD_MAXG; g++)
#pragma unroll
            for (int e = 0; e < V; e++) {
                float v = cacc[g][e];
                for (int o = LPR; o < 32; o <<= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
                if (rg == 0) colred[warp][(g * LPR + lr) * V + e] = v;
            }
        __syncthreads();
        const int ncols = (int)(j1 - j0);
        for (int c = threadIdx.x; c < ncols; c += blockDim.x) {
            float s = 0.f;
            for (int w = 0; w < nw; w++) s += colred[w][c];
            atomicAdd(p.colout + j0 + c, p.ac * s);
        }
    }
}

// out[i] = out[i] * scale + (add ? add[i] : 0)   (output initialisation, gemver's x = x + z)
__global__ void lowdim_axpy(float *out, const float *add, float scale, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = out[i] * scale + (add ? add[i] : 0.f);
}

// ------------------------------------------------------------------ host
bool lowdim_tile_ok(int64_t Ti, int64_t Tj) { return Ti >= 1 && Tj >= 1; }

// Column tiles wider than LD_MAXG * 32 * V columns are split into sub-tiles of that width
// (the tile's row/column partial sums are then added by more atomics; the mapping of rows to
// CTAs -- the ti loop -- is unchanged).
cudaError_t launch_lowdim(const LowdimArgs &a0, bool row, bool col, bool upd, cudaStream_t s, int64_t *launched) {
    LowdimArgs a = a0;
    const bool v4 = a.ny % 4 == 0 && a.Tj % 4 == 0 && (reinterpret_cast<uintptr_t>(a.A) & 15) == 0 &&
                    (!upd || (reinterpret_cast<uintptr_t>(a.Aout) & 15) == 0);
    const int V = v4 ? 4 : 1;
    // lanes per row: enough 16-byte groups to cover the tile's width, at most a warp
    int LPR = 1;
    while (LPR < 32 && (int64_t)LPR * V < std::min<int64_t>(a.Tj, a.ny)) LPR *= 2;
    a.Tj = (int)std::min<int64_t>(a.Tj, (int64_t)LD_MAXG * LPR * V);
    a.Ti = (int)std::min<int64_t>(a.Ti, a.nx);
    const int64_t gx = (a.ny + a.Tj - 1) / a.Tj, ntile_i = (a.nx + a.Ti - 1) / a.Ti;
    int64_t gy = std::min<int64_t>(ntile_i, 65535);  // > 65535 row tiles: CTAs walk several
    // column form: each CTA adds one atomic per column, so with narrow row tiles (the EATSS picks)
    // the atomics, not the matrix stream, dominate; CTAs then walk several row tiles each, the grid
    // sized to ~8 resident CTAs per SM (one atomic per column and CTA). EATSS_LOWDIM_WALK=0: one tile
    // per CTA.
    static const bool walk = [] {
        const char *e = getenv("EATSS_LOWDIM_WALK");
        return !(e && atoi(e) == 0);
    }();
    if (col && walk) {
        static int nsm = 0;
        if (!nsm) {
            int dev = 0;
            cudaGetDevice(&dev);
            if (cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || nsm <= 0) nsm = 148;
        }
        const int64_t target = 8LL * nsm;
        gy = std::max<int64_t>(1, std::min<int64_t>(gy, (target + gx - 1) / gx));
    }
    if (gx > INT32_MAX) return cudaErrorInvalidConfiguration;
    dim3 grid((unsigned)gx, (unsigned)gy), block(LD_THREADS);
#define LDK(R, C, U)                                                                   \
    do {                                                                               \
        if (v4 && LPR == 32) lowdim_kernel<R, C, U, 4, 32><<<grid, block, 0, s>>>(a, LPR); \
        else if (v4) lowdim_kernel<R, C, U, 4, 0><<<grid, block, 0, s>>>(a, LPR);      \
        else if (LPR == 32) lowdim_kernel<R, C, U, 1, 32><<<grid, block, 0, s>>>(a, LPR); \
        else lowdim_kernel<R, C, U, 1, 0><<<grid, block, 0, s>>>(a, LPR);              \
    } while (0)
    if (upd) LDK(false, true, true);
    else if (row && col) LDK(true, true, false);
    else if (row) LDK(true, false, false);
    else LDK(false, true, false);
#undef LDK
    if (launched) (*launched)++;
    return cudaGetLastError();
}

cudaError_t launch_lowdim_axpy(float *out, const float *add, float scale, int64_t n, cudaStream_t s,
                               int64_t *launched) {
    const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, 148 * 8));
    lowdim_axpy<<<(unsigned)blocks, 256, 0, s>>>(out, add, scale, n);
    if (launched) (*launched)++;
    return cudaGetLastError();
}

}  // namespace eatss
