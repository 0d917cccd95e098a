// lowdim.cu -- tiled executor of the paper's low-dimensional PolyBench kernels (SURVEY §8(f) row 4:
// mvt, atax, bicg, gemver; Fig. 7; mvt in Fig. 9).
//
// Every nest of these kernels is a matrix-vector product over a row-major matrix A[nx][ny], in
// one of two forms (reading R-N7):
//   row form   rowout[i] (+)= ar * sum_j A[i][j] * vr[j]   (i parallel, j reduction: stride-1 j)
//   col form   colout[j] (+)= ac * sum_i A[i][j] * vc[i]   (j parallel, i reduction)
// One tile (Ti, Tj) is executed whole by one CTA (tj -> blockIdx.x; a CTA walks the row
// tiles ti = blockIdx.y, + gridDim.y, ... in turn), clipped with min() (reading Q25).  A CTA streams its Ti x Tj block of A once, with 16-byte loads along j (the CMA
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

template <bool ROW, bool COL, bool UPD, int V>
__global__ void __launch_bounds__(LD_THREADS) lowdim_kernel(const LowdimArgs p) {
    __shared__ float colred[LD_THREADS / 32][32 * V * LD_MAXG];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    // a CTA executes the tiles (ti, tj = blockIdx.x) for ti = blockIdx.y, + gridDim.y, ... one after
    // the other (each tile whole, by this CTA), carrying its column partial sums across them, so a
    // column costs one atomic per CTA instead of one per row tile
    const int64_t j0 = (int64_t)blockIdx.x * p.Tj, j1 = min(j0 + (int64_t)p.Tj, p.ny);
    const int64_t ntile_i = (p.nx + p.Ti - 1) / p.Ti;
    if (j0 >= j1 || (int64_t)blockIdx.y >= ntile_i) return;
    const int ng = (int)((j1 - j0 + 32 * V - 1) / (32 * V));  // column groups per lane (<= LD_MAXG)
    float vrr[LD_MAXG][V], v1r[LD_MAXG][V], v2r[LD_MAXG][V], cacc[LD_MAXG][V];
#pragma unroll
    for (int g = 0; g < LD_MAXG; g++)
#pragma unroll
        for (int e = 0; e < V; e++) {
            const int64_t j = j0 + (int64_t)(g * 32 + lane) * V + e;
            const bool ok = g < ng && j < j1;
            vrr[g][e] = (ROW && ok) ? __ldg(p.vr + j) : 0.f;
            v1r[g][e] = (UPD && ok) ? __ldg(p.v1 + j) : 0.f;
            v2r[g][e] = (UPD && ok) ? __ldg(p.v2 + j) : 0.f;
            cacc[g][e] = 0.f;
        }
    for (int64_t ti = blockIdx.y; ti < ntile_i; ti += gridDim.y) {
    const int64_t i0 = ti * p.Ti, i1 = min(i0 + (int64_t)p.Ti, p.nx);
    for (int64_t i = i0 + warp; i < i1; i += nw) {
        const float *arow = p.A + i * p.ny;
        const float vci = COL ? __ldg(p.vc + i) : 0.f;
        const float u1i = UPD ? __ldg(p.u1 + i) : 0.f, u2i = UPD ? __ldg(p.u2 + i) : 0.f;
        float racc = 0.f;
#pragma unroll
        for (int g = 0; g < LD_MAXG; g++) {
            if (g >= ng) break;
            const int64_t j = j0 + (int64_t)(g * 32 + lane) * V;
            float a[V];
            if constexpr (V == 4) {
                if (j + 3 < j1) {
                    const float4 x = __ldcs(reinterpret_cast<const float4 *>(arow + j));
                    a[0] = x.x; a[1] = x.y; a[2] = x.z; a[3] = x.w;
                } else {
#pragma unroll
                    for (int e = 0; e < 4; e++) a[e] = j + e < j1 ? arow[j + e] : 0.f;
                }
            } else {
                a[0] = j < j1 ? __ldcs(arow + j) : 0.f;
            }
            if constexpr (UPD) {
#pragma unroll
                for (int e = 0; e < V; e++) a[e] = (a[e] + u1i * v1r[g][e]) + u2i * v2r[g][e];
                float *orow = p.Aout + i * p.ny;
                if constexpr (V == 4) {
                    if (j + 3 < j1) {
                        __stcs(reinterpret_cast<float4 *>(orow + j), make_float4(a[0], a[1], a[2], a[3]));
                    } else {
#pragma unroll
                        for (int e = 0; e < 4; e++)
                            if (j + e < j1) orow[j + e] = a[e];
                    }
                } else if (j < j1) {
                    orow[j] = a[0];
                }
            }
#pragma unroll
            for (int e = 0; e < V; e++) {
                if constexpr (ROW) racc = fmaf(a[e], vrr[g][e], racc);
                if constexpr (COL) cacc[g][e] = fmaf(a[e], vci, cacc[g][e]);
            }
        }
        if constexpr (ROW) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) racc += __shfl_xor_sync(0xffffffffu, racc, o);
            if (lane == 0) atomicAdd(p.rowout + i, p.ar * racc);
        }
    }
    }
    if constexpr (COL) {  // reduce the column partials of the CTA's warps, one atomic per column
#pragma unroll
        for (int g = 0; g < LD_MAXG; g++)
#pragma unroll
            for (int e = 0; e < V; e++) colred[warp][(g * 32 + lane) * V + e] = cacc[g][e];
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
    a.Tj = (int)std::min<int64_t>(a.Tj, (int64_t)LD_MAXG * 32 * V);
    a.Ti = (int)std::min<int64_t>(a.Ti, a.nx);
    const int64_t gx = (a.ny + a.Tj - 1) / a.Tj, ntile_i = (a.nx + a.Ti - 1) / a.Ti;
    // enough CTAs to keep every SM streaming (8 per SM), each walking several row tiles
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    const int64_t gy = std::min<int64_t>(std::min<int64_t>(ntile_i, 65535),
                                         std::max<int64_t>(1, ((int64_t)nsm * 8 + gx - 1) / gx));
    if (gx > INT32_MAX) return cudaErrorInvalidConfiguration;
    dim3 grid((unsigned)gx, (unsigned)gy), block(LD_THREADS);
#define LDK(R, C, U)                                                                   \
    do {                                                                               \
        if (v4) lowdim_kernel<R, C, U, 4><<<grid, block, 0, s>>>(a);                   \
        else lowdim_kernel<R, C, U, 1><<<grid, block, 0, s>>>(a);                      \
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
