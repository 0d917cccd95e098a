// stencil_staged.cu -- shared-memory-staged stencil sweeps (jacobi-2d, heat-3d), the fast path of
// stencil.cu for fp32 tiles whose halo window fits in shared memory.
//
// Same tiling semantics as stencil.cu (only the space dimensions are tiled, one CTA per
// tile, tiles aligned to multiples of T and clipped to the interior 1..n-2, reading Q25), same
// per-point arithmetic (bit-identical to the column-walk kernels), different data movement:
// the tile's halo window is brought into shared memory by the bulk-copy / TMA engine in ONE
// asynchronous transaction per CTA (jacobi-2d: one cp.async.bulk per window row; heat-3d: one
// 3-D cp.async.bulk.tensor box), completion on an mbarrier.  No thread spends issue slots or
// registers on outstanding loads, so every resident CTA keeps its whole window (74 KB for the
// EATSS jacobi tile (16,1024), 52 KB for the heat tile (16,16,32)) in flight at once -- the
// bytes-in-flight a B200 SM needs to run at HBM speed (Little's law) -- and the column walks
// then read neighbours from shared memory instead of re-fetching them through L1.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include "contract.cuh"
#include "devsw.hpp"

#include "tc_ptx.cuh"

namespace eatss {

using tcm::mbar_expect_tx;
using tcm::mbar_init;
using tcm::mbar_wait;
using tcm::su32;

namespace {

// Programmatic dependent launch (sweep t+1 of a time loop is launched while sweep t drains): the
// dependent grid is scheduled early, then waits here until the previous grid has completed and its
// writes are visible -- before any global access, since sweep t+1 writes the array sweep t reads.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;\n" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory"); }

__device__ __forceinline__ void bulk_row_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(su32(dst)),
        "l"(src), "r"(bytes), "r"(su32(bar))
        : "memory");
}

// L2 residency hints for the jacobi-2d ping-pong at L2-sized grids (N = 4000: 2 x 64 MB against 126 MB of
// L2): the source window is read evict-first (a line, once read, is the preferred victim) and the
// destination is written evict-last, so the array the next sweep reads stays in L2 while the one just read
// makes room.
using tcm::policy_evict_last;
__device__ __forceinline__ void bulk_row_g2s_hint(void *dst, const void *src, unsigned bytes, uint64_t *bar,
                                                  uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;\n" ::"r"(
            su32(dst)),
        "l"(src), "r"(bytes), "r"(su32(bar)), "l"(pol)
        : "memory");
}
__device__ __forceinline__ void st_hint_v4(float *p, float4 v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;\n" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
                 "f"(v.w), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void st_hint(float *p, float v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;\n" ::"l"(p), "f"(v), "l"(pol) : "memory");
}

// Work items (a, b) of an A x B space, a = the 16-byte column group along the CMA loop l_s1.  waf = 0:
// linear order (a fastest); waf in {4, 8, 16, 32}: the warp-fraction layout -- lane l of
// virtual warp w takes a = (w % wa)*waf + l % waf and b = (w / wa)*(32/waf) + l / waf (wa = ceil(A/waf)),
// i.e. WAF lanes of every warp contiguous along l_s1 and the other 32/WAF lanes on the next rows.
// Visits every item exactly once; returns false when v is past the space.
__device__ __forceinline__ bool waf_item(int v, int A, int B, int waf, int &a, int &b) {
    if (waf <= 0) {
        a = v % A;
        b = v / A;
        return b < B;
    }
    const int w = v >> 5, l = v & 31, wa = (A + waf - 1) / waf;
    a = (w % wa) * waf + l % waf;
    b = (w / wa) * (32 / waf) + l / waf;
    return b < B;
}

// ------------------------------------------------------------------ jacobi-2d
// Window: rows [ilo-1, ihi+1), columns [cs, ce) = [tj0-4, tj0+Tj+4) clipped to [0, n); n, Tj, tj0
// multiples of 4, so every window row is a 16-byte-aligned run of (ce-cs)*4 bytes.
// Boundary cells of the window come from bsrc when bsrc != src (stencil.cu: the ping-pong sweep
// that reads B takes its boundary from A).
template <bool COVER>
__global__ void __launch_bounds__(256) jacobi2d_staged(float *__restrict__ dst, const float *__restrict__ src,
                                                       const float *__restrict__ bsrc, int64_t n, int Ti, int Tj,
                                                       int32_t *counts, int waf, int l2hint) {
    extern __shared__ __align__(16) float win[];
    __shared__ uint64_t bar;
    const int64_t ti0 = (int64_t)blockIdx.y * Ti, tj0 = (int64_t)blockIdx.x * Tj;
    const int64_t ilo = ti0 > 1 ? ti0 : 1, ihi = ti0 + Ti < n - 1 ? ti0 + Ti : n - 1;
    const int64_t jlo = tj0 > 1 ? tj0 : 1, jhi = tj0 + Tj < n - 1 ? tj0 + Tj : n - 1;
    if (ilo >= ihi || jlo >= jhi) return;
    const int64_t r0 = ilo - 1;
    const int nr = (int)(ihi - ilo + 2);
    const int64_t cs = tj0 - 4 > 0 ? tj0 - 4 : 0, ce = tj0 + Tj + 4 < n ? tj0 + Tj + 4 : n;
    const int W = (int)(ce - cs);
    const int64_t g0 = jlo >> 2, g1 = ((jhi - 1) >> 2) + 1;  // 16-byte column groups holding outputs
    if constexpr (COVER) {
        for (int64_t i = ilo; i < ihi; i++)
            for (int64_t g = g0 + threadIdx.x; g < g1; g += blockDim.x)
                for (int q = 0; q < 4; q++) {
                    const int64_t j = 4 * g + q;
                    if (j >= jlo && j < jhi) atomicAdd(counts + i * n + j, 1);
                }
        return;
    }
    const int tid = threadIdx.x;
    if (tid == 0) {
        mbar_init(&bar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    pdl_wait();
    __syncthreads();
    if (tid < 32) {
        if (tid == 0) mbar_expect_tx(&bar, (unsigned)(nr * W * 4));
        __syncwarp();
        if (l2hint) {
            const uint64_t pf = tcm::policy_evict_first();
            for (int r = tid; r < nr; r += 32)
                bulk_row_g2s_hint(win + r * W, src + (r0 + r) * n + cs, (unsigned)W * 4, &bar, pf);
        } else {
            for (int r = tid; r < nr; r += 32) bulk_row_g2s(win + r * W, src + (r0 + r) * n + cs, (unsigned)W * 4, &bar);
        }
    }
    mbar_wait(&bar, 0);
    if (bsrc != src) {  // boundary cells of the window: from bsrc
        const bool top = r0 == 0, bot = r0 + nr == n, left = cs == 0, right = ce == n;
        if (top || bot || left || right) {
            for (int c = tid; c < W; c += blockDim.x) {
                if (top) win[c] = bsrc[cs + c];
                if (bot) win[(nr - 1) * W + c] = bsrc[(n - 1) * n + cs + c];
            }
            for (int r = tid; r < nr; r += blockDim.x) {
                if (left) win[r * W] = bsrc[(r0 + r) * n];
                if (right) win[r * W + W - 1] = bsrc[(r0 + r) * n + n - 1];
            }
            __syncthreads();
        }
    }
    const float c02 = 0.2f;
    const uint64_t pl = l2hint ? policy_evict_last() : 0;
    const int rows = (int)(ihi - ilo);
    // items: (column group, row chunk); with a warp alignment the rows are cut into 32/WAF chunks
    const int ngr = (int)(g1 - g0), nch = waf > 0 ? 32 / waf : 1, per = (rows + nch - 1) / nch;
    const int span = waf > 0 ? ((ngr + waf - 1) / waf) * waf * nch : ngr;  // virtual items
    for (int v = tid; v < span; v += blockDim.x) {
        int ga, ch;
        if (!waf_item(v, ngr, nch, waf, ga, ch) || ga >= ngr) continue;
        const int rb = ch * per, re = min(rows, rb + per);
        if (rb >= re) continue;
        const int64_t g = g0 + ga;
        const int cl = (int)(4 * g - cs);  // window column of the group's first element
        const bool full = 4 * g >= jlo && 4 * g + 3 < jhi;
        const float *colp = win + cl;
        float4 u = *reinterpret_cast<const float4 *>(colp + rb * W);
        float4 c = *reinterpret_cast<const float4 *>(colp + (rb + 1) * W);
        const int lm = cl > 0 ? -1 : 0, rp = cl + 4 < W ? 4 : 3;  // clamped (unused when clamped)
        for (int r = rb + 1; r <= re; r++) {
            const float *row = colp + r * W;
            const float4 d = *reinterpret_cast<const float4 *>(row + W);
            const float l = row[lm], rr = row[rp];
            float4 o;
            o.x = c02 * ((((c.x + l) + c.y) + d.x) + u.x);
            o.y = c02 * ((((c.y + c.x) + c.z) + d.y) + u.y);
            o.z = c02 * ((((c.z + c.y) + c.w) + d.z) + u.z);
            o.w = c02 * ((((c.w + c.z) + rr) + d.w) + u.w);
            float *out = dst + (r0 + r) * n + 4 * g;
            if (full) {
                if (l2hint) st_hint_v4(out, o, pl);
                else *reinterpret_cast<float4 *>(out) = o;
            } else {
                const float ov[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
                for (int q = 0; q < 4; q++)
                    if (4 * g + q >= jlo && 4 * g + q < jhi) {
                        if (l2hint) st_hint(out + q, ov[q], pl);
                        else out[q] = ov[q];
                    }
            }
            u = c;
            c = d;
        }
    }
}

// ------------------------------------------------------------------ heat-3d
// Window: box {Tk+8, Tj+2, Ti+2} at (tk0-4, tj0-1, ti0-1) of the 3-D tensor map over src
// (out-of-range cells zero-filled by TMA; they are never used by an interior output).
// A thread owns (j, 16-byte k-group) columns and walks i with planes i-1, i in registers.
// One tile of a heat-3d sweep: tile (bx = k-tile, by = (i-tile, j-tile)); `win` is the CTA's
// 128-byte-aligned window, `bar` its mbarrier in phase `phase`.  Returns false (no window traffic,
// barrier untouched) when the tile is empty.  Ends with __syncthreads(): the window may be reused.
__device__ __forceinline__ bool heat_tile(float *__restrict__ dst, const CUtensorMap *msrc, int64_t n, int Ti,
                                          int Tj, int Tk, int nbj, int64_t bx, int64_t by, float *win,
                                          uint64_t *bar, unsigned phase, int waf) {
    const int64_t tk0 = bx * Tk;
    const int64_t ti0 = (by / nbj) * Ti, tj0 = (by % nbj) * Tj;
    const int64_t ilo = ti0 > 1 ? ti0 : 1, ihi = ti0 + Ti < n - 1 ? ti0 + Ti : n - 1;
    const int64_t jlo = tj0 > 1 ? tj0 : 1, jhi = tj0 + Tj < n - 1 ? tj0 + Tj : n - 1;
    const int64_t klo = tk0 > 1 ? tk0 : 1, khi = tk0 + Tk < n - 1 ? tk0 + Tk : n - 1;
    if (ilo >= ihi || jlo >= jhi || klo >= khi) return false;
    const int KW = Tk + 8, JW = Tj + 2;  // window pitches (elements)
    const int64_t g0 = klo >> 2, g1 = ((khi - 1) >> 2) + 1;
    const int ng = (int)(g1 - g0), nj = (int)(jhi - jlo), ni = (int)(ihi - ilo);
    const int tid = threadIdx.x;
    if (tid == 0) {
        mbar_expect_tx(bar, (unsigned)((Ti + 2) * JW * KW * 4));
        tcm::tma_3d(win, msrc, (int)(tk0 - 4), (int)(tj0 - 1), (int)(ti0 - 1), bar);
    }
    mbar_wait(bar, phase);
    const float c = 0.125f, two = 2.0f;
    const int64_t nn = n * n;
    // work items: (i-chunk, j, k-group); i is split when the columns alone do not fill the CTA
    const int cols = nj * ng;
    const int chunks = max(1, min(ni, (int)blockDim.x / cols));
    const int per = (ni + chunks - 1) / chunks;
    // items (k-group, (j, i-chunk)); with a warp alignment WAF lanes of each warp run along k
    const int nb = nj * chunks, span = waf > 0 ? ((ng + waf - 1) / waf) * waf * (((nb + 32 / waf - 1) / (32 / waf)) * (32 / waf))
                                              : cols * chunks;
    for (int e = tid; e < span; e += blockDim.x) {
        int gi, b;
        if (!waf_item(e, ng, nb, waf, gi, b) || gi >= ng) continue;
        const int jj = b % nj, ch = b / nj;
        const int ib = ch * per, ie = min(ni, ib + per);
        if (ib >= ie) continue;
        const int64_t k = 4 * (g0 + gi), j = jlo + jj;
        const int wk = (int)(k - (tk0 - 4)), wj = (int)(j - (tj0 - 1));
        const int plane = JW * KW;
        // window plane index of global row i is i - (ti0 - 1)
        const float *colp = win + wj * KW + wk;
        const bool full = k >= klo && k + 3 < khi;
        const int wi0 = (int)(ilo + ib - (ti0 - 1));
        float4 u = *reinterpret_cast<const float4 *>(colp + (wi0 - 1) * plane);
        float4 x = *reinterpret_cast<const float4 *>(colp + wi0 * plane);
        for (int wi = wi0; wi < wi0 + (ie - ib); wi++) {
            const float *p = colp + wi * plane;
            const float4 ip = *reinterpret_cast<const float4 *>(p + plane);
            const float4 jp = *reinterpret_cast<const float4 *>(p + KW);
            const float4 jm = *reinterpret_cast<const float4 *>(p - KW);
            const float km1 = p[-1], kp4 = p[4];
            float4 o;
#define HEAT_PT3(X, IP, IM, JP, JM, KP, KM) \
    (c * (IP - two * X + IM) + c * (JP - two * X + JM) + c * (KP - two * X + KM) + X)
            o.x = HEAT_PT3(x.x, ip.x, u.x, jp.x, jm.x, x.y, km1);
            o.y = HEAT_PT3(x.y, ip.y, u.y, jp.y, jm.y, x.z, x.x);
            o.z = HEAT_PT3(x.z, ip.z, u.z, jp.z, jm.z, x.w, x.y);
            o.w = HEAT_PT3(x.w, ip.w, u.w, jp.w, jm.w, kp4, x.z);
#undef HEAT_PT3
            const int64_t i = ti0 - 1 + wi;
            float *out = dst + i * nn + j * n + k;
            if (full) {
                *reinterpret_cast<float4 *>(out) = o;
            } else {
                const float ov[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
                for (int q = 0; q < 4; q++)
                    if (k + q >= klo && k + q < khi) out[q] = ov[q];
            }
            u = x;
            x = ip;
        }
    }
    __syncthreads();
    return true;
}

template <bool COVER>
__global__ void __launch_bounds__(256) heat3d_staged(float *__restrict__ dst, const __grid_constant__ CUtensorMap msrc,
                                                     int64_t n, int Ti, int Tj, int Tk, int nbj, int32_t *counts,
                                                     int waf) {
    extern __shared__ __align__(128) unsigned char win_raw[];
    // TMA destinations must be 128-byte aligned: align the dynamic window by hand
    float *win = reinterpret_cast<float *>(win_raw + ((128u - (su32(win_raw) & 127u)) & 127u));
    __shared__ uint64_t bar;
    if constexpr (COVER) {
        const int64_t tk0 = (int64_t)blockIdx.x * Tk;
        const int64_t ti0 = (int64_t)(blockIdx.y / nbj) * Ti, tj0 = (int64_t)(blockIdx.y % nbj) * Tj;
        const int64_t ilo = ti0 > 1 ? ti0 : 1, ihi = ti0 + Ti < n - 1 ? ti0 + Ti : n - 1;
        const int64_t jlo = tj0 > 1 ? tj0 : 1, jhi = tj0 + Tj < n - 1 ? tj0 + Tj : n - 1;
        const int64_t klo = tk0 > 1 ? tk0 : 1, khi = tk0 + Tk < n - 1 ? tk0 + Tk : n - 1;
        if (ilo >= ihi || jlo >= jhi || klo >= khi) return;
        const int64_t g0 = klo >> 2, g1 = ((khi - 1) >> 2) + 1;
        const int ng = (int)(g1 - g0), nj = (int)(jhi - jlo), ni = (int)(ihi - ilo);
        for (int e = threadIdx.x; e < nj * ng * ni; e += blockDim.x) {
            const int gi = e % ng, jj = (e / ng) % nj, ii = e / (ng * nj);
            for (int q = 0; q < 4; q++) {
                const int64_t k = 4 * (g0 + gi) + q;
                if (k >= klo && k < khi) atomicAdd(counts + ((ilo + ii) * n + jlo + jj) * n + k, 1);
            }
        }
        return;
    }
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&msrc)) : "memory");
    }
    pdl_wait();
    __syncthreads();
    heat_tile(dst, &msrc, n, Ti, Tj, Tk, nbj, blockIdx.x, blockIdx.y, win, &bar, 0, waf);
    pdl_trigger();  // after this CTA's stores: the next sweep's launch overlaps this grid's tail
}

constexpr int kSmemTarget = 113 * 1024;  // at least two resident CTAs per SM

// launch with programmatic stream serialization allowed (the kernel calls pdl_trigger / pdl_wait);
// EATSS_STENCIL_PDL=0 launches normally (for comparison)
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, int smem, int carveout, cudaStream_t s,
                       Args... args) {
    static const bool on = [] {
        const char *e = getenv("EATSS_STENCIL_PDL");
        return !(e && atoi(e) == 0);
    }();
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = (size_t)smem;
    cfg.stream = s;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = on ? 1 : 0;
    // the carve-out travels with the launch (and with a captured graph node), so a replayed time
    // loop keeps the carve-out it was captured with
    at[1].id = cudaLaunchAttributePreferredSharedMemoryCarveout;
    at[1].val.sharedMemCarveout = (unsigned)carveout;
    cfg.attrs = at;
    cfg.numAttrs = 2;
    note_carveout(carveout);
    return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

int jacobi_staged_smem(int64_t n, int64_t Ti, int64_t Tj) {
    const int64_t nr = std::min<int64_t>(Ti, n) + 2, W = std::min<int64_t>(Tj + 8, n);
    return (int)(nr * W * 4);
}
int heat_staged_smem(int64_t Ti, int64_t Tj, int64_t Tk) { return (int)((Ti + 2) * (Tj + 2) * (Tk + 8) * 4) + 128; }

// carve-out (percent of the maximum shared memory) that keeps `ctas` CTAs of `smem` bytes resident,
// never below the model's split (sigma) preference -- or sigma itself under exec.carveout_exact
int staged_carveout(int smem, int cv) {
    int dev = 0, maxsm = 228 * 1024;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    const int ctas = std::max(1, std::min(4, (maxsm - 1024) / (smem + 1024 + 16)));
    const int need = (int)(((int64_t)ctas * (smem + 1024 + 16) * 100 + maxsm - 1) / maxsm);
    return cv_resolve(cv, std::min(100, need));
}

}  // namespace

bool jacobi2d_staged_applicable(int64_t n, int64_t Ti, int64_t Tj, bool f64) {
    return !f64 && n % 4 == 0 && Tj % 4 == 0 && n >= 8 && jacobi_staged_smem(n, Ti, Tj) <= kSmemTarget;
}
bool heat3d_staged_applicable(int64_t n, int64_t Ti, int64_t Tj, int64_t Tk, bool f64) {
    return !f64 && n % 4 == 0 && Tk % 4 == 0 && Tk + 8 <= 256 && Tj + 2 <= 256 && Ti + 2 <= 256 && n >= 8 &&
           n <= INT32_MAX / 2 && heat_staged_smem(Ti, Tj, Tk) <= kSmemTarget && tcm::encode_fn() != nullptr;
}

cudaError_t launch_jacobi2d_staged(float *dst, const float *src, const float *bsrc, int64_t n, int64_t Ti, int64_t Tj,
                                   int split_pct, int32_t *counts, cudaStream_t s, int waf) {
    const int64_t gx = (n - 1 + Tj - 1) / Tj, gy = (n - 1 + Ti - 1) / Ti;
    if (gy > 65535 || gx > INT32_MAX) return cudaErrorInvalidConfiguration;
    const int smem = counts ? 0 : jacobi_staged_smem(n, Ti, Tj);
    dim3 grid((unsigned)gx, (unsigned)gy), block(256);
    if (counts) {
        jacobi2d_staged<true><<<grid, block, 0, s>>>(dst, src, bsrc, n, (int)Ti, (int)Tj, counts, waf, 0);
        return cudaGetLastError();
    }
    // L2 hints when the two arrays are about L2-sized (between half and twice the L2): smaller grids stay
    // resident anyway, larger ones stream from HBM whatever the hints
    int dev = 0, l2 = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    static const int hint_env = devsw("EATSS_JACOBI_L2HINT", 1);  // development A/B
    const double both = 2.0 * (double)n * (double)n * 4.0;
    const int l2hint = (hint_env && l2 > 0 && both >= 0.5 * l2 && both <= 2.0 * l2) ? 1 : 0;
    cudaFuncSetAttribute(jacobi2d_staged<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    return launch_pdl(jacobi2d_staged<false>, grid, block, smem, staged_carveout(smem, split_pct), s, dst, src, bsrc,
                      n, (int)Ti, (int)Tj, (int32_t *)nullptr, waf, l2hint);
}

cudaError_t launch_heat3d_staged(float *dst, const float *src, int64_t n, int64_t Ti, int64_t Tj, int64_t Tk,
                                 int split_pct, int32_t *counts, cudaStream_t s, int waf) {
    const int64_t nbi = (n - 1 + Ti - 1) / Ti, nbj = (n - 1 + Tj - 1) / Tj, gx = (n - 1 + Tk - 1) / Tk;
    if (nbi * nbj > 65535) return cudaErrorInvalidConfiguration;
    dim3 grid((unsigned)gx, (unsigned)(nbi * nbj)), block(256);
    CUtensorMap m{};
    if (counts) {
        heat3d_staged<true><<<grid, block, 0, s>>>(dst, m, n, (int)Ti, (int)Tj, (int)Tk, (int)nbj, counts, waf);
        return cudaGetLastError();
    }
    const cuuint64_t dims[3] = {(cuuint64_t)n, (cuuint64_t)n, (cuuint64_t)n};
    const cuuint64_t strides[2] = {(cuuint64_t)n * 4, (cuuint64_t)n * n * 4};
    const cuuint32_t box[3] = {(cuuint32_t)(Tk + 8), (cuuint32_t)(Tj + 2), (cuuint32_t)(Ti + 2)};
    const cuuint32_t es[3] = {1, 1, 1};
    if (tcm::encode_fn()(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<float *>(src), dims, strides, box, es,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return cudaErrorInvalidValue;
    const int smem = heat_staged_smem(Ti, Tj, Tk);
    cudaFuncSetAttribute(heat3d_staged<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    return launch_pdl(heat3d_staged<false>, grid, block, smem, staged_carveout(smem, split_pct), s, dst,
                      (const CUtensorMap)m, n, (int)Ti, (int)Tj, (int)Tk, (int)nbj, (int32_t *)nullptr, waf);
}

}  // namespace eatss
