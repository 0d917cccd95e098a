// conv2d.cu -- tiled executor of the 4-D convolution-2d nest (P:191, P:272-284,
// Figs. 10, 11, 13):
//
//   for i < m, j < m (m = n - f + 1):  out[i][j] = 0;
//                                      for p < f, q < f:  out[i][j] += inp[i+p][j+q] * W[p][q]   (R-N9)
//
// Tile (Ti, Tj, Tp, Tq) -> GPU mapping (Fig. 4): one CTA per (Ti x Tj) block of
// out (B-set {j, i}, l_s1 = j along the lanes).  The reduction loops p, q are not parallel; one thread
// runs all of them for its outputs in the nest's order (p, then q, ascending), which is the order any
// (Tp, Tq) tiling of those loops executes -- the filter tile sizes change nothing in the arithmetic.
// The CTA's input window (rows [ti0, ti0+Ti+f-1), columns [tj0, tj0+Tj+f-1) rounded to 16 bytes) is
// brought into shared memory by the bulk-copy engine, one cp.async.bulk per window row completing on
// an mbarrier (row chunks when a window exceeds the per-CTA budget).  Each thread owns a 16-byte
// column group (4 outputs) and walks a run of rows, keeping the last f input row segments in a
// register ring, so each output row costs one new row segment from shared memory.  The filter lives
// in registers.  HBM-bound at the config sizes (8 bytes per output, 2 f^2 flop).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include "tc_ptx.cuh"

namespace eatss {

using tcm::mbar_expect_tx;
using tcm::mbar_init;
using tcm::mbar_wait;
using tcm::su32;

namespace {

constexpr int kSmemBudget = 64 * 1024;  // bytes per window slot (several CTAs per SM in flight)

__device__ __forceinline__ void bulk_row(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(su32(dst)),
        "l"(src), "r"(bytes), "r"(su32(bar))
        : "memory");
}

struct CvArgs {
    float *out;
    const float *inp, *W;
    int64_t n, m;
    int f, Ti, Tj;
    int groups, segs;  // column groups per tile, row segments per chunk
    int rc;            // rows per chunk (outputs)
    int wc;            // window width (floats, multiple of 4)
    int64_t gx, cpt;   // tiles along j, chunks per tile
    int64_t units;     // gy * cpt * gx work units (tile row-chunks)
    int slot_f;        // floats per window slot
    int nslot;         // 1: one CTA per unit; 2: persistent CTAs with a prefetching second slot
    int tma;           // 1: the window is one 2-D TMA box {wc, rc + f - 1} (wc <= 256, rc + f - 1 <= 256)
    int32_t *counts;
};

// Work unit u -> (tile row ti0, chunk start c0, rows, tile column tj0); units run along j fastest so
// consecutive CTAs stream adjacent columns of the same input rows.
struct Unit {
    int64_t c0, tj0, jhi;
    int rows;
};
__device__ __forceinline__ Unit unit_of(const CvArgs &a, int64_t u) {
    Unit w;
    const int uu = (int)u, gx = (int)a.gx, cpt = (int)a.cpt;  // units < 2^31 (launch_conv2d)
    const int bx = uu % gx, rest = uu / gx;
    const int ch = rest % cpt, by = rest / cpt;
    const int64_t ti0 = (int64_t)by * a.Ti, ihi = min(ti0 + a.Ti, a.m);
    w.c0 = ti0 + (int64_t)ch * a.rc;
    w.rows = (int)max((int64_t)0, min((int64_t)a.rc, ihi - w.c0));
    w.tj0 = (int64_t)bx * a.Tj;
    w.jhi = min(w.tj0 + a.Tj, a.m);
    return w;
}

// CTA b runs units b, b + grid, ...  With nslot = 2 (persistent grid) the bulk copies of the next
// unit are in flight while the current one is computed; with nslot = 1 the grid has one CTA per
// unit (the default: more CTAs resident per SM, no per-CTA unit loop).  F > 0: compile-time filter size with the
// register ring; F == 0: runtime f, direct shared reads.
template <int F, bool COVER>
__global__ void __launch_bounds__(256) conv2d_kernel(CvArgs a, const __grid_constant__ CUtensorMap wmap) {
    extern __shared__ __align__(128) unsigned char win_raw[];
    // TMA destinations must be 128-byte aligned
    float *win = reinterpret_cast<float *>(win_raw + ((128u - (su32(win_raw) & 127u)) & 127u));
    __shared__ uint64_t bar[2];
    constexpr int NV = F > 0 ? (F + 6) / 4 : 1;  // float4 per row segment: 4 + F - 1 floats
    const int f = F > 0 ? F : a.f;
    const int tid = threadIdx.x;
    const int g = tid % a.groups, seg = tid / a.groups;
    if constexpr (COVER) {  // the same unit / segment / group ownership, visit counts only
        for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x) {
            const Unit w = unit_of(a, u);
            const int64_t j = w.tj0 + 4 * g;
            const int per = (w.rows + a.segs - 1) / a.segs;
            const int rs = seg * per, re = min(w.rows, rs + per);
            for (int o = rs; o < re; o++)
                for (int c = 0; c < 4; c++)
                    if (j + c < w.jhi)
                        for (int p = 0; p < f; p++)
                            for (int q = 0; q < f; q++)
                                atomicAdd(a.counts + ((((w.c0 + o) * a.m) + j + c) * f + p) * f + q, 1);
        }
        return;
    }
    float wf[F > 0 ? F * F : 1];
    if constexpr (F > 0) {
#pragma unroll
        for (int e = 0; e < F * F; e++) wf[e] = __ldg(a.W + e);
    }
    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();
    const int nt = min(32, (int)blockDim.x);  // issuing lanes (a CTA may be narrower than a warp)
    auto issue = [&](int64_t u, int slot) {
        if (tid >= nt) return;
        const Unit w = unit_of(a, u);
        if (w.rows <= 0) return;
        const int64_t ce = min(a.n, w.tj0 + a.wc);
        const unsigned rowbytes = (unsigned)((ce - w.tj0) * 4);
        const int wr = w.rows + f - 1;  // window rows (c0 + wr <= n always)
        float *dst = win + slot * a.slot_f;
        if (a.tma) {  // one box; rows / columns past the image are zero-filled (never used by an output)
            if (tid == 0) {
                mbar_expect_tx(&bar[slot], (unsigned)(a.wc * (a.rc + f - 1) * 4));
                tcm::tma_2d<1>(dst, &wmap, (int)w.tj0, (int)w.c0, su32(&bar[slot]));
            }
            return;
        }
        if (tid == 0) mbar_expect_tx(&bar[slot], rowbytes * (unsigned)wr);
        __syncwarp(nt == 32 ? 0xffffffffu : (1u << nt) - 1u);
        for (int r = tid; r < wr; r += nt)
            bulk_row(dst + r * a.wc, a.inp + (w.c0 + r) * a.n + w.tj0, rowbytes, &bar[slot]);
    };
    unsigned phase[2] = {0, 0};
    int slot = 0;
    if ((int64_t)blockIdx.x < a.units) issue(blockIdx.x, 0);
    for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x, slot ^= (a.nslot - 1)) {
        if (a.nslot == 2 && u + gridDim.x < a.units) issue(u + gridDim.x, slot ^ 1);  // freed last iteration
        const Unit w = unit_of(a, u);
        if (w.rows <= 0) continue;
        mbar_wait(&bar[slot], phase[slot]);
        phase[slot] ^= 1;
        const int64_t j = w.tj0 + 4 * g;  // first output column of the group
        if (j < w.jhi) {
            // this thread's output rows of the unit: [rs, re)
            const int per = (w.rows + a.segs - 1) / a.segs;
            const int rs = seg * per, re = min(w.rows, rs + per);
            const float *colp = win + slot * a.slot_f + 4 * g;
            const bool vec = (a.m % 4 == 0) && j + 3 < w.jhi;
            auto store = [&](int r, const float (&o)[4]) {
                float *dst = a.out + (w.c0 + r) * a.m + j;
                if (vec) {
                    *reinterpret_cast<float4 *>(dst) = make_float4(o[0], o[1], o[2], o[3]);
                } else {
#pragma unroll
                    for (int c = 0; c < 4; c++)
                        if (j + c < w.jhi) dst[c] = o[c];
                }
            };
            if constexpr (F > 0) {
                float rg[F][4 * NV];
                auto load = [&](int r, float(&dst)[4 * NV]) {
#pragma unroll
                    for (int v = 0; v < NV; v++) {
                        const float4 x = *reinterpret_cast<const float4 *>(colp + r * a.wc + 4 * v);
                        dst[4 * v] = x.x; dst[4 * v + 1] = x.y; dst[4 * v + 2] = x.z; dst[4 * v + 3] = x.w;
                    }
                };
                if (rs < re) {
#pragma unroll
                    for (int p = 0; p < F - 1; p++) load(rs + p, rg[p]);
                    for (int base = rs; base < re; base += F) {
#pragma unroll
                        for (int uu = 0; uu < F; uu++) {
                            const int o = base + uu;
                            if (o < re) {
                                load(o + F - 1, rg[(uu + F - 1) % F]);
                                float ov[4];
#pragma unroll
                                for (int c = 0; c < 4; c++) {
                                    float sacc = 0.f;
#pragma unroll
                                    for (int p = 0; p < F; p++)
#pragma unroll
                                        for (int q = 0; q < F; q++)
                                            sacc = fmaf(rg[(uu + p) % F][c + q], wf[p * F + q], sacc);
                                    ov[c] = sacc;
                                }
                                store(o, ov);
                            }
                        }
                    }
                }
            } else {
                for (int o = rs; o < re; o++) {
                    float ov[4];
                    for (int c = 0; c < 4; c++) {
                        float sacc = 0.f;
                        for (int p = 0; p < f; p++)
                            for (int q = 0; q < f; q++)
                                sacc = fmaf(colp[(o + p) * a.wc + c + q], __ldg(a.W + p * f + q), sacc);
                        ov[c] = sacc;
                    }
                    store(o, ov);
                }
            }
        }
        __syncthreads();  // this slot is refilled by the issue of the next iteration but one
    }
}

// General path (n % 4 != 0 or Tj % 4 != 0): one thread per output, reads through L1.
template <bool COVER>
__global__ void __launch_bounds__(256) conv2d_general(CvArgs a) {
    const int64_t ti0 = (int64_t)blockIdx.y * a.Ti, tj0 = (int64_t)blockIdx.x * a.Tj;
    const int64_t ihi = min(ti0 + a.Ti, a.m), jhi = min(tj0 + a.Tj, a.m);
    const int64_t cols = jhi - tj0, pts = (ihi - ti0) * cols;
    const int f = a.f;
    for (int64_t e = threadIdx.x; e < pts; e += blockDim.x) {
        const int64_t i = ti0 + e / cols, j = tj0 + e % cols;
        if constexpr (COVER) {
            for (int p = 0; p < f; p++)
                for (int q = 0; q < f; q++) atomicAdd(a.counts + ((i * a.m + j) * f + p) * f + q, 1);
        } else {
            float s = 0.f;
            for (int p = 0; p < f; p++)
                for (int q = 0; q < f; q++) s = fmaf(__ldg(a.inp + (i + p) * a.n + j + q), __ldg(a.W + p * f + q), s);
            a.out[i * a.m + j] = s;
        }
    }
}

}  // namespace

// Launch geometry (also reported by eatss_plan).  Returns false for the general path.
bool conv2d_plan(int64_t n, int64_t f, const int64_t *tiles, int64_t *gx, int64_t *gy, int *threads, int *smem,
                 int *rc, int *wc, int *groups, int *segs) {
    const int64_t m = n - f + 1;
    const int64_t Ti = std::min(tiles[0], m), Tj = std::min(tiles[1], m);
    *gx = (m + Tj - 1) / Tj;
    *gy = (m + Ti - 1) / Ti;
    // 16-byte window rows need n % 4 == 0 and tile columns starting at multiples of 4 (Tj % 4 == 0, or
    // one tile spanning all columns)
    const bool fast = n % 4 == 0 && (Tj % 4 == 0 || Tj >= m) && f <= 32;
    if (!fast) {
        *threads = 256; *smem = 0; *rc = (int)Ti; *wc = 0; *groups = 0; *segs = 0;
        return false;
    }
    const int64_t w = (Tj + f - 1 + 3) / 4 * 4;
    *wc = (int)w;
    const int pad = 32;  // register-ring over-read past the last group (<= 3 float4)
    int64_t r = kSmemBudget / (w * 4) - (f - 1);
    r = std::max<int64_t>(1, std::min<int64_t>(r, Ti));
    *rc = (int)r;
    *smem = (int)(((r + f - 1) * w + pad) * 4);  // one window slot per CTA (one unit per CTA)
    const int gr = (int)((Tj + 3) / 4);
    *groups = std::min(gr, 256);
    // row segments: each thread walks >= 8 rows of a chunk, at most 256 threads
    const int sg = (int)std::max<int64_t>(1, std::min<int64_t>(256 / *groups, (r + 7) / 8));
    *segs = sg;
    *threads = *groups * sg;
    return gr <= 256;
}

cudaError_t launch_conv2d(float *out, const float *inp, const float *W, int64_t n, int64_t f, const int64_t *tiles,
                          int32_t *counts, cudaStream_t s, int64_t *launched) {
    CvArgs a{};
    a.out = out; a.inp = inp; a.W = W; a.counts = counts;
    a.n = n; a.f = (int)f; a.m = n - f + 1;
    a.Ti = (int)std::min(tiles[0], a.m); a.Tj = (int)std::min(tiles[1], a.m);
    int64_t gx, gy;
    int threads, smem, rc, wc, groups, segs;
    const bool fast = conv2d_plan(n, f, tiles, &gx, &gy, &threads, &smem, &rc, &wc, &groups, &segs);
    a.rc = rc; a.wc = wc; a.groups = groups; a.segs = segs;
    if (!fast) {
        dim3 grid((unsigned)gx, (unsigned)gy);
        if (launched) (*launched)++;
        if (counts) conv2d_general<true><<<grid, 256, 0, s>>>(a);
        else conv2d_general<false><<<grid, 256, 0, s>>>(a);
        return cudaGetLastError();
    }
    a.gx = gx;
    a.cpt = (a.Ti + rc - 1) / rc;
    a.units = gy * a.cpt * gx;
    a.slot_f = smem / 4;  // floats of the (single) slot
    a.nslot = 1;
    CUtensorMap wmap{};
    a.tma = 0;
    static const bool tma_on = [] {
        const char *e = getenv("EATSS_CONV_TMA");
        return !(e && atoi(e) == 0);
    }();
    if (tma_on && !counts && wc <= 256 && rc + f - 1 <= 256 && tcm::encode_fn() &&
        tcm::make_map(&wmap, inp, n, n, n, wc, (int)(rc + f - 1), CU_TENSOR_MAP_SWIZZLE_NONE))
        a.tma = 1;
    smem += 128;  // manual 128-byte alignment of the window
    if (a.units >= (int64_t)1 << 31) return cudaErrorInvalidConfiguration;
    if (launched) (*launched)++;
    cudaError_t e = cudaSuccess;
#define EATSS_CV(FV)                                                                                       \
    if (counts) {                                                                                          \
        conv2d_kernel<FV, true><<<(unsigned)std::min<int64_t>(a.units, 65535), threads, 0, s>>>(a, wmap);  \
    } else {                                                                                               \
        e = cudaFuncSetAttribute(conv2d_kernel<FV, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        if (e != cudaSuccess) return e;                                                                    \
        conv2d_kernel<FV, false><<<(unsigned)a.units, threads, smem, s>>>(a, wmap);                        \
    }
    switch (f) {
        case 3: EATSS_CV(3) break;
        case 5: EATSS_CV(5) break;
        case 7: EATSS_CV(7) break;
        default: EATSS_CV(0) break;
    }
#undef EATSS_CV
    return cudaGetLastError();
}

}  // namespace eatss
