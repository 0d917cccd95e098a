// mttkrp.cu -- tiled executor of the 4-D mttkrp nest (Fig. 10):
//
//   for i < ni, j < nj, k < nk, l < nl:   A[i][j] += B[i][k][l] * C[k][j] * D[l][j]      (reading R-N8)
//
// Tile (Ti, Tj, Tk, Tl) -> GPU mapping (Fig. 4):
//   * one CTA per (Ti x Tj) block of A (the B-set {j, i} of the model, l_s1 = j along the lanes);
//   * the reduction loops k, l are not parallel; their tile sizes set the staging: a stage is
//     one k and a Tl-wide run of l (at most 32 l per stage), i.e. the SH_set reference B[i][k][l] is
//     staged in shared memory Ti rows x Tl at a time, the L1_set references C[k][j] and D[l][j] are
//     read through L1/L2 (D staged next to B because every row of the CTA reuses it);
//   * when the (i, j) blocks alone do not fill the machine, whole Tk-tiles of the k loop are split
//     across CTAs (grid.z) -- a launch-plan decision, not a tile change; the partial sums go to a
//     library-owned workspace and a second kernel adds them to A in split order (deterministic).
//
// Arithmetic (legal reassociation of the k, l sums, within the fp32 tolerance):
//   A[i][j] += sum_k C[k][j] * ( sum_l B[i][k][l] * D[l][j] )
// i.e. one FFMA per iteration point plus one per (i, j, k): the Khatri-Rao factor C[k][j]*D[l][j]
// is never formed per point.  Operands are streamed with cp.async (16-byte LDGSTS) through a
// 4-stage shared-memory ring; each thread owns RM rows x 4 consecutive columns of A.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

namespace eatss {

namespace {

constexpr int kStages = 4;
constexpr int kMaxSW = 32;  // l per stage
constexpr int kMaxSmem = 160 * 1024;  // ring bytes per CTA
constexpr int kMaxBChunks = 8;         // 16-byte chunks of B per thread and k of a stage
constexpr int kThreads = 128;
constexpr int kKS = 2;                 // k per stage when a stage spans a whole l-tile
constexpr int kMaxDChunks = 2;         // 16-byte chunks of D per thread and stage

__device__ __forceinline__ void cp16(void *smem, const void *gmem, bool valid) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    const int n = valid ? 16 : 0;  // src-size 0: zero-fill
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(n) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() {
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}

struct MtArgs {
    float *A;
    const float *B, *C, *D;
    float *ws;  // [S][ni][nj] partials when S > 1
    int64_t ni, nj, nk, nl;
    int Ti, Tj, Tk, Tl;
    int bx, by;     // threads along j (4 columns each) and along i
    int sw, lgc;    // l per stage (power of two in 4..32, divides Tl), log2(sw / 4)
    int ks;         // k per stage (> 1 only when one stage spans a whole l-tile)
    int pps;        // (k-tile, l-tile) pairs per split
    int S;          // splits (grid.z)
    int32_t *counts;
};

// Reduction cursor of a CTA: pairs (k-tile kt, l-tile lt), kt major; inside a pair the k of the
// k-tile in groups of ks, inside a group the sub-stages (sw l each) of the l-tile.  No divisions.
struct Cursor {
    int64_t kt, lt;
    int kk, sub;
};
__device__ __forceinline__ void advance(Cursor &c, const MtArgs &a, int spt, int64_t nlt, int ks) {
    if (++c.sub < spt) return;
    c.sub = 0;
    const int64_t tkl = min((int64_t)a.Tk, a.nk - c.kt * a.Tk);
    if ((c.kk += ks) < tkl) return;
    c.kk = 0;
    if (++c.lt < nlt) return;
    c.lt = 0;
    c.kt++;
}

// Fast path: nj % 4 == 0, nl % 4 == 0, Tj % 4 == 0, Tl % 4 == 0 (mttkrp_plan).  128 threads; each
// owns RM rows x 4 consecutive columns of A per row pass.  A stage holds B[R rows][ks k][sw l] and
// D[sw l][4 bx columns].
// SW, BXT, KS > 0: compile-time stage width, threads along j and k per stage (shared-memory
// addresses become immediates); 0: the runtime values of MtArgs.
template <int RM, bool COVER, int SW = 0, int BXT = 0, int KS = 0>
__global__ void __launch_bounds__(128, RM <= 4 ? 4 : 2) mttkrp_kernel(MtArgs a) {
    extern __shared__ __align__(16) float sm[];
    const int sw = SW > 0 ? SW : a.sw;
    const int bxv = BXT > 0 ? BXT : a.bx;
    const int byv = BXT > 0 ? kThreads / BXT : a.by;
    const int ksv = KS > 0 ? KS : a.ks;
    const int tx = threadIdx.x % bxv, ty = threadIdx.x / bxv;
    const int nthr = bxv * byv;
    const int R = byv * RM;             // rows per row pass
    const int bpitch = sw + 4;         // B stage row pitch (floats), staggers banks
    const int rpitch = ksv * bpitch;    // one row's ks k-slices
    const int dw = bxv * 4;             // D stage row width (floats)
    const int stage_f = R * rpitch + sw * dw;
    const int64_t ti0 = (int64_t)blockIdx.y * a.Ti, tj0 = (int64_t)blockIdx.x * a.Tj;
    const int64_t ihi = min(ti0 + a.Ti, a.ni), jhi = min(tj0 + a.Tj, a.nj);
    const int64_t nkt = (a.nk + a.Tk - 1) / a.Tk, nlt = (a.nl + a.Tl - 1) / a.Tl;
    const int spt = (a.Tl + sw - 1) / sw;  // sub-stages per l-tile
    const int64_t p0 = (int64_t)blockIdx.z * a.pps, p1 = min(p0 + a.pps, nkt * nlt);
    if (p0 >= p1) return;  // (a.S > 1: its partial plane is never read -- reduce covers z < S only)
    // stages of this CTA per pass: sum over its pairs of ceil(k in the pair's k-tile / ks) x spt
    int64_t nst;
    {
        const int64_t kf = p0 / nlt, kl = (p1 - 1) / nlt;
        auto grp = [&](int64_t kt) { return (min((int64_t)a.Tk, a.nk - kt * a.Tk) + ksv - 1) / ksv; };
        if (kf == kl) nst = (p1 - p0) * grp(kf);
        else nst = (nlt - p0 % nlt) * grp(kf) + (kl - kf - 1) * nlt * grp(kf) + ((p1 - 1) % nlt + 1) * grp(kl);
        nst *= spt;
    }
    const int64_t nknl = a.nk * a.nl;
    const int cpr = sw >> 2, lgc = SW > 0 ? (SW == 4 ? 0 : SW == 8 ? 1 : SW == 16 ? 2 : 3) : a.lgc;  // 16-byte chunks per staged B row slice
    for (int64_t jp = tj0; jp < jhi; jp += dw) {                   // column passes (Tj > 4*bx)
        const int64_t j = jp + 4 * tx;
        const bool jok = j < jhi;
        for (int64_t ip = ti0; ip < ihi; ip += R) {                // row passes (Ti > R)
            if constexpr (COVER) {
                for (int r = 0; r < RM; r++) {
                    const int64_t i = ip + ty + (int64_t)byv * r;
                    if (i >= ihi || !jok) continue;
                    for (int64_t p = p0; p < p1; p++) {
                        const int64_t kt = p / nlt, lt = p % nlt;
                        for (int64_t k = kt * a.Tk; k < min((kt + 1) * a.Tk, a.nk); k++)
                            for (int64_t l = lt * a.Tl; l < min((lt + 1) * a.Tl, a.nl); l++)
                                for (int c = 0; c < 4; c++)
                                    if (j + c < jhi)
                                        atomicAdd(a.counts + ((i * a.nj + j + c) * a.nk + k) * a.nl + l, 1);
                    }
                }
                continue;
            }
            Cursor ci{p0 / nlt, p0 % nlt, 0, 0};  // issue cursor
            Cursor cc = ci;                        // compute cursor
            // this thread's 16-byte chunks of every stage slice, fixed for the pass (mttkrp_plan caps
            // them at kMaxBChunks of B and kMaxDChunks of D per thread): global row / l (-1 = none)
            // and the shared offset with the chunk's column index packed above bit 20
            int brow_i[kMaxBChunks], bso[kMaxBChunks], dl[kMaxDChunks], dso[kMaxDChunks];
#pragma unroll
            for (int m = 0; m < kMaxBChunks; m++) {
                const int c = threadIdx.x + m * nthr;
                const int row = c >> lgc, q = c & (cpr - 1);
                // -2: no such chunk (nothing is written); -1: a row past the tile (zero-filled)
                brow_i[m] = c >= (R << lgc) ? -2 : ip + row < ihi ? (int)(ip + row) : -1;
                bso[m] = (row * rpitch + 4 * q) | (q << 20);
            }
#pragma unroll
            for (int m = 0; m < kMaxDChunks; m++) {
                const int c = threadIdx.x + m * nthr;
                const int l = c / bxv, q = c - l * bxv;
                dl[m] = (c < sw * bxv && jp + 4 * q < jhi) ? l : -1;
                dso[m] = l * dw + 4 * q;
            }
            auto issue = [&](int64_t s) {
                float *st = sm + (int)(s % kStages) * stage_f;
                const int64_t k = ci.kt * a.Tk + ci.kk;
                const int kc = (int)min((int64_t)ksv, min((ci.kt + 1) * a.Tk, a.nk) - k);
                const int64_t l0 = ci.lt * a.Tl + (int64_t)ci.sub * sw;
                const int w = (int)min((int64_t)sw, min((ci.lt + 1) * a.Tl, a.nl) - l0);
                const float *bk = a.B + k * a.nl + l0;
                for (int kk = 0; kk < kc; kk++, bk += a.nl) {
#pragma unroll
                    for (int m = 0; m < kMaxBChunks; m++) {
                        if (brow_i[m] == -2) continue;
                        const int q4 = (bso[m] >> 20) * 4;
                        const bool v = brow_i[m] >= 0 && q4 < w;
                        cp16(st + (bso[m] & 0xfffff) + kk * bpitch, v ? bk + (int64_t)brow_i[m] * nknl + q4 : a.B, v);
                    }
                }
                float *ds = st + R * rpitch;
                const float *dk = a.D + l0 * a.nj + jp;
#pragma unroll
                for (int m = 0; m < kMaxDChunks; m++) {
                    if (dl[m] < 0) continue;
                    const bool v = dl[m] < w;
                    cp16(ds + dso[m], v ? dk + (int64_t)dl[m] * a.nj + (dso[m] - dl[m] * dw) : a.D, v);
                }
                advance(ci, a, spt, nlt, ksv);
            };
            float acc[RM][4], t[RM][4];
#pragma unroll
            for (int r = 0; r < RM; r++)
#pragma unroll
                for (int c = 0; c < 4; c++) acc[r][c] = t[r][c] = 0.f;
            for (int s = 0; s < kStages - 1; s++) {
                if (s < nst) issue(s);
                cp_commit();
            }
            for (int64_t s = 0; s < nst; s++) {
                cp_wait<kStages - 2>();
                __syncthreads();
                if (s + kStages - 1 < nst) issue(s + kStages - 1);
                cp_commit();
                const float *st = sm + (int)(s % kStages) * stage_f;
                const float *ds = st + R * rpitch + 4 * tx;
                const int64_t k0s = cc.kt * a.Tk + cc.kk;
                const int kc = (int)min((int64_t)ksv, min((cc.kt + 1) * a.Tk, a.nk) - k0s);
                const bool fold = cc.sub == spt - 1;  // (k, l-tile) complete after this stage
                for (int kk = 0; kk < kc; kk++) {
                    const float *brow = st + ty * rpitch + kk * bpitch;
                    // C[k][j] of this k-slice, loaded before the slice's FFMAs hide its latency
                    float4 c = make_float4(0.f, 0.f, 0.f, 0.f);
                    if (fold && jok) c = __ldg(reinterpret_cast<const float4 *>(a.C + (k0s + kk) * a.nj + j));
#pragma unroll
                    for (int l = 0; l < sw; l += 4) {
                        float b[RM][4], d[4][4];
#pragma unroll
                        for (int r = 0; r < RM; r++) {
                            const float4 v = *reinterpret_cast<const float4 *>(brow + byv * r * rpitch + l);
                            b[r][0] = v.x; b[r][1] = v.y; b[r][2] = v.z; b[r][3] = v.w;
                        }
#pragma unroll
                        for (int u = 0; u < 4; u++) {
                            const float4 v = *reinterpret_cast<const float4 *>(ds + (l + u) * dw);
                            d[u][0] = v.x; d[u][1] = v.y; d[u][2] = v.z; d[u][3] = v.w;
                        }
                        // l-component outermost: successive updates of one accumulator are 4*RM
                        // independent FFMAs apart (covers the FMA latency at two warps per scheduler)
#pragma unroll
                        for (int u = 0; u < 4; u++)
#pragma unroll
                            for (int r = 0; r < RM; r++)
#pragma unroll
                                for (int c = 0; c < 4; c++) t[r][c] = fmaf(b[r][u], d[u][c], t[r][c]);
                    }
                    if (fold) {  // fold C[k][j] in
#pragma unroll
                        for (int r = 0; r < RM; r++) {
                            acc[r][0] = fmaf(c.x, t[r][0], acc[r][0]); acc[r][1] = fmaf(c.y, t[r][1], acc[r][1]);
                            acc[r][2] = fmaf(c.z, t[r][2], acc[r][2]); acc[r][3] = fmaf(c.w, t[r][3], acc[r][3]);
                            t[r][0] = t[r][1] = t[r][2] = t[r][3] = 0.f;
                        }
                    }
                }
                advance(cc, a, spt, nlt, ksv);
            }
            cp_wait<0>();
            __syncthreads();  // the ring is reused by the next pass
            if (!jok) continue;
#pragma unroll
            for (int r = 0; r < RM; r++) {
                const int64_t i = ip + ty + (int64_t)byv * r;
                if (i >= ihi) continue;
                const float4 v = make_float4(acc[r][0], acc[r][1], acc[r][2], acc[r][3]);
                if (a.S > 1) {
                    *reinterpret_cast<float4 *>(a.ws + ((int64_t)blockIdx.z * a.ni + i) * a.nj + j) = v;
                } else {
                    float4 *p = reinterpret_cast<float4 *>(a.A + i * a.nj + j);
                    float4 o = *p;
                    o.x += v.x; o.y += v.y; o.z += v.z; o.w += v.w;
                    *p = o;
                }
            }
        }
    }
}

// A[i][j] += sum_{z < S} ws[z][i][j], z ascending (deterministic split order).
__global__ void mttkrp_reduce(float *__restrict__ A, const float *__restrict__ ws, int64_t n4, int64_t plane4, int S) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n4; e += (int64_t)gridDim.x * blockDim.x) {
        float4 s = reinterpret_cast<const float4 *>(ws)[e];
        for (int z = 1; z < S; z++) {
            const float4 v = reinterpret_cast<const float4 *>(ws)[(int64_t)z * plane4 + e];
            s.x += v.x; s.y += v.y; s.z += v.z; s.w += v.w;
        }
        float4 o = reinterpret_cast<float4 *>(A)[e];
        o.x += s.x; o.y += s.y; o.z += s.z; o.w += s.w;
        reinterpret_cast<float4 *>(A)[e] = o;
    }
}

// General path (any sizes / tiles): one thread per A element of the CTA's (Ti x Tj) block, the same
// factorised sums read through L1.  COVER: visit counts of the iteration points instead.
template <bool COVER>
__global__ void __launch_bounds__(256) mttkrp_general(MtArgs a) {
    const int64_t ti0 = (int64_t)blockIdx.y * a.Ti, tj0 = (int64_t)blockIdx.x * a.Tj;
    const int64_t ihi = min(ti0 + a.Ti, a.ni), jhi = min(tj0 + a.Tj, a.nj);
    const int64_t cols = jhi - tj0, pts = (ihi - ti0) * cols;
    for (int64_t e = threadIdx.x; e < pts; e += blockDim.x) {
        const int64_t i = ti0 + e / cols, j = tj0 + e % cols;
        if constexpr (COVER) {
            for (int64_t k = 0; k < a.nk; k++)
                for (int64_t l = 0; l < a.nl; l++) atomicAdd(a.counts + ((i * a.nj + j) * a.nk + k) * a.nl + l, 1);
        } else {
            float acc = 0.f;
            for (int64_t k = 0; k < a.nk; k++) {
                const float *b = a.B + (i * a.nk + k) * a.nl;
                float t = 0.f;
                for (int64_t l = 0; l < a.nl; l++) t = fmaf(__ldg(b + l), __ldg(a.D + l * a.nj + j), t);
                acc = fmaf(__ldg(a.C + k * a.nj + j), t, acc);
            }
            a.A[i * a.nj + j] += acc;
        }
    }
}

int sm_count() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    }
    return n;
}

}  // namespace

// Launch geometry of the fast path (also reported by eatss_plan).  Returns false when the general
// path runs (misaligned sizes / tile).
bool mttkrp_plan(const int64_t *dims, const int64_t *tiles, int64_t *gx, int64_t *gy, int64_t *gz, int *bx, int *by,
                 int *rm, int *smem, int *splits, int *sw_out, int *ks_out) {
    const int64_t ni = dims[0], nj = dims[1], nk = dims[2], nl = dims[3];
    const int64_t Ti = std::min(tiles[0], ni), Tj = std::min(tiles[1], nj), Tk = std::min(tiles[2], nk),
                  Tl = std::min(tiles[3], nl);
    *gx = (nj + Tj - 1) / Tj;
    *gy = (ni + Ti - 1) / Ti;
    *gz = 1;
    *splits = 1;
    // 16-byte chunks: rows of A, C, D and B start at multiples of 4 columns, and every staged run of l
    // must hold whole chunks of one l-tile
    const bool fast = nj % 4 == 0 && nl % 4 == 0 && Tj % 4 == 0 && (Tl % 4 == 0 || Tl >= nl);
    if (!fast) {
        *bx = 256; *by = 1; *rm = 1; *smem = 0;
        return false;
    }
    const int b_x = (int)std::min<int64_t>(Tj / 4, 32);
    const int b_y = kThreads / b_x;
    // rows per thread: up to 8 (two CTAs of 128 threads per SM at ~230 registers: measured faster
    // than 4 rows at 128 registers and four CTAs -- 0.40 vs 0.46 ms at the config); EATSS_MT_MAXRM
    // (1, 2, 4, 8) overrides for experiments
    static const int max_rm = [] {
        const char *e = getenv("EATSS_MT_MAXRM");
        const int v = e ? atoi(e) : 8;
        return v == 1 || v == 2 || v == 4 ? v : 8;
    }();
    int r = 1;
    while (r < max_rm && (int64_t)b_y * r < Ti) r *= 2;
    // stage width: the largest power of two <= 32 dividing Tl (a stage never straddles two l-tiles)
    int sw = 4;
    while (sw < kMaxSW && Tl % (2 * sw) == 0) sw *= 2;
    auto bytes = [&](int rr, int ww, int kk) { return kStages * (b_y * rr * kk * (ww + 4) + ww * b_x * 4) * 4; };
    while (bytes(r, sw, 1) > kMaxSmem && r > 1) r /= 2;    // fewer rows per pass (more row passes)
    while (bytes(r, sw, 1) > kMaxSmem && sw > 4) sw /= 2;  // narrower stages
    // per-thread chunk caps: B slice = b_y*r rows x sw/4 chunks over b_x*b_y threads, D = sw x b_x
    while (r * sw > 4 * kMaxBChunks * b_x && sw > 4) sw /= 2;
    while (r * sw > 4 * kMaxBChunks * b_x && r > 1) r /= 2;
    while (sw > kMaxDChunks * b_y && sw > 4) sw /= 2;
    // several k per stage when one stage spans a whole l-tile (each k-slice then completes a
    // (k, l-tile) and is folded at once) and the ring stays within two CTAs per SM
    int ks = 1;
    if ((Tl + sw - 1) / sw == 1)
        while (ks < kKS && ks < Tk && bytes(r, sw, 2 * ks) <= kMaxSmem / 2 + 8192) ks *= 2;
    *bx = b_x; *by = b_y; *rm = r;
    *smem = bytes(r, sw, ks);
    if (ks_out) *ks_out = ks;
    if (sw_out) *sw_out = sw;
    // split the (k-tile, l-tile) pairs of the reduction across CTAs until ~2 CTAs per SM are in flight
    const int64_t blocks = *gx * *gy, npairs = ((nk + Tk - 1) / Tk) * ((nl + Tl - 1) / Tl);
    const int64_t target = (r <= 4 ? 4 : 2) * (int64_t)sm_count();  // CTAs resident per SM
    int64_t S = std::max<int64_t>(1, std::min<int64_t>(npairs, (target + blocks - 1) / blocks));
    const int64_t pps = (npairs + S - 1) / S;
    S = (npairs + pps - 1) / pps;
    *gz = S;
    *splits = (int)S;
    return true;
}

cudaError_t launch_mttkrp(float *A, const float *B, const float *C, const float *D, const int64_t *dims,
                          const int64_t *tiles, float *ws, int32_t *counts, cudaStream_t s, int64_t *launched) {
    MtArgs a{};
    a.A = A; a.B = B; a.C = C; a.D = D; a.ws = ws; a.counts = counts;
    a.ni = dims[0]; a.nj = dims[1]; a.nk = dims[2]; a.nl = dims[3];
    a.Ti = (int)std::min(tiles[0], a.ni); a.Tj = (int)std::min(tiles[1], a.nj);
    a.Tk = (int)std::min(tiles[2], a.nk); a.Tl = (int)std::min(tiles[3], a.nl);
    int64_t gx, gy, gz;
    int bx, by, rm, smem, S;
    int sw = 4, ks = 1;
    const bool fast = mttkrp_plan(dims, tiles, &gx, &gy, &gz, &bx, &by, &rm, &smem, &S, &sw, &ks);
    if (!fast) {
        dim3 grid((unsigned)gx, (unsigned)gy);
        if (counts) mttkrp_general<true><<<grid, 256, 0, s>>>(a);
        else mttkrp_general<false><<<grid, 256, 0, s>>>(a);
        if (launched) (*launched)++;
        return cudaGetLastError();
    }
    a.bx = bx; a.by = by;
    a.sw = sw;
    a.ks = ks;
    a.lgc = 0;
    while ((4 << a.lgc) < sw) a.lgc++;
    const int64_t npairs = ((a.nk + a.Tk - 1) / a.Tk) * ((a.nl + a.Tl - 1) / a.Tl);
    a.S = counts ? 1 : S;
    a.pps = (int)((npairs + a.S - 1) / a.S);
    if (counts) gz = 1;
    if (a.S > 1 && !ws) return cudaErrorInvalidValue;
    dim3 grid((unsigned)gx, (unsigned)gy, (unsigned)gz);
    const int threads = bx * by;
    const int sm = counts ? 0 : smem;
    cudaError_t e = cudaSuccess;
#define EATSS_MT(RMV)                                                                                   \
    if (rm == RMV) {                                                                                    \
        if (counts) {                                                                                   \
            mttkrp_kernel<RMV, true><<<grid, threads, 0, s>>>(a);                                       \
        } else {                                                                                        \
            e = cudaFuncSetAttribute(mttkrp_kernel<RMV, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm); \
            if (e != cudaSuccess) return e;                                                             \
            mttkrp_kernel<RMV, false><<<grid, threads, sm, s>>>(a);                                     \
        }                                                                                               \
    }
#define EATSS_MTS(RMV, SWV, KSV)                                                                        \
    if (!done && rm == RMV && a.sw == SWV && a.ks == KSV) {                                             \
        e = cudaFuncSetAttribute(mttkrp_kernel<RMV, false, SWV, 8, KSV>,                                 \
                                 cudaFuncAttributeMaxDynamicSharedMemorySize, sm);                      \
        if (e != cudaSuccess) return e;                                                                 \
        mttkrp_kernel<RMV, false, SWV, 8, KSV><<<grid, threads, sm, s>>>(a);                            \
        done = true;                                                                                    \
    }
    bool done = false;
    if (!counts && bx == 8) {  // Tj = 32 (the rank of the config, every EATSS tile of it): specialised
        EATSS_MTS(8, 16, 2) EATSS_MTS(8, 32, 2) EATSS_MTS(8, 8, 2) EATSS_MTS(8, 4, 2)
        EATSS_MTS(8, 16, 1) EATSS_MTS(8, 32, 1) EATSS_MTS(8, 8, 1) EATSS_MTS(8, 4, 1)
        EATSS_MTS(4, 16, 2) EATSS_MTS(4, 32, 2) EATSS_MTS(4, 8, 2) EATSS_MTS(4, 4, 2)
        EATSS_MTS(4, 16, 1) EATSS_MTS(4, 32, 1) EATSS_MTS(4, 8, 1) EATSS_MTS(4, 4, 1)
    }
    if (!done) {
        EATSS_MT(1) EATSS_MT(2) EATSS_MT(4) EATSS_MT(8)
    }
#undef EATSS_MTS
#undef EATSS_MT
    if (launched) (*launched)++;
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    if (a.S > 1) {
        const int64_t n4 = a.ni * a.nj / 4;
        const int blocks = (int)std::min<int64_t>((n4 + 255) / 256, 4 * (int64_t)sm_count());
        mttkrp_reduce<<<blocks, 256, 0, s>>>(A, ws, n4, n4, a.S);
        if (launched) (*launched)++;
        e = cudaGetLastError();
    }
    return e;
}

}  // namespace eatss
