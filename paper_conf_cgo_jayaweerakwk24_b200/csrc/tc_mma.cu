// tc_mma.cu -- tcgen05 3xTF32 GEMM for MMA-legal tiles (the
// "tensor-core EATSS mode", DESIGN.md §2.5 / §4.1c): Ti = 128 rows of i per CTA (UMMA M per
// SM), Tj <= 256 columns of j (UMMA N), k in blocks of 32 (one 128-byte swizzle atom of fp32).
//
// Same loop-nest semantics as the SIMT executor (Fig. 4: each CTA owns one Ti x Tj
// tile of C, k sequential); fp32-accurate via 3xTF32 (reading Q26):
//   C = beta*C + alpha * sum_k (Ahi*Bhi + Ahi*Blo + Alo*Bhi),
//   hi = rna_tf32(x), lo = rna_tf32(x - hi), computed once per operand by prep_kernel.
//
// B200-specific structure (what differs from the paper's one-tile-per-block CUDA code):
//  * CTA pairs (cta_group::2, cluster of 2 along i): the pair issues M = 256 MMAs; each CTA
//    keeps its own 128 x Tj accumulator tile but stages only HALF of the B tile, so shared
//    memory traffic per SM drops from 12 KB to 8 KB per MMA (the single-CTA kernel was
//    shared-memory-bandwidth bound at ~74% tensor-pipe activity).  Used when Tj/2 is a whole
//    number of 32-column swizzle atoms (or B is K-major); otherwise one CTA per tile.
//  * persistent clusters over a grouped (L2-friendly) tile order; the accumulator is drained
//    chunk by chunk (two TMEM buffers), so one tile's epilogue overlaps the next tile's MMAs.
//  * wave-quantisation tail: when the last wave would leave clusters idle, the remaining tiles
//    are split along k into `sp` parts whose partial sums are added to C with fp32 atomics
//    (C pre-scaled by beta once by prep_kernel).
// Pipeline (warp-specialised, mbarrier hand-off, one CTA per SM):
//   warp 0  TMA producer: Ahi/Alo (K-major, 128 x 32, SWIZZLE_128B) and Bhi/Blo (MN-major
//           32 x Tj/CG in 32-column SWIZZLE_128B_ATOM_32B boxes, or K-major Tj/CG x 32 when B
//           is transposed, as in syrk) into an S-stage ring;
//   warp 1  MMA issuer (leader CTA only): per 8-k step three kind::tf32 MMAs;
//           tcgen05.commit (multicast to the pair) frees ring slots / publishes chunks;
//   warp 2  TMEM allocation (512 columns = two accumulator buffers of up to 256);
//   warps 4..11 epilogue: tcgen05.ld of each finished chunk into fp32 registers, then C.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <map>
#include <mutex>
#include <string>

#include "contract.cuh"
#include "tc_ptx.cuh"

namespace eatss {
namespace tcm {


constexpr int BK = 32;   // k per stage (128-byte swizzle atom of fp32)
constexpr int BM = 128;  // rows of i per CTA (UMMA M per SM)
constexpr int NEPI = 8;  // epilogue warps (4..11): two per TMEM lane quarter
constexpr int NTHREADS = (4 + NEPI) * 32;
constexpr int GROUP_ROWS = 8;  // tile-order grouping (pair-rows per group) for L2 reuse

struct Args {
    int64_t M, N, K;
    float *__restrict__ C;
    int64_t ldc;
    float alpha, beta;
    int init_zero;
    int S;   // ring stages
    int R;   // k-blocks per accumulator chunk
    // persistent schedule
    int PI, TJ;   // row groups (of CG*128 rows) x column tiles
    int T;        // PI * TJ tiles
    int nfull;    // tiles done whole by one cluster
    int sp;       // k-parts per tail tile (1 = no split)
    int nunits;   // nfull + (T - nfull) * sp
    int nkb;      // k-blocks of 32
};

__host__ __device__ inline void tile_coords(int t, int PI, int TJ, int &pi, int &tj) {
    const int g = t / (GROUP_ROWS * TJ), r = t % (GROUP_ROWS * TJ);
    const int rows = PI - g * GROUP_ROWS < GROUP_ROWS ? PI - g * GROUP_ROWS : GROUP_ROWS;
    pi = g * GROUP_ROWS + r % rows;
    tj = r / rows;
}

struct Unit {
    int pi, tj, kb0, kb1;
    bool split;
};
__device__ __forceinline__ Unit unit_of(const Args &p, int u) {
    Unit w;
    int t;
    if (u < p.nfull) {
        t = u;
        w.kb0 = 0;
        w.kb1 = p.nkb;
        w.split = false;
    } else {
        const int v = u - p.nfull, part = v % p.sp;
        t = p.nfull + v / p.sp;
        w.kb0 = (int)((int64_t)part * p.nkb / p.sp);
        w.kb1 = (int)((int64_t)(part + 1) * p.nkb / p.sp);
        w.split = p.sp > 1;
    }
    tile_coords(t, p.PI, p.TJ, w.pi, w.tj);
    return w;
}

template <int BNT, bool TB, int CG>
__global__ void __launch_bounds__(NTHREADS, 1)
    tc_mma_kernel(const __grid_constant__ CUtensorMap mAhi, const __grid_constant__ CUtensorMap mAlo,
                  const __grid_constant__ CUtensorMap mBhi, const __grid_constant__ CUtensorMap mBlo, const Args p) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char *smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);  // stays a shared pointer
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const uint32_t rank = CG == 2 ? cta_rank() : 0u;
    const int cid = (int)blockIdx.x / CG, ncl = (int)gridDim.x / CG;
    constexpr int BNH = BNT / CG;                // B columns (rows, if TB) staged by this CTA
    constexpr int A_BYTES = BM * BK * 4;         // 16 KB
    constexpr int B_BYTES = BK * BNH * 4;        // <= 32 KB
    constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
    const int R = p.R;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)p.S * STAGE);
    uint64_t *empty = full + p.S;
    uint64_t *dfull = empty + p.S;
    uint64_t *dempty = dfull + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(dempty + 2);

    if (tid == 0) {
        for (int s = 0; s < p.S; s++) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, 1);
        }
        for (int b = 0; b < 2; b++) {
            mbar_init(dfull + b, 1);
            mbar_init(dempty + b, NEPI * CG);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&mAhi)) : "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&mBhi)) : "memory");
    }
    if (warp == 2) {
        if constexpr (CG == 1) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(su32(tmem_slot)),
                         "r"(512)
                         : "memory");
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::: "memory");
        } else {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(su32(tmem_slot)),
                         "r"(512)
                         : "memory");
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;\n" ::: "memory");
        }
    }
    fence_before();
    if constexpr (CG == 2) cluster_sync(); else __syncthreads();
    fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {  // ---------------------------------------------- TMA producer
            const uint32_t fbar0 = CG == 2 ? mapa(su32(full), 0) : su32(full);
            int it = 0;
            for (int u = cid; u < p.nunits; u += ncl) {
                const Unit w = unit_of(p, u);
                const int i0 = (w.pi * CG + (int)rank) * BM;
                const int jb = w.tj * BNT + (int)rank * BNH;
                for (int kb = w.kb0; kb < w.kb1; kb++, it++) {
                    const int s = it % p.S;
                    if (it >= p.S) mbar_wait(empty + s, (unsigned)(((it / p.S) - 1) & 1));
                    unsigned char *st = smem + (size_t)s * STAGE;
                    if (rank == 0) mbar_expect_tx(full + s, CG * STAGE);
                    const uint32_t fb = fbar0 + 8u * (uint32_t)s;
                    const int k0 = kb * BK;
                    tma_2d<CG>(st, &mAhi, k0, i0, fb);
                    tma_2d<CG>(st + A_BYTES, &mAlo, k0, i0, fb);
                    if constexpr (TB) {
                        tma_2d<CG>(st + 2 * A_BYTES, &mBhi, k0, jb, fb);
                        tma_2d<CG>(st + 2 * A_BYTES + B_BYTES, &mBlo, k0, jb, fb);
                    } else {
#pragma unroll
                        for (int g = 0; g < BNH / 32; g++) {
                            tma_2d<CG>(st + 2 * A_BYTES + g * (BK * 128), &mBhi, jb + 32 * g, k0, fb);
                            tma_2d<CG>(st + 2 * A_BYTES + B_BYTES + g * (BK * 128), &mBlo, jb + 32 * g, k0, fb);
                        }
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0 && rank == 0) {  // -------------------------------- MMA issuer (leader)
            constexpr uint32_t ID = idesc(BNT, CG, TB);
            // A (and K-major B): SW128 K-major, SBO = 8 rows x 128 B, +32 B per 8-k step.
            // MN-major B: SW128_BASE32B, LBO = stride of 32-column groups (BK rows x 128 B),
            // SBO = stride of the 4-row swizzle atoms (512 B), +1 KB per 8-k step.
            int it = 0, gc = 0;
            for (int u = cid; u < p.nunits; u += ncl) {
                const Unit w = unit_of(p, u);
                const int nk = w.kb1 - w.kb0;
                for (int x = 0; x < nk; x++, it++) {
                    const int s = it % p.S, bd = gc & 1;
                    const bool first = (x % R) == 0;
                    if (first && gc >= 2) mbar_wait_cluster(dempty + bd, (unsigned)(((gc - 2) >> 1) & 1));
                    mbar_wait(full + s, (unsigned)((it / p.S) & 1));
                    fence_after();
                    unsigned char *st = smem + (size_t)s * STAGE;
                    const uint32_t d = tmem + (uint32_t)(bd * 256);
#pragma unroll
                    for (int ks = 0; ks < BK / 8; ks++) {
                        const uint64_t ahi = desc_sw128(st + ks * 32, 16u, 1024u);
                        const uint64_t alo = desc_sw128(st + A_BYTES + ks * 32, 16u, 1024u);
                        uint64_t bhi, blo;
                        if constexpr (TB) {
                            bhi = desc_sw128(st + 2 * A_BYTES + ks * 32, 16u, 1024u);
                            blo = desc_sw128(st + 2 * A_BYTES + B_BYTES + ks * 32, 16u, 1024u);
                        } else {
                            bhi = desc_sw128(st + 2 * A_BYTES + ks * 1024, (uint32_t)(BK * 128), 512u, 1);
                            blo = desc_sw128(st + 2 * A_BYTES + B_BYTES + ks * 1024, (uint32_t)(BK * 128), 512u, 1);
                        }
                        mma_ss<CG>(d, ahi, bhi, ID, (first && ks == 0) ? 0u : 1u);
                        mma_ss<CG>(d, ahi, blo, ID, 1u);
                        mma_ss<CG>(d, alo, bhi, ID, 1u);
                    }
                    mma_commit<CG>(empty + s);
                    if ((x % R) == R - 1 || x == nk - 1) {
                        mma_commit<CG>(dfull + bd);
                        gc++;
                    }
                }
            }
        }
    } else if (warp >= 4) {  // ---------------------------------------- epilogue warps
        const int e = warp - 4, q = warp & 3, half = e >> 2;
        constexpr int CW = BNT / 2;  // columns per epilogue warp
        const uint32_t demp0 = CG == 2 ? mapa(su32(dempty), 0) : su32(dempty);
        int gc = 0;
        for (int u = cid; u < p.nunits; u += ncl) {
            const Unit w = unit_of(p, u);
            const int nch = (w.kb1 - w.kb0 + R - 1) / R;
            float acc[CW];
#pragma unroll
            for (int c = 0; c < CW; c++) acc[c] = 0.f;
            for (int ch = 0; ch < nch; ch++, gc++) {
                const int bd = gc & 1;
                mbar_wait(dfull + bd, (unsigned)((gc >> 1) & 1));
                fence_after();
#pragma unroll
                for (int c0 = 0; c0 < CW; c0 += 16) {
                    uint32_t v[16];
                    tmem_ld16(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(bd * 256 + half * CW + c0), v);
                    wait_ld();
#pragma unroll
                    for (int c = 0; c < 16; c++) acc[c0 + c] += __uint_as_float(v[c]);
                }
                fence_before();
                __syncwarp();
                if (lane == 0) {
                    if constexpr (CG == 2) mbar_arrive_cluster(demp0 + 8u * (uint32_t)bd);
                    else mbar_arrive(dempty + bd);
                }
            }
            // C(i, j) for row i = i0 + 32q + lane, columns jb .. jb + CW - 1
            const int64_t i = (int64_t)(w.pi * CG + (int)rank) * BM + q * 32 + lane;
            const int64_t jb = (int64_t)w.tj * BNT + half * CW;
            if (i < p.M && jb < p.N) {
                float *crow = p.C + i * p.ldc + jb;
                const bool vec = ((p.ldc & 3) == 0) && (jb + CW <= p.N);
                if (w.split) {  // C already holds beta*C (prep_kernel): add the partial sum
                    if (vec) {
#pragma unroll
                        for (int c = 0; c < CW; c += 4)
                            atomicAdd(reinterpret_cast<float4 *>(crow + c),
                                      make_float4(p.alpha * acc[c], p.alpha * acc[c + 1], p.alpha * acc[c + 2],
                                                  p.alpha * acc[c + 3]));
                    } else {
#pragma unroll
                        for (int c = 0; c < CW; c++)
                            if (jb + c < p.N) atomicAdd(crow + c, p.alpha * acc[c]);
                    }
                } else if (vec) {
#pragma unroll
                    for (int c = 0; c < CW; c += 4) {
                        float4 *cp = reinterpret_cast<float4 *>(crow + c);
                        float4 o = p.init_zero ? make_float4(0.f, 0.f, 0.f, 0.f) : *cp;
                        if (!p.init_zero) { o.x *= p.beta; o.y *= p.beta; o.z *= p.beta; o.w *= p.beta; }
                        o.x = fmaf(p.alpha, acc[c], o.x);
                        o.y = fmaf(p.alpha, acc[c + 1], o.y);
                        o.z = fmaf(p.alpha, acc[c + 2], o.z);
                        o.w = fmaf(p.alpha, acc[c + 3], o.w);
                        *cp = o;
                    }
                } else {
#pragma unroll
                    for (int c = 0; c < CW; c++) {
                        if (jb + c < p.N) {
                            const float o = p.init_zero ? 0.f : p.beta * crow[c];
                            crow[c] = fmaf(p.alpha, acc[c], o);
                        }
                    }
                }
            }
        }
    }
    __syncwarp();
    fence_before();
    if constexpr (CG == 2) cluster_sync(); else __syncthreads();
    if (warp == 2) {
        fence_after();
        if constexpr (CG == 1)
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(512) : "memory");
        else
            asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(512) : "memory");
    }
}

// Operand split for 3xTF32 (reading Q26).  mode 0: hi = rna_tf32(x), lo = rna_tf32(x - hi).
// mode 1 ("raw hi"): the tensor core reads only the tf32 bits of an fp32 container (it truncates),
// so the untouched operand already serves as hi = rz_tf32(x) and only lo = rna_tf32(x - rz_tf32(x))
// is materialised (hi == nullptr) -- one third less split traffic.  Rows of `cols` values at
// pitch ldx are written at pitch ldp (ldp = ldx: flat 16-byte vectors; else padded scalar copy).
__device__ __forceinline__ void split1(float v, int mode, float &h, float &l) {
    uint32_t hb, lb;
    if (mode == 0) {
        asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(hb) : "f"(v));
    } else {
        hb = __float_as_uint(v) & 0xFFFFE000u;
    }
    asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(lb) : "f"(v - __uint_as_float(hb)));
    h = mode == 0 ? __uint_as_float(hb) : v;
    l = __uint_as_float(lb);
}
struct SplitJob {
    const float *x;  // nullptr: no job
    int64_t ldx, rows, cols;
    float *hi, *lo;  // hi == nullptr: raw hi (mode 1, flat)
    int64_t ldp;
};
__device__ __forceinline__ void split_body(const SplitJob &j, int mode, int64_t t0, int64_t stride) {
    const float *__restrict__ x = j.x;
    float *__restrict__ hi = j.hi;
    float *__restrict__ lo = j.lo;
    const int64_t ldx = j.ldx, rows = j.rows, cols = j.cols, ldp = j.ldp;
    if (ldx == ldp) {  // flat over (rows - 1) * ld + cols elements
        const int64_t n = (rows - 1) * ldx + cols;
        const bool v4 = ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(lo) |
                          reinterpret_cast<uintptr_t>(hi)) & 15) == 0;
        const int64_t n4 = v4 ? n / 4 : 0;
        // SPLIT_U independent 16-byte loads in flight per thread before the first store
        // (one load per thread leaves ~32 KB per SM in flight: below the HBM latency-bandwidth product)
        constexpr int SPLIT_U = 4;
        for (int64_t v0 = t0; v0 < n4; v0 += SPLIT_U * stride) {
            float4 a[SPLIT_U];
#pragma unroll
            for (int u = 0; u < SPLIT_U; ++u)
                if (v0 + u * stride < n4) a[u] = reinterpret_cast<const float4 *>(x)[v0 + u * stride];
#pragma unroll
            for (int u = 0; u < SPLIT_U; ++u) {
                const int64_t v = v0 + u * stride;
                if (v >= n4) break;
                float4 h, l;
                split1(a[u].x, mode, h.x, l.x);
                split1(a[u].y, mode, h.y, l.y);
                split1(a[u].z, mode, h.z, l.z);
                split1(a[u].w, mode, h.w, l.w);
                if (hi) reinterpret_cast<float4 *>(hi)[v] = h;
                reinterpret_cast<float4 *>(lo)[v] = l;
            }
        }
        for (int64_t e = n4 * 4 + t0; e < n; e += stride) {
            float h, l;
            split1(x[e], mode, h, l);
            if (hi) hi[e] = h;
            lo[e] = l;
        }
    } else {
        for (int64_t e = t0; e < rows * ldp; e += stride) {
            const int64_t r = e / ldp, c = e % ldp;
            float h = 0.f, l = 0.f;
            if (c < cols) split1(x[r * ldx + c], mode, h, l);
            hi[e] = h;
            lo[e] = l;
        }
    }
}

// One launch before the GEMM: blocks [0, nb0) split operand j0, [nb0, nb0 + nb1) operand j1, the
// rest run the tail prepass (C := init_zero ? 0 : beta*C over the k-split tail tiles; rows of
// CG*128 per tile, bn columns) as a grid-stride loop over 4-column groups.  vecC: C and ldc allow
// 16-byte accesses.
__global__ void __launch_bounds__(256) prep_kernel(const SplitJob j0, const SplitJob j1, int nb0, int nb1, int mode,
                                                   const Args p, int rows_per_tile, int bn, int vecC) {
    const int b = (int)blockIdx.x;
    if (b < nb0) {
        split_body(j0, mode, (int64_t)b * blockDim.x + threadIdx.x, (int64_t)nb0 * blockDim.x);
        return;
    }
    if (b < nb0 + nb1) {
        split_body(j1, mode, (int64_t)(b - nb0) * blockDim.x + threadIdx.x, (int64_t)nb1 * blockDim.x);
        return;
    }
    const int npb = (int)gridDim.x - nb0 - nb1, g4 = (bn + 3) / 4;
    const int64_t total = (int64_t)(p.T - p.nfull) * rows_per_tile * g4;
    for (int64_t e = (int64_t)(b - nb0 - nb1) * blockDim.x + threadIdx.x; e < total; e += (int64_t)npb * blockDim.x) {
        const int64_t rowid = e / g4;
        const int x = (int)(e % g4);
        const int t = p.nfull + (int)(rowid / rows_per_tile), r = (int)(rowid % rows_per_tile);
        int pi, tj;
        tile_coords(t, p.PI, p.TJ, pi, tj);
        const int64_t i = (int64_t)pi * rows_per_tile + r, j = (int64_t)tj * bn + 4 * x;
        if (i >= p.M || j >= p.N) continue;
        float *c = p.C + i * p.ldc + j;
        if (vecC && j + 3 < p.N) {
            float4 v = *reinterpret_cast<float4 *>(c);
            v = p.init_zero ? make_float4(0.f, 0.f, 0.f, 0.f)
                            : make_float4(p.beta * v.x, p.beta * v.y, p.beta * v.z, p.beta * v.w);
            *reinterpret_cast<float4 *>(c) = v;
        } else {
            for (int q = 0; q < 4 && j + q < p.N; q++) c[q] = p.init_zero ? 0.f : p.beta * c[q];
        }
    }
}

// ------------------------------------------------------------------ host side
}  // namespace tcm

// The operand split jobs of one GEMM (j1.x == nullptr when B's split serves A too) and their
// block counts in the fused prep launch.
struct Prep {
    tcm::SplitJob j0{}, j1{};
    int nb0 = 0, nb1 = 0, mode = 1;
};

// CTA pairs whenever each CTA's half of the B tile is whole swizzle atoms (EATSS_TCM_PAIR=0 disables)
static int tcm_cg(const ContractNest &n, int bn) {
    static const int env = getenv("EATSS_TCM_PAIR") ? atoi(getenv("EATSS_TCM_PAIR")) : 1;
    if (!env) return 1;
    return n.transB ? ((bn / 2) % 8 == 0 ? 2 : 1) : ((bn / 2) % 32 == 0 ? 2 : 1);
}
static int tcm_stage_bytes(int bn, int cg) { return 2 * tcm::BM * tcm::BK * 4 + 2 * tcm::BK * (bn / cg) * 4; }
static int tcm_stages(int bn, int cg) {
    static const int env = getenv("EATSS_TCM_STAGES") ? atoi(getenv("EATSS_TCM_STAGES")) : 0;  // development
    const int S = env > 0 ? env : (int)((232448 - 2048) / tcm_stage_bytes(bn, cg));
    return std::max(2, std::min(S, 8));
}

bool tcm_applicable(const ContractNest &n, const ContractPlan &p) {
    if (n.f64) return false;
    if (p.Ti != tcm::BM || p.Tj < 32 || p.Tj > 256 || (p.Tj % 32) != 0) return false;
    if (n.M > INT32_MAX / 2 || n.N > INT32_MAX / 2 || n.K > INT32_MAX / 2) return false;
    return 2 * tcm_stage_bytes((int)p.Tj, 1) + 2048 <= 232448 && tcm::encode_fn() != nullptr;
}

// Persistent schedule: full tiles in waves of ncl clusters, the last partial wave split along k
// into sp parts (so idle clusters take k-slices instead of waiting).  nsm / CG clusters of one
// CTA per SM (shared memory admits one); the CTA-pair count is capped by the occupancy query.
static void schedule(tcm::Args &a, int ncl) {
    a.T = a.PI * a.TJ;
    ncl = std::max(1, std::min(ncl, a.T));
    const int rem = a.T % ncl;
    a.sp = 1;
    a.nfull = a.T;
    static const bool splitk = !(getenv("EATSS_TCM_SPLITK") && atoi(getenv("EATSS_TCM_SPLITK")) == 0);
    if (rem > 0 && splitk) {
        const int sp = std::min(std::min(4, ncl / rem), a.nkb);
        if (sp >= 2) {
            a.sp = sp;
            a.nfull = a.T - rem;
        }
    }
    a.nunits = a.nfull + (a.T - a.nfull) * a.sp;
}
static bool needs_prepass(const tcm::Args &a) { return a.sp > 1 && (a.init_zero || a.beta != 1.f); }

// per (kernel, device): the dynamic-smem attribute already set and the CTA-pair occupancy, so
// repeated launches do not pay for cudaFuncSetAttribute / the occupancy query on the host
namespace {
struct KernelState {
    int smem = -1;
    int active = 0;
};
std::mutex g_ks_mu;
std::map<std::pair<const void *, int>, KernelState> g_ks;
}  // namespace

template <int BN, bool TB, int CG>
static cudaError_t launch_one(const CUtensorMap *m, tcm::Args a, int smem, int nsm, const Prep &pr, cudaStream_t s,
                              cudaEvent_t *ev) {
    auto k = tcm::tc_mma_kernel<BN, TB, CG>;
    int dev = 0;
    cudaGetDevice(&dev);
    int ncl = nsm / CG;
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = CG;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.blockDim = dim3(tcm::NTHREADS);
    cfg.dynamicSmemBytes = (size_t)smem;
    cfg.stream = s;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e;
    {  // attribute and occupancy state of (kernel, device): checked and set under the lock
        std::lock_guard<std::mutex> lk(g_ks_mu);
        KernelState &ks = g_ks[{reinterpret_cast<const void *>(k), dev}];
        const bool fresh = ks.smem < smem;
        if (fresh) {
            if ((e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
            ks.smem = smem;
        }
        if (CG == 2 && (fresh || ks.active <= 0)) {
            cfg.gridDim = dim3((unsigned)(2 * ncl));
            int active = 0;
            if (cudaOccupancyMaxActiveClusters(&active, k, &cfg) != cudaSuccess) active = 0;
            cudaGetLastError();
            ks.active = active;
        }
        if (CG == 2 && ks.active > 0) ncl = std::min(ncl, ks.active);
    }
    schedule(a, ncl);
    ncl = std::max(1, std::min(ncl, a.T));
    {  // operand splits + tail prepass: one launch
        const int rows = CG * tcm::BM;
        const int64_t tail4 = needs_prepass(a) ? (int64_t)(a.T - a.nfull) * rows * ((BN + 3) / 4) : 0;
        const int npb = (int)std::min<int64_t>((tail4 + 255) / 256, (int64_t)nsm * 4);
        const int vecC = (a.ldc % 4 == 0 && (reinterpret_cast<uintptr_t>(a.C) & 15) == 0) ? 1 : 0;
        tcm::prep_kernel<<<pr.nb0 + pr.nb1 + npb, 256, 0, s>>>(pr.j0, pr.j1, pr.nb0, pr.nb1, pr.mode, a, rows, BN, vecC);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    cfg.gridDim = dim3((unsigned)(CG * ncl));
    if (ev) cudaEventRecord(ev[0], s);
    e = cudaLaunchKernelEx(&cfg, k, m[0], m[1], m[2], m[3], a);
    if (ev) cudaEventRecord(ev[1], s);
    return e;
}

template <bool TB, int CG>
static cudaError_t launch_bn(int bn, const CUtensorMap *m, const tcm::Args &a, int smem, int nsm, const Prep &pr,
                             cudaStream_t s, cudaEvent_t *ev) {
    switch (bn) {
        case 32: return launch_one<32, TB, CG>(m, a, smem, nsm, pr, s, ev);
        case 64: return launch_one<64, TB, CG>(m, a, smem, nsm, pr, s, ev);
        case 96: return launch_one<96, TB, CG>(m, a, smem, nsm, pr, s, ev);
        case 128: return launch_one<128, TB, CG>(m, a, smem, nsm, pr, s, ev);
        case 160: return launch_one<160, TB, CG>(m, a, smem, nsm, pr, s, ev);
        case 192: return launch_one<192, TB, CG>(m, a, smem, nsm, pr, s, ev);
        case 224: return launch_one<224, TB, CG>(m, a, smem, nsm, pr, s, ev);
        case 256: return launch_one<256, TB, CG>(m, a, smem, nsm, pr, s, ev);
        default: return cudaErrorNotSupported;
    }
}

namespace {
struct Operand {
    const float *x;  // source, rows x cols at pitch ld
    int64_t rows, cols, ld;
    const float *hi = nullptr, *lo = nullptr;  // split halves handed to TMA
    int64_t ldp = 0;
    bool raw_hi = false;  // hi is the source itself (mode 1, aligned)
    int64_t need = 0;     // workspace elements
};
int split_mode() {
    static const int m = [] {
        const char *e = getenv("EATSS_TCM_SPLIT");
        return e && std::string(e) == "rna" ? 0 : 1;
    }();
    return m;
}
void size_operand(Operand &o, int mode) {
    const bool aligned = (o.ld % 4) == 0 && (reinterpret_cast<uintptr_t>(o.x) & 15) == 0;
    o.ldp = aligned ? o.ld : (o.cols + 3) / 4 * 4;
    o.raw_hi = aligned && mode == 1;
    const int64_t span = aligned ? (o.rows - 1) * o.ld + o.cols : o.rows * o.ldp;
    o.need = (o.raw_hi ? 1 : 2) * ((span + 3) / 4 * 4);
}
tcm::SplitJob split_job(Operand &o, float *ws) {  // the split is run by the fused prep launch
    const int64_t span = o.need / (o.raw_hi ? 1 : 2);
    float *lo = ws, *hi = o.raw_hi ? nullptr : ws + span;
    o.lo = lo;
    o.hi = o.raw_hi ? o.x : hi;
    return tcm::SplitJob{o.x, o.ld, o.rows, o.cols, hi, lo, o.ldp};
}
}  // namespace

// The split operands of one GEMM (workspace sizing shared by tcm_ws_floats and the launcher).
struct Operands {
    Operand oa, ob;
    bool share = false;  // syrk: A is a row block of B (both row-major over k): B's split serves A
};
static Operands operands(const ContractNest &n, int mode) {
    const float *A = static_cast<const float *>(n.A), *B = static_cast<const float *>(n.B);
    Operands o{Operand{A, n.M, n.K, n.lda}, Operand{B, n.transB ? n.N : n.K, n.transB ? n.K : n.N, n.ldb}};
    size_operand(o.oa, mode);
    size_operand(o.ob, mode);
    o.share = n.transB && n.lda == n.ldb && A >= B && (A - B) % n.ldb == 0 && (A - B) / n.ldb + n.M <= o.ob.rows;
    return o;
}

size_t tcm_ws_floats(const ContractNest &n, const ContractPlan &) {
    const Operands o = operands(n, split_mode());
    return (size_t)(o.ob.need + (o.share ? 0 : o.oa.need) + 64);
}

cudaError_t launch_tcm_contraction(const ContractNest &n, const ContractPlan &p, float *ws, size_t ws_floats,
                                   cudaStream_t s, cudaEvent_t *ev) {
    if (!tcm_applicable(n, p)) return cudaErrorNotSupported;
    const int bn = (int)p.Tj, cg = tcm_cg(n, bn), mode = split_mode();
    const float *A = static_cast<const float *>(n.A), *B = static_cast<const float *>(n.B);
    Operands ops = operands(n, mode);
    Operand &oa = ops.oa, &ob = ops.ob;
    const bool share = ops.share;
    if (!ws || ws_floats < (size_t)(ob.need + (share ? 0 : oa.need) + 64)) return cudaErrorInvalidValue;
    Prep pr;
    pr.mode = mode;
    pr.j0 = split_job(ob, ws);
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    const int kSplitBlocks = nsm * 8;  // grid-stride split blocks over both operands
    if (share) {
        const int64_t r = (A - B) / n.ldb;
        oa.hi = ob.hi + r * ob.ldp;
        oa.lo = ob.lo + r * ob.ldp;
        oa.ldp = ob.ldp;
        pr.nb0 = kSplitBlocks;
    } else {
        pr.j1 = split_job(oa, ws + ob.need);
        pr.nb0 = std::max(1, std::min(kSplitBlocks - 1, (int)((double)kSplitBlocks * ob.need / (ob.need + oa.need))));
        pr.nb1 = kSplitBlocks - pr.nb0;
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    CUtensorMap m[4];
    const CUtensorMapSwizzle swK = CU_TENSOR_MAP_SWIZZLE_128B, swMN = CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
    bool ok = tcm::make_map(&m[0], oa.hi, n.M, n.K, oa.ldp, tcm::BK, tcm::BM, swK) &&
              tcm::make_map(&m[1], oa.lo, n.M, n.K, oa.ldp, tcm::BK, tcm::BM, swK);
    if (n.transB)  // B(k, j) = B[j*ldb + k]: rows j, K-major boxes of bn/cg rows x 32 k
        ok = ok && tcm::make_map(&m[2], ob.hi, n.N, n.K, ob.ldp, tcm::BK, bn / cg, swK) &&
             tcm::make_map(&m[3], ob.lo, n.N, n.K, ob.ldp, tcm::BK, bn / cg, swK);
    else  // B(k, j) = B[k*ldb + j]: MN-major boxes of 32 k x 32 j
        ok = ok && tcm::make_map(&m[2], ob.hi, n.K, n.N, ob.ldp, 32, tcm::BK, swMN) &&
             tcm::make_map(&m[3], ob.lo, n.K, n.N, ob.ldp, 32, tcm::BK, swMN);
    if (!ok) return cudaErrorInvalidValue;
    tcm::Args a;
    a.M = n.M; a.N = n.N; a.K = n.K;
    a.C = static_cast<float *>(n.C); a.ldc = n.ldc;
    a.alpha = (float)n.alpha; a.beta = (float)n.beta; a.init_zero = n.init_zero ? 1 : 0;
    a.S = tcm_stages(bn, cg);
    static const int chunk_env = getenv("EATSS_TCM_CHUNK") ? atoi(getenv("EATSS_TCM_CHUNK")) : 0;  // development
    a.R = chunk_env > 0 ? chunk_env : 16;  // 16 k-blocks = 512 k per accumulator chunk
    a.nkb = (int)((n.K + tcm::BK - 1) / tcm::BK);
    a.PI = (int)((n.M + cg * tcm::BM - 1) / (cg * tcm::BM));
    a.TJ = (int)((n.N + bn - 1) / bn);
    const int smem = a.S * tcm_stage_bytes(bn, cg) + 1024 /*align*/ + 8 * (2 * a.S + 4) + 16;
    if (n.transB)
        return cg == 2 ? launch_bn<true, 2>(bn, m, a, smem, nsm, pr, s, ev) : launch_bn<true, 1>(bn, m, a, smem, nsm, pr, s, ev);
    return cg == 2 ? launch_bn<false, 2>(bn, m, a, smem, nsm, pr, s, ev) : launch_bn<false, 1>(bn, m, a, smem, nsm, pr, s, ev);
}

int tcm_launches(const ContractNest &, const ContractPlan &) {
    return 2;  // the fused prep launch (splits + tail prepass) and the GEMM
}

}  // namespace eatss
