// tc_mma.cu -- tcgen05 3xTF32 GEMM for MMA-legal tiles (the "tensor-core
// EATSS mode", DESIGN.md §2.5 / §4.1c).  The tile vector (Ti, Tj, Tk) is honoured as written:
//   Ti in {128, 256}  rows of i per cluster tile: 128 = one CTA (UMMA M = 128, cta_group::1),
//                     256 = a CTA pair (cta_group::2, cluster of 2 along i: M = 256, each CTA keeps
//                     its own 128 x Tj accumulator but stages only half of the B tile);
//   Tj in 16..256, multiple of 16: UMMA N (columns of j per tile);
//   Tk in {8, 16, 32, 64}: k per pipeline stage (one TMA box per operand and stage; 8 / 16 k are
//                     one 32 / 64-byte swizzle row, 32 one 128-byte atom, 64 two atoms).
//
// Same loop-nest semantics as the SIMT executor (Fig. 4: each cluster owns one Ti x Tj
// tile of C, k sequential); fp32-accurate via 3xTF32 (reading Q26):
//   C = beta*C + alpha * sum_k (Ahi*Bhi + Ahi*Blo + Alo*Bhi),
//   hi = the fp32 operand itself (the tensor core reads its tf32 bits), lo = rna_tf32(x - rz_tf32(x))
//   materialised once per operand by prep_kernel.
// The tensor core's own fp32 accumulation truncates, so the accumulator is drained into fp32
// registers every CHUNK_K = 128 k (two TMEM buffers alternate; a drain overlaps the next chunk's
// MMAs): 1.2e-6 normwise at N = 4000 (16 chunks of 512 k: 4.0e-6; one chunk: 2.8e-5;
// profiles/r02/chunk_ab*.jsonl) -- chained products (3mm) need the fp32-level error.
//
// B200-specific structure (what differs from the paper's one-tile-per-block CUDA code):
//  * persistent clusters over a grouped (L2-friendly) tile order; one CTA per SM;
//  * wave-quantisation tail: when the last wave would leave clusters idle, the remaining tiles
//    are split along k into `sp` parts whose partial sums are added to C with fp32 atomics
//    (C pre-scaled by beta once by prep_kernel).
// Pipeline (warp-specialised, mbarrier hand-off):
//   warp 0  TMA producer: Ahi/Alo (K-major, 128 x Tk, swizzled) and Bhi/Blo (MN-major boxes of
//           32 columns x Tk rows, SWIZZLE_128B_ATOM_32B -- UMMA SWIZZLE_128B_BASE32B -- or K-major
//           Tj/CG x Tk when B is transposed, as in syrk) into an S-stage ring;
//   warp 1  MMA issuer (leader CTA only): per 8-k step three kind::tf32 MMAs;
//           tcgen05.commit (multicast to the pair) frees ring slots / publishes chunks;
//   warp 2  TMEM allocation (512 columns = two accumulator buffers of up to 256);
//   warps 4..19 epilogue: tcgen05.ld of each finished chunk into fp32 registers, then C (16 warps:
//           a drain of Tj/4 columns per warp keeps short chunks cheap).
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <mutex>
#include <string>

#include "contract.cuh"
#include "devsw.hpp"
#include "tc_ptx.cuh"

namespace eatss {
namespace tcm {

constexpr int BM = 128;      // rows of i per CTA (UMMA M per SM)
#ifndef EATSS_TCM_NEPI
#define EATSS_TCM_NEPI 12
#endif
// epilogue warps (4 .. 3+NEPI): NEPI/4 per TMEM lane quarter, each a contiguous column range of the tile.
// 12 (16 warps in all, four per SM sub-partition) leaves 128 registers per thread for up to 88 fp32
// accumulators; 16 (20 warps) caps every thread at 96 and spills accumulators around the drains.
constexpr int NEPI = EATSS_TCM_NEPI;
constexpr int NEPQ = NEPI / 4;   // epilogue warps per lane quarter
constexpr int NTHREADS = (4 + NEPI) * 32;
constexpr int MAXBN = 256;   // UMMA N limit
constexpr int CHUNK_K = 128; // k per accumulator chunk (fp32 drain of the truncating accumulation), 3xTF32
constexpr int CHUNK_K_F16 = 256;  // 3xFP16: K = 16 per MMA, half the truncating accumulations per k

struct Args {
    int64_t M, N, K;
    float *__restrict__ C;
    int64_t ldc;
    float alpha, beta;
    int init_zero;
    int S;        // ring stages
    int R;        // k-blocks per accumulator chunk
    int BNT;      // Tj: UMMA N of the cluster tile (multiple of 16, <= 256)
    int BNH;      // B columns (rows, if K-major) staged by one CTA: BNT / CG
    int bgroups;  // MN-major B: 32-column swizzle atoms per CTA and stage
    int b_bytes;  // bytes of one B half (hi or lo) per CTA and stage
    int stage;    // bytes per stage (per CTA)
    uint32_t idesc;
    // persistent schedule
    int PI, TJ;   // row groups (of CG*128 rows) x column tiles
    int T;        // PI * TJ tiles
    int nfull;    // tiles done whole by one cluster
    int sp;       // k-parts per tail tile (1 = no split)
    int nunits;   // nfull + (T - nfull) * sp
    int nkb;      // k-blocks of Tk
    int group_rows;  // tile-order grouping (row groups per group) for L2 reuse
    const int *__restrict__ rexp;  // 3xFP16 engine: power-of-two exponent of each row of A (scale 2^rexp)
    const int *__restrict__ cexp;  // ... of each column of B
    unsigned long long *prof;  // development (EATSS_TCM_PROF): per-site cycle counters, else nullptr
    int dbg;  // -DEATSS_DEVTOOLS builds only (EATSS_TCM_DBG; results then wrong): 1 no TMEM drain,
              // 4 no accumulator reset at chunk starts, 16 no MMAs, 32 no operand TMA loads, 8 no
              // wait for the drained buffer at chunk starts inside a tile (only at tile starts)
};

__host__ __device__ inline void tile_coords(int t, int PI, int TJ, int G, int &pi, int &tj) {
    const int g = t / (G * TJ), r = t % (G * TJ);
    const int rows = PI - g * G < G ? PI - g * G : G;
    pi = g * G + r % rows;
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
    tile_coords(t, p.PI, p.TJ, p.group_rows, w.pi, w.tj);
    return w;
}

// K-major operand rows of BKB bytes per stage (fp32: 4*Tk, fp16: 2*Tk; TMA box inner = min(BKB, 128) bytes):
// swizzle span, UMMA layout type, and the descriptor of the 32-byte k step ks (one MMA: 8 tf32 / 16 fp16 k);
// 128-byte atoms along k are rows*128 bytes apart
template <int BKB>
struct KMajor {
    static constexpr int SW = BKB >= 128 ? 128 : BKB;                     // bytes per swizzled row
    static constexpr uint32_t LAYOUT = SW == 128 ? 2u : SW == 64 ? 4u : 6u;  // SW128 / SW64 / SW32
    static constexpr int NA = BKB > 128 ? BKB / 128 : 1;                  // 128-byte atoms along k
    __device__ static uint64_t desc(const unsigned char *base, int rows, int ks) {
        const unsigned char *p = base + (ks / 4) * rows * 128 + (ks % 4) * 32;
        return desc_sw128(p, 16u, (uint32_t)(8 * SW), LAYOUT);
    }
};

// programmatic dependent launch (the launches of one GEMM are chained with it)
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;\n" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory"); }
// BKB: bytes of k per operand row and stage; F16: 3xFP16 operands (K-major A and B, per-row / per-column
// power-of-two scales undone in the epilogue), else 3xTF32
template <int BKB, bool TB, int CG, bool F16>
__global__ void __launch_bounds__(NTHREADS, 1)
    tc_mma_kernel(const __grid_constant__ CUtensorMap mAhi, const __grid_constant__ CUtensorMap mAlo,
                  const __grid_constant__ CUtensorMap mBhi, const __grid_constant__ CUtensorMap mBlo, const Args p) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char *smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);  // stays a shared pointer
    using KA = KMajor<BKB>;
    constexpr int ESZ = F16 ? 2 : 4;      // operand element bytes
    constexpr int BK = BKB / ESZ;         // k per stage (elements)
    constexpr int KA_E = 128 / ESZ;       // k per 128-byte atom (elements)
    static_assert(!F16 || TB, "the 3xFP16 engine stages B K-major (transposed by its prep pass)");
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const uint32_t rank = CG == 2 ? cta_rank() : 0u;
    const int cid = (int)blockIdx.x / CG, ncl = (int)gridDim.x / CG;
    constexpr int A_BYTES = BM * BKB;  // one A half (hi or lo) per stage
    const int BNH = p.BNH, B_BYTES = p.b_bytes, STAGE = p.stage;
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
    // programmatic dependent launch: the prologue above overlapped the split launch's tail; operands,
    // exponents and the pre-scaled C are read only after it has completed (a no-op without the attribute)
    pdl_wait();

    if (warp == 0) {
        if (lane == 0) {  // ---------------------------------------------- TMA producer
            const uint32_t fbar0 = CG == 2 ? mapa(su32(full), 0) : su32(full);
            int it = 0;
            for (int u = cid; u < p.nunits; u += ncl) {
                const Unit w = unit_of(p, u);
                const int i0 = (w.pi * CG + (int)rank) * BM;
                const int jb = w.tj * p.BNT + (int)rank * BNH;
                for (int kb = w.kb0; kb < w.kb1; kb++, it++) {
                    const int s = it % p.S;
                    if (it >= p.S) mbar_wait(empty + s, (unsigned)(((it / p.S) - 1) & 1));
                    unsigned char *st = smem + (size_t)s * STAGE;
                    if (p.dbg & 32) {  // development: no operand loads (MMA-only cost isolation)
                        if (rank == 0) mbar_arrive(full + s);
                        continue;
                    }
                    if (rank == 0) mbar_expect_tx(full + s, CG * STAGE);
                    const uint32_t fb = fbar0 + 8u * (uint32_t)s;
                    const int k0 = kb * BK;
#pragma unroll
                    for (int a = 0; a < KA::NA; a++) {
                        tma_2d<CG>(st + a * BM * 128, &mAhi, k0 + KA_E * a, i0, fb);
                        tma_2d<CG>(st + A_BYTES + a * BM * 128, &mAlo, k0 + KA_E * a, i0, fb);
                    }
                    unsigned char *sb = st + 2 * A_BYTES;
                    if constexpr (TB) {
#pragma unroll
                        for (int a = 0; a < KA::NA; a++) {
                            tma_2d<CG>(sb + a * BNH * 128, &mBhi, k0 + KA_E * a, jb, fb);
                            tma_2d<CG>(sb + B_BYTES + a * BNH * 128, &mBlo, k0 + KA_E * a, jb, fb);
                        }
                    } else {
                        for (int g = 0; g < p.bgroups; g++) {
                            tma_2d<CG>(sb + g * (BK * 128), &mBhi, jb + 32 * g, k0, fb);
                            tma_2d<CG>(sb + B_BYTES + g * (BK * 128), &mBlo, jb + 32 * g, k0, fb);
                        }
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0 && rank == 0) {  // -------------------------------- MMA issuer (leader)
            const uint32_t ID = p.idesc;
            // K-major operands: swizzled rows (SBO = 8 rows), atoms of 32 k; MN-major B: SW128_BASE32B,
            // LBO = stride of 32-column groups (Tk rows x 128 B), SBO = 512 B, +1 KB per 8-k step.
            int it = 0, gc = 0;
            for (int u = cid; u < p.nunits; u += ncl) {
                const Unit w = unit_of(p, u);
                const int nk = w.kb1 - w.kb0;
                for (int x = 0; x < nk; x++, it++) {
                    const int s = it % p.S, bd = gc & 1;
                    const bool first = (p.dbg & 4) ? x == 0 : (x % R) == 0;
                    const long long t0 = p.prof ? clock64() : 0;
                    if (first && gc >= 2 && !((p.dbg & 8) && x > 0)) mbar_wait_cluster(dempty + bd, (unsigned)(((gc - 2) >> 1) & 1));
                    const long long t1 = p.prof ? clock64() : 0;
                    mbar_wait(full + s, (unsigned)((it / p.S) & 1));
                    if (p.prof) {
                        atomicAdd(p.prof + 0, (unsigned long long)(t1 - t0));
                        atomicAdd(p.prof + 1, (unsigned long long)(clock64() - t1));
                    }
                    fence_after();
                    const unsigned char *st = smem + (size_t)s * STAGE;
                    const unsigned char *sb = st + 2 * A_BYTES;
                    const uint32_t d = tmem + (uint32_t)(bd * 256);
#pragma unroll
                    for (int ks = 0; ks < BKB / 32; ks++) {
                        if (p.dbg & 16) break;  // development: no MMAs (operand-delivery cost isolation)
                        const uint64_t ahi = KA::desc(st, BM, ks);
                        const uint64_t alo = KA::desc(st + A_BYTES, BM, ks);
                        uint64_t bhi, blo;
                        if constexpr (TB) {
                            bhi = KA::desc(sb, BNH, ks);
                            blo = KA::desc(sb + B_BYTES, BNH, ks);
                        } else {
                            bhi = desc_sw128(sb + ks * 1024, (uint32_t)(BK * 128), 512u, 1);
                            blo = desc_sw128(sb + B_BYTES + ks * 1024, (uint32_t)(BK * 128), 512u, 1);
                        }
                        if constexpr (F16) {
                            mma_ss_f16<CG>(d, ahi, bhi, ID, (first && ks == 0) ? 0u : 1u);
                            mma_ss_f16<CG>(d, ahi, blo, ID, 1u);
                            mma_ss_f16<CG>(d, alo, bhi, ID, 1u);
                        } else {
                            mma_ss<CG>(d, ahi, bhi, ID, (first && ks == 0) ? 0u : 1u);
                            mma_ss<CG>(d, ahi, blo, ID, 1u);
                            mma_ss<CG>(d, alo, bhi, ID, 1u);
                        }
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
        const int e = warp - 4, q = warp & 3, cq = e >> 2;  // TMEM lane quarter, column quarter
        // columns per epilogue warp: ceil(Tj / NEPQ) rounded up to 8 (16-byte fp32 runs), the last warp of a
        // quarter takes the rest
        const int CW0 = ((p.BNT + NEPQ - 1) / NEPQ + 7) / 8 * 8;
        const int CW = max(0, min(CW0, p.BNT - cq * CW0));
        constexpr int MAXCW = ((MAXBN + NEPQ - 1) / NEPQ + 7) / 8 * 8;
        const uint32_t demp0 = CG == 2 ? mapa(su32(dempty), 0) : su32(dempty);
        int gc = 0;
        for (int u = cid; u < p.nunits; u += ncl) {
            const Unit w = unit_of(p, u);
            const int nch = (w.kb1 - w.kb0 + R - 1) / R;
            float acc[MAXCW];
#pragma unroll
            for (int c = 0; c < MAXCW; c++) acc[c] = 0.f;
            for (int ch = 0; ch < nch; ch++, gc++) {
                const int bd = gc & 1;
                const long long t0 = p.prof ? clock64() : 0;
                mbar_wait(dfull + bd, (unsigned)((gc >> 1) & 1));
                const long long t1 = p.prof ? clock64() : 0;
                fence_after();
                const uint32_t ta = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(bd * 256 + cq * CW0);
                // drain: four 4-column loads in flight per wait
#pragma unroll
                for (int c0 = 0; c0 < MAXCW; c0 += 16) {
                    if (c0 < CW && !(p.dbg & 1)) {
                        uint32_t v[4][4];
#pragma unroll
                        for (int g = 0; g < 4; g++)
                            if (c0 + 4 * g < CW) tmem_ld4(ta + (uint32_t)(c0 + 4 * g), v[g]);
                        wait_ld();
#pragma unroll
                        for (int g = 0; g < 4; g++)
                            if (c0 + 4 * g < CW) {
#pragma unroll
                                for (int c = 0; c < 4; c++) acc[c0 + 4 * g + c] += __uint_as_float(v[g][c]);
                            }
                    }
                }
                fence_before();
                __syncwarp();
                if (lane == 0) {
                    if constexpr (CG == 2) mbar_arrive_cluster(demp0 + 8u * (uint32_t)bd);
                    else mbar_arrive(dempty + bd);
                    if (p.prof) {
                        atomicAdd(p.prof + 2, (unsigned long long)(t1 - t0));
                        atomicAdd(p.prof + 3, (unsigned long long)(clock64() - t1));
                        atomicAdd(p.prof + 4, 1ull);
                    }
                }
            }
            const long long te = p.prof ? clock64() : 0;
            // C(i, j) for row i = i0 + 32q + lane, columns jb .. jb + CW - 1
            const int64_t i = (int64_t)(w.pi * CG + (int)rank) * BM + q * 32 + lane;
            const int64_t jb = (int64_t)w.tj * p.BNT + cq * CW0;
            if constexpr (F16) {  // undo the power-of-two row / column scales: acc * 2^-(rexp_i + cexp_j), exact
                if (i < p.M && jb < p.N) {
                    const float fr = __int_as_float((127 - p.rexp[i]) << 23);
#pragma unroll
                    for (int c = 0; c < MAXCW; c++)
                        if (c < CW && jb + c < p.N) acc[c] = (acc[c] * fr) * __int_as_float((127 - __ldg(p.cexp + jb + c)) << 23);
                }
            }
            if (i < p.M && jb < p.N) {
                float *crow = p.C + i * p.ldc + jb;
                const bool vec = ((p.ldc & 3) == 0) && (jb + CW <= p.N);
                if (w.split) {  // C already holds beta*C (prep_kernel): add the partial sum
                    if (vec) {
#pragma unroll
                        for (int c = 0; c < MAXCW; c += 4)
                            if (c < CW)
                                atomicAdd(reinterpret_cast<float4 *>(crow + c),
                                          make_float4(p.alpha * acc[c], p.alpha * acc[c + 1], p.alpha * acc[c + 2],
                                                      p.alpha * acc[c + 3]));
                    } else {
#pragma unroll
                        for (int c = 0; c < MAXCW; c++)
                            if (c < CW && jb + c < p.N) atomicAdd(crow + c, p.alpha * acc[c]);
                    }
                } else if (vec) {
                    // four 16-byte loads of C in flight before their stores
#pragma unroll
                    for (int c0 = 0; c0 < MAXCW; c0 += 16) {
                        if (c0 < CW) {
                            float4 o[4];
#pragma unroll
                            for (int g = 0; g < 4; g++)
                                if (c0 + 4 * g < CW)
                                    o[g] = p.init_zero ? make_float4(0.f, 0.f, 0.f, 0.f)
                                                       : *reinterpret_cast<const float4 *>(crow + c0 + 4 * g);
#pragma unroll
                            for (int g = 0; g < 4; g++)
                                if (c0 + 4 * g < CW) {
                                    const int c = c0 + 4 * g;
                                    float4 r = o[g];
                                    if (!p.init_zero) { r.x *= p.beta; r.y *= p.beta; r.z *= p.beta; r.w *= p.beta; }
                                    r.x = fmaf(p.alpha, acc[c], r.x);
                                    r.y = fmaf(p.alpha, acc[c + 1], r.y);
                                    r.z = fmaf(p.alpha, acc[c + 2], r.z);
                                    r.w = fmaf(p.alpha, acc[c + 3], r.w);
                                    *reinterpret_cast<float4 *>(crow + c) = r;
                                }
                        }
                    }
                } else {
#pragma unroll
                    for (int c = 0; c < MAXCW; c++) {
                        if (c < CW && jb + c < p.N) {
                            const float o = p.init_zero ? 0.f : p.beta * crow[c];
                            crow[c] = fmaf(p.alpha, acc[c], o);
                        }
                    }
                }
            }
            if (p.prof && lane == 0) {
                atomicAdd(p.prof + 5, (unsigned long long)(clock64() - te));
                atomicAdd(p.prof + 6, 1ull);
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
        tile_coords(t, p.PI, p.TJ, p.group_rows, pi, tj);
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


// ------------------------------------------------------------------ 3xFP16 operand split
// x = a * 2^-s with a = x * 2^s, s chosen per row (A) / per column (B) so that max|a| lies in [2^14, 2^15):
// hi = rn_f16(a), lo = rn_f16(a - hi) -- a - hi is exact in fp32 -- so hi + lo carries 22 significant
// bits of a (the same as tf32 hi + lo) and fp16's range is never exceeded; the GEMM accumulates
// hi*hi + hi*lo + lo*hi in fp32 and its epilogue multiplies by 2^-(s_i + u_j) (exact).
__device__ __forceinline__ int f16_scale_exp(float m) {
    if (!(m > 0.f)) return 0;
    int e;
    frexpf(m, &e);  // m = f * 2^e, f in [0.5, 1)  ->  m * 2^(15 - e) in [2^14, 2^15)
    return max(-100, min(100, 15 - e));
}
__device__ __forceinline__ void f16_split(float x, float sc, __half &h, __half &l) {
    const float a = x * sc;
    h = __float2half_rn(a);
    l = __float2half_rn(a - __half2float(h));
}
struct F16Rows {  // rows x cols fp32 (pitch ldx) -> hi / lo fp16 [rows][ldp], exps[rows]
    const float *x;
    int64_t rows, cols, ldx, ldp;
    __half *hi, *lo;
    int *exps;
    const unsigned *maxbits;  // row maxima (bit patterns) from f16_max_kernel
};
struct F16Cols {  // K x N fp32 (pitch ldx) -> transposed hi / lo fp16 [N][ldp] (K-major), exps[N]
    const float *x;
    int64_t K, N, ldx, ldp;
    __half *hi, *lo;
    int *exps;
};
// one warp per row: the scaled split with the row's exponent from its maximum (f16_max_kernel); 16-byte
// loads, 8-byte fp16 stores, eight column groups in flight per lane
__device__ void f16_rows_body(const F16Rows &j, int64_t w0, int64_t wstride) {
    const int lane = threadIdx.x & 31;
    const bool v4 = ((j.ldx & 3) == 0) && ((reinterpret_cast<uintptr_t>(j.x) & 15) == 0);
    for (int64_t r = w0; r < j.rows; r += wstride) {
        const float *xr = j.x + r * j.ldx;
        const int s = f16_scale_exp(__uint_as_float(j.maxbits[r]));
        if (lane == 0) j.exps[r] = s;
        const float sc = __int_as_float((127 + s) << 23);
        __half *hr = j.hi + r * j.ldp, *lr = j.lo + r * j.ldp;
        for (int64_t c0 = 4 * lane; c0 < j.ldp; c0 += 4 * 256) {  // groups of 4 columns (ldp % 8 == 0)
            float x[8][4];
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int64_t c = c0 + 128 * u;
                if (v4 && c + 3 < j.cols) {
                    const float4 t = *reinterpret_cast<const float4 *>(xr + c);
                    x[u][0] = t.x; x[u][1] = t.y; x[u][2] = t.z; x[u][3] = t.w;
                } else {
#pragma unroll
                    for (int q = 0; q < 4; q++) x[u][q] = c + q < j.cols ? xr[c + q] : 0.f;
                }
            }
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int64_t c = c0 + 128 * u;
                if (c >= j.ldp) break;
                __half h[4], l[4];
#pragma unroll
                for (int q = 0; q < 4; q++) f16_split(x[u][q], sc, h[q], l[q]);
                *reinterpret_cast<uint2 *>(hr + c) =
                    make_uint2(*reinterpret_cast<uint32_t *>(&h[0]), *reinterpret_cast<uint32_t *>(&h[2]));
                *reinterpret_cast<uint2 *>(lr + c) =
                    make_uint2(*reinterpret_cast<uint32_t *>(&l[0]), *reinterpret_cast<uint32_t *>(&l[2]));
            }
        }
    }
}
// row maxima of up to two row operands: CTA (4 rows per warp, 1024-column chunk), a warp per row and chunk, 16-byte
// loads (eight per lane in flight); partial maxima meet via atomicMax on the bit pattern
__device__ void f16_rowmax_block(const F16Rows &j, unsigned *maxbits, int64_t blk) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int64_t nch = (j.cols + 1023) / 1024;
    const int64_t r0 = (blk / nch) * (4 * nw), c0 = (blk % nch) * 1024;
    const bool v4 = ((j.ldx & 3) == 0) && ((reinterpret_cast<uintptr_t>(j.x) & 15) == 0);
    for (int q = 0; q < 4; q++) {
        const int64_t r = r0 + 4 * w + q;
        if (r >= j.rows) break;
        const float *xr = j.x + r * j.ldx;
        float m = 0.f;
        if (v4) {
            float4 v[8];  // all eight loads issued before the first use
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int64_t c = c0 + 4 * (lane + 32 * u);
                v[u] = c + 3 < j.cols ? __ldg(reinterpret_cast<const float4 *>(xr + c)) : make_float4(0.f, 0.f, 0.f, 0.f);
            }
#pragma unroll
            for (int u = 0; u < 8; u++)
                m = fmaxf(m, fmaxf(fmaxf(fabsf(v[u].x), fabsf(v[u].y)), fmaxf(fabsf(v[u].z), fabsf(v[u].w))));
            const int64_t ce = c0 + 1024 < j.cols ? c0 + 1024 : j.cols;  // a ragged last group of < 4 columns
            for (int64_t c = (ce & ~3LL) + lane; c < ce && (ce & 3); c += 32) m = fmaxf(m, fabsf(xr[c]));
        } else {
            for (int64_t c = c0 + lane; c < c0 + 1024 && c < j.cols; c += 32) m = fmaxf(m, fabsf(xr[c]));
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
        if (lane == 0) atomicMax(maxbits + r, __float_as_uint(m));
    }
}
// column maxima of a row-major B (K x N): CTA (128-column strip, 256-row chunk), <= 8 warps -- a thread
// owns four adjacent columns (16-byte loads when aligned), the warps split the chunk, eight loads in
// flight per thread; partial maxima meet in colmax via atomicMax on the bit pattern (non-negative floats
// order like their bits)
__device__ void f16_colmax_block(const float *__restrict__ x, int64_t K, int64_t N, int64_t ldx,
                                 unsigned *__restrict__ colmax, int64_t bx, int64_t by) {
    __shared__ float4 red[8][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int64_t c0 = bx * 128 + 4 * lane, k0 = by * 256;
    const bool v4 = ((ldx & 3) == 0) && ((reinterpret_cast<uintptr_t>(x) & 15) == 0) && c0 + 3 < N;
    float4 m = make_float4(0.f, 0.f, 0.f, 0.f);
    if (c0 < N) {
        for (int i0 = w; i0 < 256; i0 += 8 * nw) {  // eight rows per pass, all loads issued before their use
            float4 v[8];
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int64_t k = k0 + i0 + nw * u;
                const float *row = x + k * ldx + c0;
                if (k >= K) {
                    v[u] = make_float4(0.f, 0.f, 0.f, 0.f);
                } else if (v4) {
                    v[u] = __ldg(reinterpret_cast<const float4 *>(row));
                } else {
                    v[u].x = row[0];
                    v[u].y = c0 + 1 < N ? row[1] : 0.f;
                    v[u].z = c0 + 2 < N ? row[2] : 0.f;
                    v[u].w = c0 + 3 < N ? row[3] : 0.f;
                }
            }
#pragma unroll
            for (int u = 0; u < 8; u++) {
                m.x = fmaxf(m.x, fabsf(v[u].x)); m.y = fmaxf(m.y, fabsf(v[u].y));
                m.z = fmaxf(m.z, fabsf(v[u].z)); m.w = fmaxf(m.w, fabsf(v[u].w));
            }
        }
    }
    red[w][lane] = m;
    __syncthreads();
    if (w == 0 && c0 < N) {
        for (int q = 1; q < nw; q++) {
            const float4 o = red[q][lane];
            m.x = fmaxf(m.x, o.x); m.y = fmaxf(m.y, o.y); m.z = fmaxf(m.z, o.z); m.w = fmaxf(m.w, o.w);
        }
        const float mm[4] = {m.x, m.y, m.z, m.w};
        for (int q = 0; q < 4 && c0 + q < N; q++) atomicMax(colmax + c0 + q, __float_as_uint(mm[q]));
    }
}
// Row operand read ONCE: each warp brings a whole row into its shared buffer with one bulk copy (no thread
// holds the loads: a 16 KB row per warp in flight), takes the maximum from shared memory, then writes the
// scaled split from it -- max and split fused, so the row operand costs one HBM read instead of two.
// Needs 16-byte aligned rows of a multiple of 4 columns (the host checks); `buf` = this warp's row buffer.
__device__ void f16_rows_staged(const F16Rows &j, float *buf, uint64_t *bar, int64_t w0, int64_t wstride) {
    const int lane = threadIdx.x & 31;
    const int c4n = (int)(j.cols >> 2), p4n = (int)(j.ldp >> 2);
    const float4 *b4 = reinterpret_cast<const float4 *>(buf);
    unsigned phase = 0;
    for (int64_t r = w0; r < j.rows; r += wstride) {
        if (lane == 0) {
            fence_proxy_async_smem();  // the previous row's generic reads before the async-proxy overwrite
            mbar_expect_tx(bar, (unsigned)(j.cols * 4));
            bulk_g2s(buf, j.x + r * j.ldx, (unsigned)(j.cols * 4), bar);
        }
        mbar_wait(bar, phase);
        phase ^= 1u;
        float m = 0.f;
        for (int c = lane; c < c4n; c += 32) {
            const float4 v = b4[c];
            m = fmaxf(m, fmaxf(fmaxf(fabsf(v.x), fabsf(v.y)), fmaxf(fabsf(v.z), fabsf(v.w))));
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
        const int s = f16_scale_exp(m);
        if (lane == 0) j.exps[r] = s;
        const float sc = __int_as_float((127 + s) << 23);
        __half *hr = j.hi + r * j.ldp, *lr = j.lo + r * j.ldp;
        for (int c = lane; c < p4n; c += 32) {  // 4 columns per lane and step: 8-byte fp16 stores
            const float4 v = c < c4n ? b4[c] : make_float4(0.f, 0.f, 0.f, 0.f);
            __half h[4], l[4];
            f16_split(v.x, sc, h[0], l[0]);
            f16_split(v.y, sc, h[1], l[1]);
            f16_split(v.z, sc, h[2], l[2]);
            f16_split(v.w, sc, h[3], l[3]);
            *reinterpret_cast<uint2 *>(hr + 4 * c) =
                make_uint2(*reinterpret_cast<uint32_t *>(&h[0]), *reinterpret_cast<uint32_t *>(&h[2]));
            *reinterpret_cast<uint2 *>(lr + 4 * c) =
                make_uint2(*reinterpret_cast<uint32_t *>(&l[0]), *reinterpret_cast<uint32_t *>(&l[2]));
        }
        __syncwarp();
    }
}
// The first launch of the 3xFP16 engine (F16_PASS1_THREADS per block, every block independent):
//   fused = 1: blocks [0, nr0) split the row operands r0 then r1 read once (f16_rows_staged; dynamic shared
//              memory = one row buffer per warp);
//   fused = 0: blocks [0, nr0) row maxima of r0, [nr0, nr0 + nr1) of r1 (the split follows in prep_f16_kernel);
// the rest: the column maxima of a row-major B (cj; colmax).
constexpr int F16_PASS1_THREADS = 128;
__device__ __forceinline__ void f16_max_body(const F16Rows &r0, unsigned *m0, const F16Rows &r1, unsigned *m1,
                                             const F16Cols &cj, unsigned *colmax, int nr0, int nr1, int fused,
                                             int rowbuf_floats) {
    const int64_t b = blockIdx.x;
    if (fused && b < nr0) {
        extern __shared__ __align__(16) float f16_rowbuf[];
        __shared__ __align__(8) uint64_t bars[F16_PASS1_THREADS / 32];
        const int w = threadIdx.x >> 5, nw = blockDim.x >> 5;
        if ((threadIdx.x & 31) == 0) {
            mbar_init(bars + w, 1);
            asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        }
        __syncwarp();
        const int64_t w0 = b * nw + w, ws = (int64_t)nr0 * nw;
        float *buf = f16_rowbuf + (size_t)w * rowbuf_floats;
        if (r0.x) f16_rows_staged(r0, buf, bars + w, w0, ws);
        if (r1.x) f16_rows_staged(r1, buf, bars + w, w0, ws);
        return;
    }
    if (fused) {
        const int64_t c = b - nr0, nsx = (cj.N + 127) / 128;
        f16_colmax_block(cj.x, cj.K, cj.N, cj.ldx, colmax, c % nsx, c / nsx);
        return;
    }
    if (b < nr0) {
        f16_rowmax_block(r0, m0, b);
        return;
    }
    if (b < nr0 + nr1) {
        f16_rowmax_block(r1, m1, b - nr0);
        return;
    }
    const int64_t c = b - nr0 - nr1, nsx = (cj.N + 127) / 128;
    f16_colmax_block(cj.x, cj.K, cj.N, cj.ldx, colmax, c % nsx, c / nsx);
}
// Launch 1 of the 3xFP16 chain.  Each block lets the split launch be scheduled once its own stores are
// issued (programmatic dependent launch); the split launch still waits for this whole grid.
__global__ void __launch_bounds__(F16_PASS1_THREADS) f16_max_kernel(const F16Rows r0, unsigned *m0, const F16Rows r1,
                                                                   unsigned *m1, const F16Cols cj, unsigned *colmax,
                                                                   int nr0, int nr1, int fused, int rowbuf_floats) {
    f16_max_body(r0, m0, r1, m1, cj, colmax, nr0, nr1, fused, rowbuf_floats);
    pdl_trigger();
}
// one 32-column x 128-k tile of a row-major B, no shared memory: lane = column, warp w = k rows
// [16w, 16w + 16) of the tile.  Each of the 16 loads is one coalesced 128-byte row segment across the warp
// (all issued before the first use); the thread then owns 16 consecutive k of its column and writes them
// K-major as two 16-byte stores per half (32 bytes = one sector).  The column exponents come from colmax
// (the k-chunk 0 tile records them).
__device__ void f16_cols_tile(const F16Cols &j, const unsigned *colmax, int64_t tile, int w) {
    const int lane = threadIdx.x & 31;
    const int64_t nstrip = (j.N + 31) / 32;
    const int64_t col = (tile % nstrip) * 32 + lane, k0 = (tile / nstrip) * 128 + 16 * w;
    if (col >= j.N || k0 >= j.ldp) return;
    const int s = f16_scale_exp(__uint_as_float(colmax[col]));
    if (k0 == 0) j.exps[col] = s;
    const float sc = __int_as_float((127 + s) << 23);
    float v[16];
#pragma unroll
    for (int u = 0; u < 16; u++) v[u] = k0 + u < j.K ? __ldg(j.x + (k0 + u) * j.ldx + col) : 0.f;
    __half h[16], l[16];
#pragma unroll
    for (int u = 0; u < 16; u++) f16_split(v[u], sc, h[u], l[u]);
    uint4 *hp = reinterpret_cast<uint4 *>(j.hi + col * j.ldp + k0), *lp = reinterpret_cast<uint4 *>(j.lo + col * j.ldp + k0);
    hp[0] = *reinterpret_cast<const uint4 *>(&h[0]);
    lp[0] = *reinterpret_cast<const uint4 *>(&l[0]);
    if (k0 + 8 < j.ldp) {  // ldp % 8 == 0: the second half exists unless the padded k ends here
        hp[1] = *reinterpret_cast<const uint4 *>(&h[8]);
        lp[1] = *reinterpret_cast<const uint4 *>(&l[8]);
    }
}
// The same 32-column x 128-k tile through shared memory (256 threads): the loads are the coalesced row
// segments of f16_cols_tile, the split halves of each column are parked in shared memory, and every
// column's K-major run (128 k = 256 bytes per half) then leaves as ONE contiguous warp store -- instead of
// 16-byte pieces of 32 different columns per store instruction.
constexpr int F16T_LD = 128 + 8;  // halves per parked column (16-byte pad: 16-byte lane stores stay 4 wavefronts)
__device__ void f16_cols_tile_smem(const F16Cols &j, const unsigned *colmax, int64_t tile, __half *sh, __half *sl) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t nstrip = (j.N + 31) / 32;
    const int64_t c0 = (tile % nstrip) * 32, kt0 = (tile / nstrip) * 128;
    const int64_t col = c0 + lane, k0 = kt0 + 16 * w;
    if (col < j.N && k0 < j.ldp) {
        const int s = f16_scale_exp(__uint_as_float(colmax[col]));
        if (kt0 == 0 && w == 0) j.exps[col] = s;
        const float sc = __int_as_float((127 + s) << 23);
        float v[16];
#pragma unroll
        for (int u = 0; u < 16; u++) v[u] = k0 + u < j.K ? __ldg(j.x + (k0 + u) * j.ldx + col) : 0.f;
        __half h[16], l[16];
#pragma unroll
        for (int u = 0; u < 16; u++) f16_split(v[u], sc, h[u], l[u]);
        uint4 *hp = reinterpret_cast<uint4 *>(sh + lane * F16T_LD + 16 * w);
        uint4 *lp = reinterpret_cast<uint4 *>(sl + lane * F16T_LD + 16 * w);
        hp[0] = *reinterpret_cast<const uint4 *>(&h[0]);
        hp[1] = *reinterpret_cast<const uint4 *>(&h[8]);
        lp[0] = *reinterpret_cast<const uint4 *>(&l[0]);
        lp[1] = *reinterpret_cast<const uint4 *>(&l[8]);
    }
    __syncthreads();
    // warp w writes columns 4w .. 4w+3: lane l the 4 halves at k = kt0 + 4l (ldp % 8 == 0: whole or none)
    const int64_t k = kt0 + 4 * lane;
#pragma unroll
    for (int q = 0; q < 4; q++) {
        const int cl = 4 * w + q;
        const int64_t c = c0 + cl;
        if (c < j.N && k < j.ldp) {
            *reinterpret_cast<uint2 *>(j.hi + c * j.ldp + k) = *reinterpret_cast<const uint2 *>(sh + cl * F16T_LD + 4 * lane);
            *reinterpret_cast<uint2 *>(j.lo + c * j.ldp + k) = *reinterpret_cast<const uint2 *>(sl + cl * F16T_LD + 4 * lane);
        }
    }
    __syncthreads();  // the parked tile may be overwritten by the block's next tile
}
__device__ void tail_prepass_block(const Args &p, int blk, int npb, int rows_per_tile, int bn, int vecC);
// The launch before the 3xFP16 GEMM: blocks [0, nbr) split the row operands (A, and B when it is K-major
// -- syrk), [nbr, nbr + nbc) the 32 x 128 tiles of a row-major B (its column maxima from f16_max_kernel),
// the rest the split-k tail pre-pass.
__device__ __forceinline__ void prep_f16_body(const F16Rows &r0, const F16Rows &r1, const F16Cols &cj,
                                              const unsigned *colmax, int nbr, int nbc, const Args &p,
                                              int rows_per_tile, int bn, int vecC, int parked) {
    const int b = (int)blockIdx.x;
    if (b < nbr) {
        const int64_t wstride = (int64_t)nbr * 8, w0 = (int64_t)b * 8 + (threadIdx.x >> 5);
        if (r0.x) f16_rows_body(r0, w0, wstride);
        if (r1.x) f16_rows_body(r1, w0, wstride);
        return;
    }
    if (b < nbr + nbc) {
        const int64_t ntiles = ((cj.N + 31) / 32) * ((cj.ldp + 127) / 128);
        __shared__ __align__(16) __half park[2][32 * F16T_LD];
        for (int64_t tile = b - nbr; tile < ntiles; tile += nbc) {
            if (parked) f16_cols_tile_smem(cj, colmax, tile, park[0], park[1]);
            else f16_cols_tile(cj, colmax, tile, threadIdx.x >> 5);
        }
        return;
    }
    tail_prepass_block(p, b - nbr - nbc, (int)gridDim.x - nbr - nbc, rows_per_tile, bn, vecC);
}
__global__ void __launch_bounds__(256, 4) prep_f16_kernel(const F16Rows r0, const F16Rows r1, const F16Cols cj,
                                                       const unsigned *colmax, int nbr, int nbc, const Args p,
                                                       int rows_per_tile, int bn, int vecC, int parked) {
    pdl_wait();  // launch 1 complete and visible (column maxima, row splits)
    prep_f16_body(r0, r1, cj, colmax, nbr, nbc, p, rows_per_tile, bn, vecC, parked);
    pdl_trigger();
}
// split-k tail pre-pass: C := init_zero ? 0 : beta*C on the tiles t >= nfull, block `blk` of `npb`
__device__ void tail_prepass_block(const Args &p, int blk, int npb, int rows_per_tile, int bn, int vecC) {
    const int g4 = (bn + 3) / 4;
    const int64_t total = (int64_t)(p.T - p.nfull) * rows_per_tile * g4;
    for (int64_t e = (int64_t)blk * blockDim.x + threadIdx.x; e < total; e += (int64_t)npb * blockDim.x) {
        const int64_t rowid = e / g4;
        const int x = (int)(e % g4);
        const int t = p.nfull + (int)(rowid / rows_per_tile), r = (int)(rowid % rows_per_tile);
        int pi, tj;
        tile_coords(t, p.PI, p.TJ, p.group_rows, pi, tj);
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
    // 3xFP16: row splits (A; B when K-major) and the column strips of a row-major B
    tcm::F16Rows r0{}, r1{};
    tcm::F16Cols cj{};
    unsigned *colmax = nullptr;  // row-major B: per-column max bits (f16_max_kernel before the prep launch)
    unsigned *maxes = nullptr;   // the zero-initialised region holding every max array of this GEMM
    size_t maxes_bytes = 0;
    unsigned *m0 = nullptr, *m1 = nullptr;  // row maxima of r0 / r1
    bool fused_rows = false;  // row operands split in the first launch, each row read once (f16_rows_staged)
    int nbr = 0, nbc = 0;
};

// Geometry of one tile vector on this engine (shared by applicability, workspace and launch).
struct TcmGeom {
    bool ok = false;
    int bk = 0, bn = 0, cg = 1, bnh = 0, bgroups = 0, a_bytes = 0, b_bytes = 0, stage = 0, S = 0, smem = 0;
};
// f16: the 3xFP16 engine (operands 2 bytes, B always K-major after its transposing split)
static TcmGeom tcm_geom(const ContractNest &n, const ContractPlan &p, bool f16 = false) {
    TcmGeom g;
    const int64_t Ti = p.rTi, Tj = p.rTj, Tk = p.rTk;
    if (n.f64 || (Ti != 128 && Ti != 256)) return g;
    if (Tj < 16 || Tj > tcm::MAXBN || Tj % 16) return g;
    const int esz = f16 ? 2 : 4;
    if (Tk * esz != 32 && Tk * esz != 64 && Tk * esz != 128 && Tk * esz != 256) return g;  // bytes per stage row
    if (n.M > INT32_MAX / 2 || n.N > INT32_MAX / 2 || n.K > INT32_MAX / 2) return g;
    const bool kmaj_b = n.transB || f16;
    g.bk = (int)Tk;
    g.bn = (int)Tj;
    g.cg = Ti == 256 ? 2 : 1;           // Ti = 256: a CTA pair (cta_group::2) per tile
    g.bnh = g.bn / g.cg;
    if (g.bnh % (kmaj_b ? 8 : 16)) return g;  // UMMA N per CTA half: K-major rows in 8s, MN-major in 16s
    g.bgroups = (g.bnh + 31) / 32;
    g.a_bytes = tcm::BM * g.bk * esz;
    g.b_bytes = kmaj_b ? g.bnh * g.bk * esz : g.bgroups * 32 * g.bk * esz;
    g.stage = 2 * g.a_bytes + 2 * g.b_bytes;
    static const int env_s = devsw("EATSS_TCM_STAGES", 0);  // development
    g.S = std::min(8, (232448 - 2048) / g.stage);
    if (env_s > 0) g.S = std::min(g.S, env_s);
    if (g.S < 2) return g;
    g.smem = g.S * g.stage + 1024 /*align*/ + 8 * (2 * g.S + 4) + 16;
    g.ok = tcm::encode_fn() != nullptr;
    return g;
}

bool tcm_applicable(const ContractNest &n, const ContractPlan &p, bool f16) { return tcm_geom(n, p, f16).ok; }

// Persistent schedule: full tiles in waves of ncl clusters, the last partial wave split along k
// into sp parts (so idle clusters take k-slices instead of waiting).  nsm / CG clusters of one
// CTA per SM (shared memory admits one); the CTA-pair count is capped by the occupancy query.
static void schedule(tcm::Args &a, int ncl) {
    a.T = a.PI * a.TJ;
    ncl = std::max(1, std::min(ncl, a.T));
    const int rem = a.T % ncl;
    a.sp = 1;
    a.nfull = a.T;
    static const bool splitk = devsw("EATSS_TCM_SPLITK", 1) != 0;
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

template <int BKB, bool TB, int CG, bool F16>
static cudaError_t launch_one(const CUtensorMap *m, tcm::Args a, int smem, int nsm, const Prep &pr, cudaStream_t s,
                              cudaEvent_t *ev) {
    auto k = tcm::tc_mma_kernel<BKB, TB, CG, F16>;
    int dev = 0;
    cudaGetDevice(&dev);
    int ncl = nsm / CG;
    // programmatic dependent launch of the split launch(es) and the GEMM (EATSS_TCM_PDL=0: plain launches);
    // not when the GEMM is bracketed by timing events (exec.time_kernels): the event record between the
    // launches would put the early-launched GEMM's wait inside its own timed window
    static const bool pdl_env = devsw("EATSS_TCM_PDL", 1) != 0;
    const bool pdl = pdl_env && ev == nullptr;
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = CG;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = pdl ? 1 : 0;
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
        const int64_t tail4 = needs_prepass(a) ? (int64_t)(a.T - a.nfull) * rows * ((a.BNT + 3) / 4) : 0;
        const int npb = (int)std::min<int64_t>((tail4 + 255) / 256, (int64_t)nsm * 4);
        const int vecC = (a.ldc % 4 == 0 && (reinterpret_cast<uintptr_t>(a.C) & 15) == 0) ? 1 : 0;
        if constexpr (F16) {
            {  // first launch: the row operands (fused: split, each row read once; else their maxima) and the
               // column maxima of a row-major B
                if ((e = cudaMemsetAsync(pr.maxes, 0, pr.maxes_bytes, s)) != cudaSuccess) return e;
                constexpr int TPB = tcm::F16_PASS1_THREADS, NW = TPB / 32;
                const int ncb = pr.colmax ? (int)(((pr.cj.N + 127) / 128) * ((pr.cj.K + 255) / 256)) : 0;
                int nr0 = 0, nr1 = 0, rowbuf = 0;
                size_t dsm = 0;
                if (pr.fused_rows) {
                    const tcm::F16Rows &rr = pr.r0.x ? pr.r0 : pr.r1;
                    rowbuf = (int)((rr.cols + 3) / 4 * 4);
                    dsm = (size_t)NW * rowbuf * sizeof(float);
                    const int64_t nrows = std::max(pr.r0.x ? pr.r0.rows : 0, pr.r1.x ? pr.r1.rows : 0);
                    nr0 = (int)std::min<int64_t>((nrows + NW - 1) / NW, (int64_t)nsm * 3);
                    auto kf = tcm::f16_max_kernel;
                    std::lock_guard<std::mutex> lk(g_ks_mu);
                    KernelState &ks = g_ks[{reinterpret_cast<const void *>(kf), dev}];
                    if (ks.smem < (int)dsm) {
                        if ((e = cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsm)) !=
                            cudaSuccess)
                            return e;
                        ks.smem = (int)dsm;
                    }
                } else {
                    auto nrb = [](const tcm::F16Rows &r) {
                        return r.x ? (int)(((r.rows + 4 * NW - 1) / (4 * NW)) * ((r.cols + 1023) / 1024)) : 0;
                    };
                    nr0 = nrb(pr.r0);
                    nr1 = nrb(pr.r1);
                }
                tcm::f16_max_kernel<<<nr0 + nr1 + ncb, TPB, dsm, s>>>(pr.r0, pr.m0, pr.r1, pr.m1, pr.cj, pr.colmax,
                                                                      nr0, nr1, pr.fused_rows ? 1 : 0, rowbuf);
                if ((e = cudaGetLastError()) != cudaSuccess) return e;
            }
            const int nbr = pr.fused_rows ? 0 : pr.nbr;  // fused: the rows are already split
            cudaLaunchConfig_t pc = {};
            cudaLaunchAttribute pa[1];
            pa[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            pa[0].val.programmaticStreamSerializationAllowed = pdl ? 1 : 0;
            pc.gridDim = dim3((unsigned)std::max(1, nbr + pr.nbc + npb));
            pc.blockDim = dim3(256);
            pc.stream = s;
            pc.attrs = pa;
            pc.numAttrs = 1;
            e = cudaLaunchKernelEx(&pc, tcm::prep_f16_kernel, pr.r0, pr.r1, pr.cj, (const unsigned *)pr.colmax, nbr,
                                   pr.nbc, (const tcm::Args)a, rows, (int)a.BNT, vecC, devsw("EATSS_TCF_PARKED", 1));
            if (e != cudaSuccess) return e;
        } else {
            tcm::prep_kernel<<<pr.nb0 + pr.nb1 + npb, 256, 0, s>>>(pr.j0, pr.j1, pr.nb0, pr.nb1, pr.mode, a, rows,
                                                                   a.BNT, vecC);
        }
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    cfg.gridDim = dim3((unsigned)(CG * ncl));
    cfg.numAttrs = 2;  // + programmatic serialization (the occupancy query above used the cluster attribute only)
    if (ev) cudaEventRecord(ev[0], s);
    e = cudaLaunchKernelEx(&cfg, k, m[0], m[1], m[2], m[3], a);
    if (ev) cudaEventRecord(ev[1], s);
    return e;
}

template <bool TB, int CG, bool F16>
static cudaError_t launch_bk(int bkb, const CUtensorMap *m, const tcm::Args &a, int smem, int nsm, const Prep &pr,
                             cudaStream_t s, cudaEvent_t *ev) {
    switch (bkb) {  // bytes of k per operand row and stage
        case 32: return launch_one<32, TB, CG, F16>(m, a, smem, nsm, pr, s, ev);
        case 64: return launch_one<64, TB, CG, F16>(m, a, smem, nsm, pr, s, ev);
        case 128: return launch_one<128, TB, CG, F16>(m, a, smem, nsm, pr, s, ev);
        case 256: return launch_one<256, TB, CG, F16>(m, a, smem, nsm, pr, s, ev);
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
        const char *e = getenv("EATSS_TCM_SPLIT");  // development: "rna" = hi = rna_tf32(x) materialised too
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

// development switches of one GEMM launch: EATSS_TCM_DBG (-DEATSS_DEVTOOLS builds only; results then
// wrong) and EATSS_TCM_PROF (wait / drain / epilogue cycle profile, printed after the launch)
static void dev_setup(tcm::Args &a, cudaStream_t s) {
    a.prof = nullptr;
#ifdef EATSS_DEVTOOLS
    a.dbg = devsw("EATSS_TCM_DBG", 0);
#else
    a.dbg = 0;
#endif
    static unsigned long long *prof = nullptr;
    if (devsw("EATSS_TCM_PROF", 0)) {
        if (!prof) cudaMalloc(&prof, 16 * sizeof(unsigned long long));
        cudaMemsetAsync(prof, 0, 16 * sizeof(unsigned long long), s);
        a.prof = prof;
    }
}
static void dev_report(const tcm::Args &a, cudaStream_t s) {
    if (a.prof) {
        unsigned long long h[16];
        cudaMemcpyAsync(h, a.prof, sizeof(h), cudaMemcpyDeviceToHost, s);
        cudaStreamSynchronize(s);
        const double nmma = (double)a.PI * a.TJ * a.nkb;  // k-blocks issued
        fprintf(stderr,
                "tc_mma prof: MMA wait dempty %.0f / wait full %.0f cycles per k-block | EPI wait dfull %.0f / "
                "drain %.0f per chunk-warp (%llu) | C epilogue %.0f per tile-warp (%llu)\n",
                h[0] / nmma, h[1] / nmma, h[2] / (double)h[4], h[3] / (double)h[4], h[4], h[5] / (double)h[6], h[6]);
    }
}

cudaError_t launch_tcm_contraction(const ContractNest &n, const ContractPlan &p, float *ws, size_t ws_floats,
                                   cudaStream_t s, cudaEvent_t *ev) {
    const TcmGeom g = tcm_geom(n, p);
    if (!g.ok) return cudaErrorNotSupported;
    const int bn = g.bn, cg = g.cg, bk = g.bk, mode = split_mode();
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
    // K-major boxes: min(Tk, 32) k (one swizzled row: 32 / 64 / 128 bytes) x rows
    const int kbox = std::min(bk, 32);
    const CUtensorMapSwizzle swK = kbox == 32   ? CU_TENSOR_MAP_SWIZZLE_128B
                                   : kbox == 16 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                : CU_TENSOR_MAP_SWIZZLE_32B;
    const CUtensorMapSwizzle swMN = CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
    bool ok = tcm::make_map(&m[0], oa.hi, n.M, n.K, oa.ldp, kbox, tcm::BM, swK) &&
              tcm::make_map(&m[1], oa.lo, n.M, n.K, oa.ldp, kbox, tcm::BM, swK);
    if (n.transB)  // B(k, j) = B[j*ldb + k]: rows j, K-major boxes of bn/cg rows x kbox k
        ok = ok && tcm::make_map(&m[2], ob.hi, n.N, n.K, ob.ldp, kbox, g.bnh, swK) &&
             tcm::make_map(&m[3], ob.lo, n.N, n.K, ob.ldp, kbox, g.bnh, swK);
    else  // B(k, j) = B[k*ldb + j]: MN-major boxes of Tk k x 32 j
        ok = ok && tcm::make_map(&m[2], ob.hi, n.K, n.N, ob.ldp, 32, bk, swMN) &&
             tcm::make_map(&m[3], ob.lo, n.K, n.N, ob.ldp, 32, bk, swMN);
    if (!ok) return cudaErrorInvalidValue;
    tcm::Args a;
    a.M = n.M; a.N = n.N; a.K = n.K;
    a.C = static_cast<float *>(n.C); a.ldc = n.ldc;
    a.alpha = (float)n.alpha; a.beta = (float)n.beta; a.init_zero = n.init_zero ? 1 : 0;
    a.S = g.S;
    static const int chunk_env = devsw("EATSS_TCM_CHUNK_K", 0);  // development: k per accumulator chunk
    a.R = std::max(1, (chunk_env > 0 ? chunk_env : tcm::CHUNK_K) / bk);
    a.BNT = bn; a.BNH = g.bnh; a.bgroups = g.bgroups; a.b_bytes = g.b_bytes; a.stage = g.stage;
    a.idesc = tcm::idesc(bn, cg, n.transB);
    a.nkb = (int)((n.K + bk - 1) / bk);
    a.PI = (int)((n.M + cg * tcm::BM - 1) / (cg * tcm::BM));
    a.TJ = (int)((n.N + bn - 1) / bn);
    static const int group_env = devsw("EATSS_TCM_GROUP", 8);  // development: row groups per raster group
    a.group_rows = std::max(1, group_env);
    dev_setup(a, s);
    a.rexp = a.cexp = nullptr;
    cudaError_t r;
    const int bkb = 4 * bk;
    if (n.transB)
        r = cg == 2 ? launch_bk<true, 2, false>(bkb, m, a, g.smem, nsm, pr, s, ev)
                    : launch_bk<true, 1, false>(bkb, m, a, g.smem, nsm, pr, s, ev);
    else
        r = cg == 2 ? launch_bk<false, 2, false>(bkb, m, a, g.smem, nsm, pr, s, ev)
                    : launch_bk<false, 1, false>(bkb, m, a, g.smem, nsm, pr, s, ev);
    dev_report(a, s);
    return r;
}

// ------------------------------------------------------------------ 3xFP16 engine (engine = TENSOR_F16)
namespace {
struct F16Layout {  // workspace offsets (bytes, 256-aligned): hi/lo fp16 operands and their exponents
    int64_t Kp = 0;
    size_t a_hi = 0, a_lo = 0, a_exp = 0, b_hi = 0, b_lo = 0, b_exp = 0, b_max = 0, a_max = 0, max_end = 0, total = 0;
    bool share = false;  // syrk: A is a row block of the K-major B
};
F16Layout f16_layout(const ContractNest &n) {
    F16Layout L;
    const float *A = static_cast<const float *>(n.A), *B = static_cast<const float *>(n.B);
    L.Kp = (n.K + 7) / 8 * 8;  // 16-byte fp16 rows (TMA strides)
    L.share = n.transB && n.lda == n.ldb && A >= B && (A - B) % n.ldb == 0 && (A - B) / n.ldb + n.M <= n.N;
    auto al = [](size_t v) { return (v + 255) / 256 * 256; };
    size_t o = 0;
    L.b_hi = o; o = al(o + (size_t)n.N * L.Kp * 2);
    L.b_lo = o; o = al(o + (size_t)n.N * L.Kp * 2);
    L.b_exp = o; o = al(o + (size_t)n.N * 4);
    L.b_max = o; o = o + (size_t)n.N * 4;   // maxima: b_max then a_max, contiguous (one memset)
    L.a_max = o; o = o + (L.share ? 0 : (size_t)n.M * 4);
    L.max_end = o; o = al(o);
    if (!L.share) {
        L.a_hi = o; o = al(o + (size_t)n.M * L.Kp * 2);
        L.a_lo = o; o = al(o + (size_t)n.M * L.Kp * 2);
        L.a_exp = o; o = al(o + (size_t)n.M * 4);
    }
    L.total = o;
    return L;
}
}  // namespace

bool tcf_applicable(const ContractNest &n, const ContractPlan &p) { return tcm_geom(n, p, true).ok; }
size_t tcf_ws_floats(const ContractNest &n, const ContractPlan &) { return f16_layout(n).total / 4 + 64; }

cudaError_t launch_tcf_contraction(const ContractNest &n, const ContractPlan &p, float *ws, size_t ws_floats,
                                   cudaStream_t s, cudaEvent_t *ev) {
    const TcmGeom g = tcm_geom(n, p, true);
    if (!g.ok) return cudaErrorNotSupported;
    const F16Layout L = f16_layout(n);
    if (!ws || ws_floats * 4 < L.total) return cudaErrorInvalidValue;
    char *w = reinterpret_cast<char *>(ws);
    const float *A = static_cast<const float *>(n.A), *B = static_cast<const float *>(n.B);
    __half *bhi = reinterpret_cast<__half *>(w + L.b_hi), *blo = reinterpret_cast<__half *>(w + L.b_lo);
    int *bexp = reinterpret_cast<int *>(w + L.b_exp);
    const __half *ahi, *alo;
    const int *aexp;
    Prep pr;
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    unsigned *bmax = reinterpret_cast<unsigned *>(w + L.b_max), *amax = reinterpret_cast<unsigned *>(w + L.a_max);
    pr.maxes = bmax;
    pr.maxes_bytes = L.max_end - L.b_max;
    if (n.transB) {  // B(k, j) = B[j*ldb + k]: rows j are already K-major -> row split, row scale = column scale
        pr.r0 = tcm::F16Rows{B, n.N, n.K, n.ldb, L.Kp, bhi, blo, bexp, bmax};
        pr.m0 = bmax;
    } else {  // row-major B[k][j]: column strips, transposed to K-major
        pr.cj = tcm::F16Cols{B, n.K, n.N, n.ldb, L.Kp, bhi, blo, bexp};
        pr.colmax = bmax;
        pr.nbc = (int)std::min<int64_t>(((n.N + 31) / 32) * ((L.Kp + 127) / 128), (int64_t)nsm * 8);
    }
    if (L.share) {
        const int64_t r = (A - B) / n.ldb;
        ahi = bhi + r * L.Kp;
        alo = blo + r * L.Kp;
        aexp = bexp + r;
    } else {
        __half *h = reinterpret_cast<__half *>(w + L.a_hi), *l = reinterpret_cast<__half *>(w + L.a_lo);
        int *e = reinterpret_cast<int *>(w + L.a_exp);
        (n.transB ? pr.r1 : pr.r0) = tcm::F16Rows{A, n.M, n.K, n.lda, L.Kp, h, l, e, amax};
        (n.transB ? pr.m1 : pr.m0) = amax;
        ahi = h;
        alo = l;
        aexp = e;
    }
    pr.nbr = nsm * 4;
    {  // the row operands can be read once (bulk-copied rows) when 16-byte aligned, whole float4s, <= 48 KB
        auto ok = [](const tcm::F16Rows &r) {
            return !r.x || ((r.ldx & 3) == 0 && (reinterpret_cast<uintptr_t>(r.x) & 15) == 0 && (r.cols & 3) == 0 &&
                            r.cols * 4 <= 48 * 1024);
        };
        static const bool staged_rows = devsw("EATSS_TCF_STAGED_ROWS", 1) != 0;  // development: 0 = two reads
        pr.fused_rows = staged_rows && ok(pr.r0) && ok(pr.r1) && (pr.r0.x || pr.r1.x);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    CUtensorMap m[4];
    const int bkb = g.bk * 2, kbytes = std::min(bkb, 128), kbox = kbytes / 2;
    const CUtensorMapSwizzle sw = kbytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                  : kbytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                 : CU_TENSOR_MAP_SWIZZLE_32B;
    const bool ok = tcm::make_map(&m[0], ahi, n.M, n.K, L.Kp, kbox, tcm::BM, sw, true) &&
                    tcm::make_map(&m[1], alo, n.M, n.K, L.Kp, kbox, tcm::BM, sw, true) &&
                    tcm::make_map(&m[2], bhi, n.N, n.K, L.Kp, kbox, g.bnh, sw, true) &&
                    tcm::make_map(&m[3], blo, n.N, n.K, L.Kp, kbox, g.bnh, sw, true);
    if (!ok) return cudaErrorInvalidValue;
    tcm::Args a;
    a.M = n.M; a.N = n.N; a.K = n.K;
    a.C = static_cast<float *>(n.C); a.ldc = n.ldc;
    a.alpha = (float)n.alpha; a.beta = (float)n.beta; a.init_zero = n.init_zero ? 1 : 0;
    a.S = g.S;
    static const int chunk_env = devsw("EATSS_TCM_CHUNK_K", 0);  // development: k per accumulator chunk
    a.R = std::max(1, (chunk_env > 0 ? chunk_env : tcm::CHUNK_K_F16) / g.bk);
    a.BNT = g.bn; a.BNH = g.bnh; a.bgroups = g.bgroups; a.b_bytes = g.b_bytes; a.stage = g.stage;
    a.idesc = tcm::idesc_f16(g.bn, g.cg);
    a.nkb = (int)((n.K + g.bk - 1) / g.bk);
    a.PI = (int)((n.M + g.cg * tcm::BM - 1) / (g.cg * tcm::BM));
    a.TJ = (int)((n.N + g.bn - 1) / g.bn);
    static const int group_env = devsw("EATSS_TCM_GROUP", 8);
    a.group_rows = std::max(1, group_env);
    dev_setup(a, s);
    a.rexp = aexp;
    a.cexp = bexp;
    const cudaError_t r = g.cg == 2 ? launch_bk<true, 2, true>(bkb, m, a, g.smem, nsm, pr, s, ev)
                                    : launch_bk<true, 1, true>(bkb, m, a, g.smem, nsm, pr, s, ev);
    dev_report(a, s);
    return r;
}

int tcm_launches(const ContractNest &, const ContractPlan &) {
    return 2;  // the fused prep launch (splits + tail prepass) and the GEMM
}

}  // namespace eatss
