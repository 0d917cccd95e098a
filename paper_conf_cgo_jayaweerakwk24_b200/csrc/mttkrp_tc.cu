// mttkrp_tc.cu -- mttkrp (reading R-N8) on the tensor pipe (tcgen05 3xTF32):
//
//   A[i][j] += sum_k C[k][j] * T[(i,k)][j],   T[(i,k)][j] = sum_l B[i][k][l] * D[l][j]
//
// T is a dense GEMM: M = ni*nk rows (i, k) of B viewed as a row-major matrix Bm[(i,k)][l] (K-major
// A operand, no copy), N = nj (D[l][j] as an MN-major B operand), K = nl.  Tile vector:
// (Ti, Tj, Tk, Tl) = (1, nj, 128, 32): one UMMA M = 128 block is one i and 128 consecutive k, the
// whole rank as N, l in 32-float TMA atoms -- the MMA-legal point of the mttkrp tile space (the
// analogue of reading T for this nest; the SIMT executor takes any tile).
//
// B is the only large operand (ni*nk*nl floats, 512 MiB at the config) and is read exactly once:
// its tf32 lo half is NOT materialised in HBM (that would triple the traffic) -- converter warps
// form it in shared memory from the TMA-landed tile (same swizzled layout, elementwise), as
//   hi = B itself (the tensor core truncates fp32 to tf32), lo = rna_tf32(B - rz_tf32(B)),
// and D's lo half (64 KB) is formed once per call.  3xTF32: T = Bhi*Dhi + Bhi*Dlo + Blo*Dhi, issued as
// two MMAs per 8-k step -- Bhi x [Dhi | Dlo] (N = 2 NJ) and Blo x Dhi (N = NJ) -- because the small-N
// MMAs are bound by their per-instruction cost (measured: 12 -> 8 MMAs per stage).
// Epilogue: a thread per TMEM lane (= one (i, k) row) scales its N accumulators by C[k][:], the
// 128 rows are reduced across lanes (shuffle reduce-scatter) and warps (shared memory, fixed
// order) and written as one partial row per block; a second kernel adds the nk/128 partials of
// each i to A in block order (deterministic bits).
// Warp roles (persistent, one CTA per SM): warp 0 TMA producer (ring stage: B hi tile + D hi/lo,
// plus the stage's B lo tile), warp 1 MMA issuer, warp 2 TMEM, warps 4-7 lo converters, warps 8-11
// epilogue.  Measured alternatives that were slower: a separate 2- or 4-slot lo ring with a deeper
// TMA ring (0.196 ms vs 0.171), an L2 bulk prefetch of the next block's rows (re-reads from DRAM).
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include "tc_ptx.cuh"

namespace eatss {
namespace mttc {

using namespace tcm;

constexpr int BM = 128, BK = 32;
constexpr int NCONV = 4, NEPI = 4;
constexpr int NTHREADS = (4 + NCONV + NEPI) * 32;
constexpr int SMAX = 4;  // ring stages (measured: 4 beats 5: 0.171 vs 0.189 ms)

struct Args {
    int64_t ni, nj, nk, nl;
    int nblk;   // ni * nk / 128 row blocks
    int nkb;    // nl / 32
    int S;      // ring stages
    int dbg;    // development only (EATSS_MTC_DBG): 1 skip the lo conversion, 2 skip the MMAs
    const float *C;
    float *part;  // [nblk][nj]
};

__device__ __forceinline__ float lo_of(float x) {
    const float hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
    uint32_t lb;
    asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(lb) : "f"(x - hi));
    return __uint_as_float(lb);
}

template <int NJ>
__global__ void __launch_bounds__(NTHREADS, 1)
    mttkrp_tc_kernel(const __grid_constant__ CUtensorMap mB, const __grid_constant__ CUtensorMap mDhi,
                     const __grid_constant__ CUtensorMap mDlo, const Args p) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char *smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    constexpr int A_BYTES = BM * BK * 4;       // 16 KB
    constexpr int D_BYTES = BK * NJ * 4;       // NJ/32 groups of 32 l x 128 B
    constexpr int HSTAGE = 2 * A_BYTES + 2 * D_BYTES;  // ring stage: B hi tile, B lo tile, D hi, D lo
    constexpr uint32_t ID = idesc(NJ, 1, false);       // A_lo x D_hi          (N = NJ)
    constexpr uint32_t ID2 = idesc(2 * NJ, 1, false);  // A_hi x [D_hi | D_lo] (N = 2 NJ: both D tiles are
                                                       // adjacent 32-column groups of one MN-major operand)
    const int SH = p.S;                        // ring depth
    // the lo tile of a stage is rewritten only after the TMA of a later use of that stage landed,
    // which the producer issues only after the MMAs of the earlier use finished
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)SH * HSTAGE);
    uint64_t *empty = full + SH;   // MMAs of the stage done (tcgen05.commit)
    uint64_t *conv = empty + SH;   // lo of the stage written (NCONV warps arrive)
    uint64_t *dfull = conv + SH;   // accumulator buffer ready (2)
    uint64_t *dempty = dfull + 2;  // accumulator buffer drained (NEPI warps arrive) (2)
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(dempty + 2);
    float *red = reinterpret_cast<float *>(tmem_slot + 4);  // [NEPI][NJ] cross-warp reduction
    const int cid = blockIdx.x, ncl = gridDim.x;

    if (tid == 0) {
        for (int s = 0; s < SH; s++) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, 1);
            mbar_init(conv + s, NCONV);
        }
        for (int b = 0; b < 2; b++) {
            mbar_init(dfull + b, 1);
            mbar_init(dempty + b, NEPI);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    // two accumulator buffers of 2 NJ columns: [hi*hi + lo*hi | hi*lo], summed by the epilogue
    constexpr uint32_t TCOLS = 4 * NJ <= 32 ? 32 : 4 * NJ <= 64 ? 64 : 4 * NJ <= 128 ? 128 : 4 * NJ <= 256 ? 256 : 512;
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(su32(tmem_slot)),
                     "r"(TCOLS)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::: "memory");
    }
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {  // ------------------------------------------------ TMA producer
            int it = 0;
            for (int t = cid; t < p.nblk; t += ncl) {
                for (int kb = 0; kb < p.nkb; kb++, it++) {
                    const int s = it % SH;
                    if (it >= SH) mbar_wait(empty + s, (unsigned)(((it / SH) - 1) & 1));
                    unsigned char *st = smem + (size_t)s * HSTAGE;
                    mbar_expect_tx(full + s, A_BYTES + 2 * D_BYTES);
                    tma_2d<1>(st, &mB, kb * BK, t * BM, su32(full + s));
#pragma unroll
                    for (int g = 0; g < NJ / 32; g++) {
                        tma_2d<1>(st + 2 * A_BYTES + g * (BK * 128), &mDhi, 32 * g, kb * BK, su32(full + s));
                        tma_2d<1>(st + 2 * A_BYTES + D_BYTES + g * (BK * 128), &mDlo, 32 * g, kb * BK, su32(full + s));
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {  // ------------------------------------------------ MMA issuer
            int it = 0, gc = 0;
            for (int t = cid; t < p.nblk; t += ncl, gc++) {
                const int bd = gc & 1;
                if (gc >= 2) mbar_wait(dempty + bd, (unsigned)(((gc - 2) >> 1) & 1));
                fence_after();
                const uint32_t d = tmem + (uint32_t)(bd * 2 * NJ);
                for (int kb = 0; kb < p.nkb; kb++, it++) {
                    const int s = it % SH;
                    mbar_wait(full + s, (unsigned)((it / SH) & 1));
                    mbar_wait(conv + s, (unsigned)((it / SH) & 1));
                    fence_after();
                    unsigned char *st = smem + (size_t)s * HSTAGE;
                    unsigned char *lo = st + A_BYTES;
#pragma unroll
                    for (int ks = 0; ks < BK / 8; ks++) {
                        if (p.dbg & 2) break;
                        const uint64_t ahi = desc_sw128(st + ks * 32, 16u, 1024u);
                        const uint64_t alo = desc_sw128(lo + ks * 32, 16u, 1024u);
                        // the D hi groups, then the D lo groups: LBO = stride of 32-column groups
                        const uint64_t bcat = desc_sw128(st + 2 * A_BYTES + ks * 1024, (uint32_t)(BK * 128), 512u, 1);
                        mma_ss<1>(d, ahi, bcat, ID2, (kb == 0 && ks == 0) ? 0u : 1u);
                        mma_ss<1>(d, alo, bcat, ID, 1u);
                    }
                    mma_commit<1>(empty + s);
                }
                mma_commit<1>(dfull + bd);
            }
        }
    } else if (warp >= 4 && warp < 4 + NCONV) {  // --------------------------- lo converters
        const int ct = tid - 4 * 32;
        int it = 0;
        for (int t = cid; t < p.nblk; t += ncl) {
            for (int kb = 0; kb < p.nkb; kb++, it++) {
                const int s = it % SH;
                mbar_wait(full + s, (unsigned)((it / SH) & 1));
                const float4 *src = reinterpret_cast<const float4 *>(smem + (size_t)s * HSTAGE);
                float4 *dst = reinterpret_cast<float4 *>(smem + (size_t)s * HSTAGE + A_BYTES);
#pragma unroll
                for (int v = 0; v < A_BYTES / 16 / (NCONV * 32); v++) {
                    if (p.dbg & 1) break;
                    const int e = ct + v * NCONV * 32;  // consecutive threads: consecutive 16-byte chunks
                    const float4 x = src[e];
                    dst[e] = make_float4(lo_of(x.x), lo_of(x.y), lo_of(x.z), lo_of(x.w));
                }
                fence_proxy_async_smem();  // generic-proxy writes -> tensor-core (async proxy) reads
                __syncwarp();
                if (lane == 0) mbar_arrive(conv + s);
            }
        }
    } else if (warp >= 4 + NCONV) {  // ---------------------------------------- epilogue
        const int q = warp & 3;  // TMEM lane quarter (warp id % 4 selects the accessible lanes)
        const int e = warp - (4 + NCONV);
        int gc = 0;
        for (int t = cid; t < p.nblk; t += ncl, gc++) {
            const int bd = gc & 1;
            // row of this lane: (i, k) = block row t*128 + 32q + lane
            const int64_t grow = (int64_t)t * BM + q * 32 + lane;
            const float *crow = p.C + (grow % p.nk) * p.nj;
            mbar_wait(dfull + bd, (unsigned)((gc >> 1) & 1));
            fence_after();
            float v[NJ];
#pragma unroll
            for (int c0 = 0; c0 < NJ; c0 += 16) {
                uint32_t r[16];
                uint32_t r2[16];
                tmem_ld16(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(bd * 2 * NJ + c0), r);
                tmem_ld16(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(bd * 2 * NJ + NJ + c0), r2);
                wait_ld();
#pragma unroll
                for (int c = 0; c < 16; c++) v[c0 + c] = __uint_as_float(r[c]) + __uint_as_float(r2[c]);
            }
            fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(dempty + bd);
#pragma unroll
            for (int c = 0; c < NJ; c += 4) {
                const float4 cv = __ldg(reinterpret_cast<const float4 *>(crow + c));
                v[c] *= cv.x; v[c + 1] *= cv.y; v[c + 2] *= cv.z; v[c + 3] *= cv.w;
            }
            // sum over the warp's 32 rows, column by column (butterfly: every lane ends with all sums)
#pragma unroll
            for (int c = 0; c < NJ; c++) {
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) v[c] += __shfl_xor_sync(0xffffffffu, v[c], o);
            }
            // warps in fixed order through shared memory, then one partial row per block
            named_bar(1, NEPI * 32);  // previous block's red[] consumed
#pragma unroll
            for (int c = 0; c < NJ; c++)
                if ((c & 31) == lane) red[e * NJ + c] = v[c];  // static register indices
            named_bar(1, NEPI * 32);
            if (e == 0) {
                for (int c = lane; c < NJ; c += 32) {
                    float s = red[c];
#pragma unroll
                    for (int w = 1; w < NEPI; w++) s += red[w * NJ + c];
                    p.part[(int64_t)t * p.nj + c] = s;
                }
            }
        }
    }
    __syncwarp();
    fence_before();
    __syncthreads();
    if (warp == 2) {
        fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(TCOLS) : "memory");
    }
}

// lo half of D (raw-hi split)
__global__ void mttc_dlo(const float *__restrict__ D, float *__restrict__ lo, int64_t n) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
        lo[e] = lo_of(D[e]);
}

// A[i][j] += sum over the nk/128 blocks of row i, in block order
__global__ void mttc_reduce(float *__restrict__ A, const float *__restrict__ part, int64_t ni, int64_t nj, int bpi) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ni * nj; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = e / nj, j = e % nj;
        float s = part[(i * bpi) * nj + j];
        for (int b = 1; b < bpi; b++) s += part[(i * bpi + b) * nj + j];
        A[e] += s;
    }
}

}  // namespace mttc

// The tensor path applies when the tile is the MMA-legal point (1, nj, 128, 32) and the shapes fit it.
bool mttkrp_tc_applicable(const int64_t *dims, const int64_t *tiles) {
    const int64_t ni = dims[0], nj = dims[1], nk = dims[2], nl = dims[3];
    if (tiles[0] != 1 || tiles[1] != nj || tiles[2] != 128 || tiles[3] != 32) return false;
    if (nj != 32 && nj != 64 && nj != 128) return false;
    if (nk % 128 != 0 || nl % 32 != 0 || ni * nk / 128 > INT32_MAX) return false;
    return tcm::encode_fn() != nullptr;
}

// ws: nj*nl (D lo) + ni*nk/128*nj (block partials) floats
size_t mttkrp_tc_ws_floats(const int64_t *dims) { return (size_t)(dims[1] * dims[3] + dims[0] * dims[2] / 128 * dims[1]); }

cudaError_t launch_mttkrp_tc(float *A, const float *B, const float *C, const float *D, const int64_t *dims, float *ws,
                             cudaStream_t s, cudaEvent_t *ev, int64_t *launched) {
    using namespace mttc;
    Args p{};
    p.ni = dims[0]; p.nj = dims[1]; p.nk = dims[2]; p.nl = dims[3];
    p.nblk = (int)(p.ni * p.nk / BM);
    p.nkb = (int)(p.nl / BK);
    p.C = C;
#ifdef EATSS_DEVTOOLS  // cost-isolation switches (results then wrong): never in the product build
    p.dbg = getenv("EATSS_MTC_DBG") ? atoi(getenv("EATSS_MTC_DBG")) : 0;
#else
    p.dbg = 0;
#endif
    float *dlo = ws;
    p.part = ws + p.nj * p.nl;
    CUtensorMap mB, mDhi, mDlo;
    const CUtensorMapSwizzle swK = CU_TENSOR_MAP_SWIZZLE_128B, swMN = CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
    if (!tcm::make_map(&mB, B, p.ni * p.nk, p.nl, p.nl, BK, BM, swK) ||
        !tcm::make_map(&mDhi, D, p.nl, p.nj, p.nj, 32, BK, swMN) ||
        !tcm::make_map(&mDlo, dlo, p.nl, p.nj, p.nj, 32, BK, swMN))
        return cudaErrorInvalidValue;
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    mttc_dlo<<<64, 256, 0, s>>>(D, dlo, p.nj * p.nl);
    if (launched) (*launched)++;
    const int grid = std::min(p.nblk, nsm);
    cudaError_t e = cudaSuccess;
    auto go = [&](auto kern, int nj) -> cudaError_t {
        const int hstage = 2 * BM * BK * 4 + 2 * BK * nj * 4;
        int optin = 232448;
        cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        auto bytes = [&](int sh) { return 1024 + sh * hstage + 256 + NEPI * nj * 4; };
        p.S = SMAX;
        static const int st_env = getenv("EATSS_MTC_STAGES") ? atoi(getenv("EATSS_MTC_STAGES")) : 0;  // development
        if (st_env > 0) p.S = std::max(2, std::min(8, st_env));
        while (p.S > 2 && bytes(p.S) > optin) p.S--;
        const int smem = bytes(p.S);
        cudaError_t r = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (r != cudaSuccess) return r;
        if (ev) cudaEventRecord(ev[0], s);
        kern<<<grid, NTHREADS, smem, s>>>(mB, mDhi, mDlo, p);
        if (ev) cudaEventRecord(ev[1], s);
        return cudaGetLastError();
    };
    if (p.nj == 32) e = go(mttkrp_tc_kernel<32>, 32);
    else if (p.nj == 64) e = go(mttkrp_tc_kernel<64>, 64);
    else e = go(mttkrp_tc_kernel<128>, 128);
    if (launched) (*launched)++;
    if (e != cudaSuccess) return e;
    mttc_reduce<<<256, 256, 0, s>>>(A, p.part, p.ni, p.nj, (int)(p.nk / BM));
    if (launched) (*launched)++;
    return cudaGetLastError();
}

}  // namespace eatss
