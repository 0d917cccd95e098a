// tc_gemm.cu -- tensor-core (tcgen05) executor of a tiled gemm-family nest, fp32-accurate
// via 3xTF32 (sm_100a).
//
// Same tile semantics as the SIMT executor (Fig. 4): one CTA owns the
// Ti x Tj output tile of (ti, tj) = (blockIdx.y, blockIdx.x) and walks k.
// The tile is computed TRANSPOSED on the tensor core, D[j][i] = sum_k B[k][j] A[i][k]:
//   * M = j (the CMA loop l_s1, 128 rows per MMA; ceil(Tj/128) M-blocks per CTA),
//   * N = i (Ti rounded up to 16), K = k (8 tf32 per MMA = one pipeline stage),
// so the wide EATSS dimension (Tj = 1024) feeds the 128-row MMA and the narrow one
// (Ti = 16) is the N extent.  Warp-specialised pipeline (all hand-off via mbarriers):
//   * warp 0 (one lane)  -- PRODUCER: cp.async.bulk copies of the raw fp32 slices
//     B(k0..k0+8, j-tile) and A(i-tile, k0..k0+8) into an S-slot shared-memory ring;
//   * warps 4..11        -- CONVERTERS: split B into tf32 hi/lo (hi = rna(x),
//     lo = rna(x - hi); reading Q26) and write both to TMEM with tcgen05.st (the
//     M-side operand of a TS-MMA: lane = j, column = k); split A into hi/lo K-major
//     core matrices in shared memory (the N-side operand, UMMA smem descriptor);
//     two operand buffers in flight; afterwards they run the epilogue;
//   * warp 1 (one lane)  -- MMA ISSUER: per stage and M-block 3 MMAs
//     (hi*hi + hi*lo + lo*hi, fp32 accumulation in TMEM), tcgen05.commit frees the
//     operand buffer; a final commit hands the accumulators to the epilogue;
//   * warp 2             -- TMEM allocator (alloc / dealloc).
// Epilogue: tcgen05.ld (one TMEM lane per thread = one j) and C = beta*C + alpha*D,
// coalesced along j.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include "contract.cuh"
#include "devsw.hpp"

namespace eatss {

namespace tc {

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *b, unsigned c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(su32(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, unsigned parity) {
    asm volatile(
        "{\n.reg .pred p;\nW_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra W_%=;\n}\n" ::"r"(su32(b)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                     su32(dst)),
                 "l"(src), "r"(bytes), "r"(su32(bar))
                 : "memory");
}
__device__ __forceinline__ uint32_t to_tf32(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(r) : "f"(x));
    return r;
}
__device__ __forceinline__ void split3(float x, uint32_t &hi, uint32_t &lo) {
    hi = to_tf32(x);
    lo = to_tf32(x - __uint_as_float(hi));
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&v)[8]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};\n" ::"r"(taddr),
                 "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
                 : "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15}, [%16];\n"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr)
        : "memory");
}
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory"); }
__device__ __forceinline__ void wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory"); }
__device__ __forceinline__ void wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }

// D[tmem] (+)= A[tmem] * B[smem desc], kind::tf32, cta_group::1
__device__ __forceinline__ void mma_tf32_ts(uint32_t d, uint32_t a, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(d),
        "r"(a), "l"(bdesc), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t *bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(su32(bar))
                 : "memory");
}

// UMMA shared-memory descriptor, K-major, SWIZZLE_NONE (canonical ((8,n),2):((1,SBO),LBO)
// in 16-byte units): core matrix = 8 rows x 16 B contiguous; LBO = stride between the two
// 16-byte K chunks of one MMA (K = 8 tf32); SBO = stride between 8-row groups.
__device__ __forceinline__ uint64_t smem_desc(const void *p, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((su32(p) >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;  // descriptor version (sm_100)
    return d;                // base_offset 0, lbo_mode 0, layout SWIZZLE_NONE
}

// kind::tf32 instruction descriptor: D f32, A/B tf32, both K-major, M=128, N=n
__host__ __device__ constexpr uint32_t idesc_tf32(int n) {
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}

struct Args {
    int64_t M, N, K;
    const float *__restrict__ A;
    int64_t lda;
    const float *__restrict__ B;
    int64_t ldb;
    float *__restrict__ C;
    int64_t ldc;
    float alpha, beta;
    int init_zero;
    int Ti, Tj;   // clipped tile
    int NM;       // MMA N (Ti rounded up to 16)
    int MB;       // 128-row M-blocks per CTA
    int S;        // raw ring depth
    int bjp;      // raw B row pitch (floats)
    uint32_t tmem_cols;
    int a_bulk;   // A rows by bulk copy (1) or by converter loads (0)
    int R;        // stages per accumulator chunk
};

constexpr int KS = 8;            // k per stage = one tf32 MMA
constexpr int NCONV = 8;         // converter warps (4..11): two per TMEM lane quarter
constexpr int NTHREADS = (4 + NCONV) * 32;

template <int NMT>  // MMA N (= Ti rounded up to 16), compile-time so the fp32 chunk sums stay in registers
__global__ void __launch_bounds__(NTHREADS, 1) tc3_gemm_kernel(const Args p) {
    extern __shared__ __align__(1024) unsigned char smem[];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t i0 = (int64_t)blockIdx.y * p.Ti, j0 = (int64_t)blockIdx.x * p.Tj;
    const int rows = (int)min((int64_t)p.Ti, p.M - i0);
    const int cols = (int)min((int64_t)p.Tj, p.N - j0);
    const int nst = (int)((p.K + KS - 1) / KS);

    // ---- shared memory carve-up
    const int ring_b = KS * p.bjp;  // floats
    const int slot = ring_b + p.NM * KS;
    float *ring = reinterpret_cast<float *>(smem);
    unsigned char *nside = smem + (((size_t)p.S * slot * 4 + 127) & ~(size_t)127);
    const int nbuf_bytes = p.NM * 32;  // one operand (hi or lo) of NM rows x 8 k
    uint64_t *full = reinterpret_cast<uint64_t *>(nside + 4 * nbuf_bytes);
    uint64_t *empty = full + p.S;
    uint64_t *opnd_full = empty + p.S;   // [2]
    uint64_t *opnd_empty = opnd_full + 2; // [2]
    uint64_t *acc_done = opnd_empty + 2;
    uint64_t *dfull = acc_done + 1;   // [2] accumulator chunk ready (MMA commit)
    uint64_t *dempty = dfull + 2;     // [2] accumulator chunk drained (converter warps)
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(dempty + 2);

    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(su32(tmem_slot)),
                     "r"(p.tmem_cols)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::: "memory");
    }
    if (tid == 0) {
        for (int s = 0; s < p.S; s++) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, NCONV);
        }
        for (int b = 0; b < 2; b++) {
            mbar_init(opnd_full + b, NCONV);
            mbar_init(opnd_empty + b, 1);
        }
        mbar_init(acc_done, 1);
        for (int b = 0; b < 2; b++) {
            mbar_init(dfull + b, 1);
            mbar_init(dempty + b, NCONV);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tmem_slot;
    // TMEM columns: 2 accumulator buffers [0, 2*MB*NM) (the k-loop is split into chunks of R
    // stages accumulated in alternate buffers and summed in fp32 registers: the tensor core
    // accumulates with truncation, so a single K=4000 accumulation drifts by ~K*2^-24);
    // then 2 operand buffers x MB x 16 (8 hi + 8 lo) columns
    const uint32_t acol0 = (uint32_t)(2 * p.MB * p.NM);
    const int R = p.R;
    const int nchunks = (nst + R - 1) / R;
    const bool bulk_b = (cols & 3) == 0;
    const bool a_bulk_enabled = p.a_bulk != 0;

    if (warp == 0) {
        // ------------------------------------------------------------ producer
        if (lane == 0) {
            for (int t = 0; t < nst; t++) {
                const int s = t % p.S;
                if (t >= p.S) mbar_wait(empty + s, (unsigned)(((t / p.S) - 1) & 1));
                float *Bs = ring + (size_t)s * slot;
                float *As = Bs + ring_b;
                const int64_t k0 = (int64_t)t * KS;
                const int kt = (int)min((int64_t)KS, p.K - k0);
                const bool abulk = (kt == KS) && a_bulk_enabled;
                const unsigned bytes = (bulk_b ? (unsigned)(kt * cols * 4) : 0u) + (abulk ? (unsigned)(rows * KS * 4) : 0u);
                mbar_expect_tx(full + s, bytes);
                if (bulk_b)
                    for (int kk = 0; kk < kt; kk++)
                        bulk_g2s(Bs + kk * p.bjp, p.B + (k0 + kk) * p.ldb + j0, (unsigned)(cols * 4), full + s);
                if (abulk)
                    for (int r = 0; r < rows; r++) bulk_g2s(As + r * KS, p.A + (i0 + r) * p.lda + k0, KS * 4, full + s);
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------------------ MMA issuer
        if (lane == 0) {
            const uint32_t idesc = idesc_tf32(p.NM);
            for (int t = 0; t < nst; t++) {
                const int b = t & 1;
                const int ch = t / R, bd = ch & 1;
                const bool first = (t % R) == 0;
                if (first && ch >= 2) mbar_wait(dempty + bd, (unsigned)(((ch - 2) >> 1) & 1));
                mbar_wait(opnd_full + b, (unsigned)((t >> 1) & 1));
                fence_after();
                const unsigned char *nhi = nside + (size_t)b * 2 * nbuf_bytes;
                const uint64_t dhi = smem_desc(nhi, 128, 256), dlo = smem_desc(nhi + nbuf_bytes, 128, 256);
                for (int mb = 0; mb < p.MB; mb++) {
                    const uint32_t d = tmem + (uint32_t)((bd * p.MB + mb) * p.NM);
                    const uint32_t ahi = tmem + acol0 + (uint32_t)(b * p.MB * 16 + mb * 16), alo = ahi + 8;
                    mma_tf32_ts(d, ahi, dhi, idesc, first ? 0u : 1u);
                    mma_tf32_ts(d, ahi, dlo, idesc, 1u);
                    mma_tf32_ts(d, alo, dhi, idesc, 1u);
                }
                mma_commit(opnd_empty + b);  // operand buffer b may be overwritten once these MMAs finish
                if ((t % R) == R - 1 || t == nst - 1) mma_commit(dfull + bd);  // chunk ready for draining
            }
        }
    } else if (warp >= 4) {
        // ------------------------------------------------------------ converters
        const int c = warp - 4;       // 0..NCONV-1
        const int q = warp & 3;       // TMEM lane quarter (warp id within its warpgroup)
        const int mg = c >> 2, ngroups = NCONV / 4;
        const int ctid = c * 32 + lane;
        // fp32 register sums of the drained accumulator chunks: [my M-blocks][NM columns]
        constexpr int MW = 64 / NMT;  // M-blocks per converter warp (host guarantees ceil(MB/2) <= MW)
        float acc[MW][NMT];
#pragma unroll
        for (int m = 0; m < MW; m++)
#pragma unroll
            for (int x = 0; x < NMT; x++) acc[m][x] = 0.f;
        int next_drain = 0;
        auto drain = [&](int ch) {
            const int bd = ch & 1;
            mbar_wait(dfull + bd, (unsigned)((ch >> 1) & 1));
            fence_after();
#pragma unroll
            for (int m = 0; m < MW; m++) {
                const int mb = mg + m * ngroups;
                if (mb < p.MB) {
#pragma unroll
                    for (int c0 = 0; c0 < NMT; c0 += 16) {
                        uint32_t v[16];
                        tmem_ld16(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)((bd * p.MB + mb) * NMT + c0), v);
                        wait_ld();
#pragma unroll
                        for (int cc = 0; cc < 16; cc++) acc[m][c0 + cc] += __uint_as_float(v[cc]);
                    }
                }
            }
            fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(dempty + bd);
        };
        auto chunk_end = [&](int ch) { return min((ch + 1) * R, nst) - 1; };
        for (int t = 0; t < nst; t++) {
            const int s = t % p.S, b = t & 1;
            const int64_t k0 = (int64_t)t * KS;
            const int kt = (int)min((int64_t)KS, p.K - k0);
            const float *Bs = ring + (size_t)s * slot;
            const float *As = Bs + ring_b;
            mbar_wait(full + s, (unsigned)((t / p.S) & 1));
            if (t >= 2) mbar_wait(opnd_empty + b, (unsigned)(((t - 2) >> 1) & 1));
            fence_after();
            // M-side: B(k, j) -> TMEM lanes j, columns [hi 0..7 | lo 8..15] of buffer b
            for (int mb = mg; mb < p.MB; mb += ngroups) {
                const int jl = mb * 128 + q * 32 + lane;
                uint32_t hi[8], lo[8];
#pragma unroll
                for (int kk = 0; kk < KS; kk++) {
                    float x = 0.f;
                    if (kk < kt && jl < cols) x = bulk_b ? Bs[kk * p.bjp + jl] : __ldg(p.B + (k0 + kk) * p.ldb + j0 + jl);
                    split3(x, hi[kk], lo[kk]);
                }
                const uint32_t ta = tmem + ((uint32_t)(q * 32) << 16) + acol0 + (uint32_t)(b * p.MB * 16 + mb * 16);
                tmem_st8(ta, hi);
                tmem_st8(ta + 8, lo);
            }
            // N-side: A(i, k) -> smem hi/lo in K-major core matrices (LBO 128 B, SBO 256 B)
            unsigned char *nhi = nside + (size_t)b * 2 * nbuf_bytes, *nlo = nhi + nbuf_bytes;
            for (int e = ctid; e < p.NM * KS; e += NCONV * 32) {
                const int r = e >> 3, kk = e & 7;
                float x = 0.f;
                if (r < rows && kk < kt)
                    x = (kt == KS && a_bulk_enabled) ? As[r * KS + kk] : __ldg(p.A + (i0 + r) * p.lda + k0 + kk);
                uint32_t h, l;
                split3(x, h, l);
                const int off = (r >> 3) * 256 + (kk >> 2) * 128 + (r & 7) * 16 + (kk & 3) * 4;
                *reinterpret_cast<uint32_t *>(nhi + off) = h;
                *reinterpret_cast<uint32_t *>(nlo + off) = l;
            }
            wait_st();
            fence_proxy_async();
            fence_before();
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(opnd_full + b);
                mbar_arrive(empty + s);
            }
            // drain every chunk whose last stage was fed at least one stage ago
            while (next_drain < nchunks && chunk_end(next_drain) <= t - 1) drain(next_drain++);
        }
        while (next_drain < nchunks) drain(next_drain++);
        // ------------------------------------------------------------ epilogue
#pragma unroll
        for (int m = 0; m < MW; m++) {
            const int mb = mg + m * ngroups;
            const int jl = mb * 128 + q * 32 + lane;
            if (mb < p.MB && jl < cols) {
#pragma unroll
                for (int il = 0; il < NMT; il++) {
                    if (il < rows) {
                        float *cp = p.C + (i0 + il) * p.ldc + j0 + jl;
                        const float o = p.init_zero ? 0.f : p.beta * *cp;
                        *cp = fmaf(p.alpha, acc[m][il], o);
                    }
                }
            }
        }
    }
    fence_before();
    __syncthreads();
    if (warp == 2) {
        fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(p.tmem_cols)
                     : "memory");
    }
}

}  // namespace tc

static inline uint32_t pow2_cols(uint32_t c) {
    uint32_t r = 32;
    while (r < c) r <<= 1;
    return r;
}

static int tc_stages() {
    int S = 4;
    if (devsw("EATSS_TC_STAGES", 0) > 0) S = std::max(2, devsw("EATSS_TC_STAGES", 0));
    return S;
}

// Applicability + smem size of the tensor-core executor for a plan.
bool tc_plan(const ContractNest &n, const ContractPlan &p, int *smem_bytes, int *tmem_cols) {
    if (n.f64 || n.transB) return false;
    const int NM = (int)(((p.Ti + 15) / 16) * 16);
    const int MB = (int)((p.Tj + 127) / 128);
    if (NM > 64 || MB < 1) return false;
    if (((MB + 1) / 2) * NM > 64) return false;  // fp32 chunk sums per converter thread
    const uint32_t cols = (uint32_t)(2 * MB * NM + 2 * MB * 16);  // 2 accumulator + 2 operand buffers
    if (cols > 512) return false;
    if ((n.lda % 4) || (n.ldb % 4) || (reinterpret_cast<uintptr_t>(n.A) & 15) ||
        (reinterpret_cast<uintptr_t>(n.B) & 15))
        return false;
    const int bjp = (int)(((p.Tj + 3) / 4) * 4);
    const int S = tc_stages();
    const int64_t slot = (int64_t)(tc::KS * bjp + NM * tc::KS) * 4;
    const int64_t bytes = ((S * slot + 127) & ~127LL) + 4 * NM * 32 + 8 * (2 * S + 9) + 16;
    if (bytes > 232448) return false;
    *smem_bytes = (int)bytes;
    *tmem_cols = (int)pow2_cols(cols);
    return true;
}

cudaError_t launch_tc_contraction(const ContractNest &n, const ContractPlan &p, int carveout, cudaStream_t s) {
    int smem = 0, tcols = 0;
    if (!tc_plan(n, p, &smem, &tcols)) return cudaErrorNotSupported;
    tc::Args a;
    a.M = n.M; a.N = n.N; a.K = n.K;
    a.A = static_cast<const float *>(n.A); a.lda = n.lda;
    a.B = static_cast<const float *>(n.B); a.ldb = n.ldb;
    a.C = static_cast<float *>(n.C); a.ldc = n.ldc;
    a.alpha = (float)n.alpha; a.beta = (float)n.beta; a.init_zero = n.init_zero ? 1 : 0;
    a.Ti = (int)p.Ti; a.Tj = (int)p.Tj;
    a.NM = (int)(((p.Ti + 15) / 16) * 16);
    a.MB = (int)((p.Tj + 127) / 128);
    a.S = tc_stages();
    a.bjp = (int)(((p.Tj + 3) / 4) * 4);
    a.tmem_cols = (uint32_t)tcols;
    a.a_bulk = 0;
    a.a_bulk = devsw("EATSS_TC_ABULK", 0);
    a.R = 16;  // stages per accumulator chunk (128 k): drift ~128 * 2^-24 per chunk
    if (devsw("EATSS_TC_CHUNK", 0) > 0) a.R = std::max(2, devsw("EATSS_TC_CHUNK", 0));
    void (*k)(const tc::Args) = nullptr;
    switch (a.NM) {
        case 16: k = tc::tc3_gemm_kernel<16>; break;
        case 32: k = tc::tc3_gemm_kernel<32>; break;
        case 48: k = tc::tc3_gemm_kernel<48>; break;
        case 64: k = tc::tc3_gemm_kernel<64>; break;
        default: return cudaErrorNotSupported;
    }
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    (void)carveout;
    dim3 grid((unsigned)p.grid_x, (unsigned)p.grid_y, 1);
    k<<<grid, tc::NTHREADS, smem, s>>>(a);
    return cudaGetLastError();
}

}  // namespace eatss
