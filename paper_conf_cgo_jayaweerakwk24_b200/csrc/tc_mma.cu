// tc_mma.cu -- tcgen05 3xTF32 GEMM for MMA-legal tiles (the
// "tensor-core EATSS mode"): Ti = 128 rows of i per CTA (UMMA M), Tj <= 256 columns of j
// (UMMA N, multiple of 16), k in blocks of 32 (one 128-byte swizzle atom of fp32/tf32).
//
// Same loop-nest semantics as the SIMT executor (Fig. 4: ti -> blockIdx.y,
// tj -> blockIdx.x, k sequential); fp32-accurate via 3xTF32 (reading Q26):
//   C = beta*C + alpha * sum_k (Ahi*Bhi + Ahi*Blo + Alo*Bhi),
//   hi = rna_tf32(x), lo = rna_tf32(x - hi), computed once per operand by split_kernel.
// Pipeline (warp-specialised, mbarrier hand-off, one CTA per SM):
//   warp 0  TMA producer: 2-D tensor-map loads (SWIZZLE_128B) of Ahi/Alo (K-major, 128 x 32)
//           and Bhi/Blo (MN-major, 32 x Tj) into an S-stage ring;
//   warp 1  MMA issuer: per 8-k step three kind::tf32 MMAs (M=128, N=Tj) from shared-memory
//           descriptors into a TMEM accumulator; tcgen05.commit frees the ring slot;
//   warps 4..11 epilogue: the k loop is split into chunks of R k-blocks accumulated in two
//           alternating TMEM buffers (the tensor core accumulates with truncation); each
//           chunk is drained with tcgen05.ld into fp32 registers, then C is updated.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <mutex>

#include "contract.cuh"

namespace eatss {
namespace tcm {

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
__device__ __forceinline__ void tma_2d(void *dst, const CUtensorMap *map, int c0, int c1, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n" ::"r"(
            su32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(su32(bar))
        : "memory");
}
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory"); }
__device__ __forceinline__ void wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory"); }
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15}, [%16];\n"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr)
        : "memory");
}
__device__ __forceinline__ void mma_ss(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t *bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(su32(bar))
                 : "memory");
}
// UMMA smem descriptor with SWIZZLE_128B (layout type 2), sm_100 version bit
// layout type 2 = SWIZZLE_128B (K-major A), 1 = SWIZZLE_128B_BASE32B (the only smem layout
// UMMA accepts for MN-major tf32 operands: 32-byte chunks XOR-swizzled over 4-row atoms)
__device__ __forceinline__ uint64_t desc_sw128(const void *p, uint32_t lbo, uint32_t sbo, uint32_t layout = 2) {
    uint64_t d = 0;
    d |= (uint64_t)((su32(p) >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)layout << 61;
    return d;
}
// kind::tf32: D f32, A tf32 K-major, B tf32 MN-major, M = 128, N = n
__host__ __device__ constexpr uint32_t idesc(int n) {
    return (1u << 4) | (2u << 7) | (2u << 10) | (1u << 16) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}

constexpr int BK = 32;         // k per stage (128-byte swizzle atom of fp32)
constexpr int BM = 128;        // rows of i per CTA (UMMA M)
constexpr int NEPI = 8;        // epilogue warps (4..11): two per TMEM lane quarter
constexpr int NTHREADS = (4 + NEPI) * 32;

struct Args {
    int64_t M, N, K;
    float *__restrict__ C;
    int64_t ldc;
    float alpha, beta;
    int init_zero;
    int BN;   // Tj (multiple of 16, <= 256)
    int S;    // ring stages
    int R;    // k-blocks per accumulator chunk
    int debug;
};

template <int BNT>  // columns of j per CTA (compile-time: per-thread chunk sums live in registers)
__global__ void __launch_bounds__(NTHREADS, 1)
    tc_mma_kernel(const __grid_constant__ CUtensorMap mAhi, const __grid_constant__ CUtensorMap mAlo,
                  const __grid_constant__ CUtensorMap mBhi, const __grid_constant__ CUtensorMap mBlo, const Args p) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char *smem = reinterpret_cast<unsigned char *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t i0 = (int64_t)blockIdx.y * BM, j0 = (int64_t)blockIdx.x * BNT;
    const int nkb = (int)((p.K + BK - 1) / BK);
    const int R = p.R, nchunks = (nkb + R - 1) / R;
    constexpr int A_BYTES = BM * BK * 4;        // 16 KB
    constexpr int B_BYTES = BK * BNT * 4;       // <= 32 KB
    constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)p.S * STAGE);
    uint64_t *empty = full + p.S;
    uint64_t *dfull = empty + p.S;
    uint64_t *dempty = dfull + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(dempty + 2);

    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(su32(tmem_slot)),
                     "r"(512)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::: "memory");
    }
    if (tid == 0) {
        for (int s = 0; s < p.S; s++) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, 1);
        }
        for (int b = 0; b < 2; b++) {
            mbar_init(dfull + b, 1);
            mbar_init(dempty + b, NEPI);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&mAhi)) : "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&mBhi)) : "memory");
    }
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {  // ---------------------------------------------- TMA producer
            for (int kb = 0; kb < nkb; kb++) {
                const int s = kb % p.S;
                if (kb >= p.S) mbar_wait(empty + s, (unsigned)(((kb / p.S) - 1) & 1));
                unsigned char *st = smem + (size_t)s * STAGE;
                mbar_expect_tx(full + s, STAGE);
                const int k0 = kb * BK;
                tma_2d(st, &mAhi, k0, (int)i0, full + s);
                tma_2d(st + A_BYTES, &mAlo, k0, (int)i0, full + s);
#pragma unroll
                for (int g = 0; g < BNT / 32; g++) {
                    tma_2d(st + 2 * A_BYTES + g * (BK * 128), &mBhi, (int)j0 + 32 * g, k0, full + s);
                    tma_2d(st + 2 * A_BYTES + B_BYTES + g * (BK * 128), &mBlo, (int)j0 + 32 * g, k0, full + s);
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {  // ---------------------------------------------- MMA issuer
            constexpr uint32_t ID = idesc(BNT);
            // A: K-major SW128, SBO = 8 rows x 128 B.  B: MN-major SW128_BASE32B, LBO = stride of the
            // 32-column groups (BK rows x 128 B), SBO = stride of the 4-row swizzle atoms (512 B)
            constexpr uint32_t a_lbo = 16u, b_lbo = (uint32_t)(BK * 128), b_sbo = 512u;
            for (int kb = 0; kb < nkb; kb++) {
                const int s = kb % p.S;
                const int ch = kb / R, bd = ch & 1;
                const bool first = (kb % R) == 0;
                if (first && ch >= 2) mbar_wait(dempty + bd, (unsigned)(((ch - 2) >> 1) & 1));
                mbar_wait(full + s, (unsigned)((kb / p.S) & 1));
                fence_after();
                unsigned char *st = smem + (size_t)s * STAGE;
                if (p.debug && kb == 0 && blockIdx.x == 0 && blockIdx.y == 0) {
                    // debug: dump raw stage words (Ahi then Bhi) into C's first row(s)
                    const float *w = reinterpret_cast<const float *>(st);
                    for (int x = 0; x < 256; x++) p.C[x] = w[x];
                    const float *wb = reinterpret_cast<const float *>(st + 2 * A_BYTES);
                    for (int x = 0; x < 256; x++) p.C[256 + x] = wb[x];
                }
                const uint32_t d = tmem + (uint32_t)(bd * 256);
#pragma unroll
                for (int ks = 0; ks < BK / 8; ks++) {
                    // A K-major: 8 tf32 = 32 B into each 128-B row; B MN-major: one 8-k atom = 1 KB
                    const uint64_t ahi = desc_sw128(st + ks * 32, a_lbo, 1024);
                    const uint64_t alo = desc_sw128(st + A_BYTES + ks * 32, a_lbo, 1024);
                    const uint64_t bhi = desc_sw128(st + 2 * A_BYTES + ks * 1024, b_lbo, b_sbo, 1);
                    const uint64_t blo = desc_sw128(st + 2 * A_BYTES + B_BYTES + ks * 1024, b_lbo, b_sbo, 1);
                    mma_ss(d, ahi, bhi, ID, (first && ks == 0) ? 0u : 1u);
                    mma_ss(d, ahi, blo, ID, 1u);
                    mma_ss(d, alo, bhi, ID, 1u);
                }
                mma_commit(empty + s);
                if ((kb % R) == R - 1 || kb == nkb - 1) mma_commit(dfull + bd);
            }
        }
    } else if (warp >= 4) {  // ---------------------------------------- epilogue warps
        const int e = warp - 4, q = warp & 3, half = e >> 2;
        constexpr int CW = BNT / 2;  // columns per epilogue warp
        float acc[CW];
#pragma unroll
        for (int c = 0; c < CW; c++) acc[c] = 0.f;
        for (int ch = 0; ch < nchunks; ch++) {
            const int bd = ch & 1;
            mbar_wait(dfull + bd, (unsigned)((ch >> 1) & 1));
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
            if (lane == 0) mbar_arrive(dempty + bd);
        }
        // C = beta*C + alpha*acc for row i = i0 + 32q + lane, columns j0 + half*CW + c
        const int64_t i = i0 + q * 32 + lane;
        if (i < p.M && !(p.debug && i < 16)) {
            float *crow = p.C + i * p.ldc + j0 + half * CW;
            const int64_t jb = j0 + half * CW;
            const bool vec = ((p.ldc & 3) == 0) && (jb + CW <= p.N);
            if (vec) {
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
    fence_before();
    __syncthreads();
    if (warp == 2) {
        fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(512) : "memory");
    }
}

// hi = rna_tf32(x), lo = rna_tf32(x - hi)  (elementwise, 16-byte vectors)
__global__ void split_kernel(const float *__restrict__ x, float *__restrict__ hi, float *__restrict__ lo, int64_t n) {
    const int64_t n4 = n / 4;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n4; v += (int64_t)gridDim.x * blockDim.x) {
        const float4 a = reinterpret_cast<const float4 *>(x)[v];
        float4 h, l;
        float *ap = (float *)&a, *hp = (float *)&h, *lp = (float *)&l;
#pragma unroll
        for (int q = 0; q < 4; q++) {
            uint32_t hb, lb;
            asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(hb) : "f"(ap[q]));
            asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(lb) : "f"(ap[q] - __uint_as_float(hb)));
            hp[q] = __uint_as_float(hb);
            lp[q] = __uint_as_float(lb);
        }
        reinterpret_cast<float4 *>(hi)[v] = h;
        reinterpret_cast<float4 *>(lo)[v] = l;
    }
    for (int64_t t = n4 * 4 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
        uint32_t hb, lb;
        asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(hb) : "f"(x[t]));
        asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(lb) : "f"(x[t] - __uint_as_float(hb)));
        hi[t] = __uint_as_float(hb);
        lo[t] = __uint_as_float(lb);
    }
}

// ------------------------------------------------------------------ host side
typedef CUresult (*EncodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiled encode_fn() {
    static EncodeTiled fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &p, 12000, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeTiled>(p);
    });
    return fn;
}

// 2-D fp32 row-major [rows][cols] (row pitch `ld` elements), box {bc cols (inner), br rows}
static bool make_map(CUtensorMap *m, const float *base, int64_t rows, int64_t cols, int64_t ld, int bc, int br,
                     CUtensorMapSwizzle sw) {
    EncodeTiled enc = encode_fn();
    if (!enc) return false;
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 4)};
    cuuint32_t box[2] = {(cuuint32_t)bc, (cuuint32_t)br};
    cuuint32_t es[2] = {1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float *>(base), dims, strides, box, es,
               CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace tcm

// Workspace for the split operands (library-owned, grown on demand, per device).
namespace {
std::mutex g_ws_mu;
float *g_ws = nullptr;
size_t g_ws_elems = 0;
int g_ws_dev = -1;
}  // namespace

static float *workspace(size_t elems) {
    std::lock_guard<std::mutex> lk(g_ws_mu);
    int dev = 0;
    cudaGetDevice(&dev);
    if (g_ws && (g_ws_elems < elems || g_ws_dev != dev)) {
        cudaFree(g_ws);
        g_ws = nullptr;
    }
    if (!g_ws) {
        if (cudaMalloc(&g_ws, elems * 4) != cudaSuccess) {
            g_ws = nullptr;
            return nullptr;
        }
        g_ws_elems = elems;
        g_ws_dev = dev;
    }
    return g_ws;
}

static int tcm_stages(int bn) {
    const int stage = 2 * tcm::BM * tcm::BK * 4 + 2 * tcm::BK * bn * 4;
    int S = (int)((232448 - 2048) / stage);
    if (const char *e = getenv("EATSS_TCM_STAGES")) S = atoi(e);
    return std::max(2, std::min(S, 8));
}

bool tcm_applicable(const ContractNest &n, const ContractPlan &p) {
    if (n.f64 || n.transB) return false;
    if (p.Ti != tcm::BM || p.Tj < 32 || p.Tj > 256 || (p.Tj % 32) != 0) return false;
    if ((n.lda % 4) || (n.ldb % 4)) return false;
    if (n.M > INT32_MAX || n.N > INT32_MAX || n.K > INT32_MAX) return false;
    const int stage = 2 * tcm::BM * tcm::BK * 4 + 2 * tcm::BK * (int)p.Tj * 4;
    return 2 * stage + 2048 <= 232448 && tcm::encode_fn() != nullptr;
}

cudaError_t launch_tcm_contraction(const ContractNest &n, const ContractPlan &p, cudaStream_t s) {
    if (!tcm_applicable(n, p)) return cudaErrorNotSupported;
    const int64_t a_elems = n.M * n.lda, b_elems = n.K * n.ldb;
    float *ws = workspace((size_t)(2 * a_elems + 2 * b_elems + 64));
    if (!ws) return cudaErrorMemoryAllocation;
    float *Ahi = ws, *Alo = Ahi + a_elems, *Bhi = Alo + a_elems, *Blo = Bhi + b_elems;
    const float *A = static_cast<const float *>(n.A), *B = static_cast<const float *>(n.B);
    tcm::split_kernel<<<148 * 8, 256, 0, s>>>(A, Ahi, Alo, a_elems);
    tcm::split_kernel<<<148 * 8, 256, 0, s>>>(B, Bhi, Blo, b_elems);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    CUtensorMap mAhi, mAlo, mBhi, mBlo;
    const int bn = (int)p.Tj;
    const CUtensorMapSwizzle swA = CU_TENSOR_MAP_SWIZZLE_128B, swB = CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
    if (!tcm::make_map(&mAhi, Ahi, n.M, n.K, n.lda, tcm::BK, tcm::BM, swA) ||
        !tcm::make_map(&mAlo, Alo, n.M, n.K, n.lda, tcm::BK, tcm::BM, swA) ||
        !tcm::make_map(&mBhi, Bhi, n.K, n.N, n.ldb, 32, tcm::BK, swB) ||
        !tcm::make_map(&mBlo, Blo, n.K, n.N, n.ldb, 32, tcm::BK, swB))
        return cudaErrorInvalidValue;
    tcm::Args a;
    a.M = n.M; a.N = n.N; a.K = n.K;
    a.C = static_cast<float *>(n.C); a.ldc = n.ldc;
    a.alpha = (float)n.alpha; a.beta = (float)n.beta; a.init_zero = n.init_zero ? 1 : 0;
    a.BN = bn;
    a.S = tcm_stages(bn);
    a.R = 16;  // 16 k-blocks = 512 k per accumulator chunk
    if (const char *ev = getenv("EATSS_TCM_CHUNK")) a.R = std::max(1, atoi(ev));
    a.debug = getenv("EATSS_TCM_DEBUG") ? atoi(getenv("EATSS_TCM_DEBUG")) : 0;
    const int stage = 2 * tcm::BM * tcm::BK * 4 + 2 * tcm::BK * bn * 4;
    const int smem = a.S * stage + 1024 /*align*/ + 8 * (2 * a.S + 4) + 16;
    void (*k)(const CUtensorMap, const CUtensorMap, const CUtensorMap, const CUtensorMap, const tcm::Args) = nullptr;
    switch (bn) {
        case 32: k = tcm::tc_mma_kernel<32>; break;
        case 64: k = tcm::tc_mma_kernel<64>; break;
        case 96: k = tcm::tc_mma_kernel<96>; break;
        case 128: k = tcm::tc_mma_kernel<128>; break;
        case 160: k = tcm::tc_mma_kernel<160>; break;
        case 192: k = tcm::tc_mma_kernel<192>; break;
        case 224: k = tcm::tc_mma_kernel<224>; break;
        case 256: k = tcm::tc_mma_kernel<256>; break;
        default: return cudaErrorNotSupported;
    }
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    dim3 grid((unsigned)((n.N + bn - 1) / bn), (unsigned)((n.M + tcm::BM - 1) / tcm::BM));
    k<<<grid, tcm::NTHREADS, smem, s>>>(mAhi, mAlo, mBhi, mBlo, a);
    return cudaGetLastError();
}

}  // namespace eatss
