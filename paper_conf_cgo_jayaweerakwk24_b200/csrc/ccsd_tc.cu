// ccsd_tc.cu -- the 6-D CCSD(T) d1 contraction (BASELINE config 5) on
// the tensor pipe (tcgen05 3xTF32):
//
//   t3[h3][h2][h1][p6][p5][p4] -= sum_h7 t2[h7][p4][p5][h1] * v2[h3][h2][p6][h7]
//
// The update has AI = 12 flop/B (t3 is read and written once, K = H7 = 48), so on B200 it is
// HBM-bound once the arithmetic leaves the FFMA pipe: this executor makes the t3 stream the only
// thing the SMs wait for.  Tile vector (Th3, Th2, Th1, Tp6, Tp5, Tp4, Th7) with Th3 = 1,
// Th7 = H7 (whole reduction per tile), M = Th1*Tp5*Tp4 <= 128 output rows on the MMA M axis and
// N = Th2*Tp6 (multiple of 16, <= 256; Th2 > 1 needs Tp6 = P6) on the MMA N axis:
//   D[(h1,p5,p4)][(h2,p6)] = sum_h7 t2[h7][p4][p5][h1] * v2[h3][h2][p6][h7]   (UMMA M=128, A in TMEM)
//   t3[h3][h2][h1][p6][p5][p4] -= D   (epilogue, read-modify-write of t3 in global memory)
// The A operand depends on (h1,p5,p4) only: an epilogue group writes its tf32 hi/lo halves into
// TMEM once per A tile (lane = output row, 16 columns per 8-k step) and the CTA then walks every
// (h3,h2) unit that reuses it, so the MMAs read only the small v2 tile from shared memory.
// 3xTF32 with the raw-hi split (tc_mma.cu): hi = the operand itself (the tensor core truncates to
// tf32), lo = rna_tf32(x - rz_tf32(x)); v2's lo half is materialised once per call (21 MB).
//
// Warp roles (persistent, one CTA per SM): warp 0 loads the per-unit v2 tile (hi, lo) into an
// SV-stage ring by TMA; warp 1 issues the MMAs into NB TMEM accumulators; warp 2 owns TMEM; warps
// 4.. are NGRP epilogue groups of four warps, each taking every NGRP-th unit.  A group brings its
// unit's t3 tile into XB group-private shared buffers by TMA (XB = 2: the next owned unit's tile
// is requested before the current one is processed), subtracts the TMEM accumulator and writes
// the result straight to global memory (lane = output row m: a warp's 32 rows are contiguous t3
// elements, one coalesced streaming store per column).
// Measured history at dims 48: a single TMA ring + a separate store-issuer role
// ran at 3.6 TB/s, bounded by per-unit hand-offs between four single-thread roles, not by HBM;
// keeping shared pointers in the shared window (no generic accesses), blocking Th2 = 2 h2 per unit
// (MMA N = 96: half the MMA instructions per byte -- the tensor pipe's per-instruction cost, not
// its FLOP rate, bounded the N = 48 MMAs) and the group-private tiles bring it to 4.7 TB/s.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <mutex>

#include "tc_ptx.cuh"

namespace eatss {
namespace ccsdtc {

using namespace tcm;

constexpr int NGRP = 3;          // epilogue groups; group g owns the units u with u % NGRP == g
constexpr int XSMAX = 8;         // t3 tile slices per unit (barriers per group)
constexpr int NEPI = 4 * NGRP;   // epilogue warps (a group = one warp per TMEM lane quarter)
constexpr int NTHREADS = (4 + NEPI) * 32;
constexpr int MROWS = 128;  // UMMA M

struct Args {
    int H3, H2, H1, P6, P5, P4, H7;
    int Th1, Tp6, Tp5, Tp4;
    int n_h1t, n_p5t, n_p4t, n_p6t;
    int Th2, n_h2t;   // h2 tile: Th2 > 1 blocks Th2 consecutive h2 into one unit (needs Tp6 = P6, Tp4 = P4)
    int NV;           // MMA N = Th2 * Tp6 output columns (h2, p6) per unit
    int hh0, nhh;     // range of (h3, h2-tile) blocks of this launch (Th2 = 1: flattened (h3, h2))
    int64_t units;    // n_a * nhh * n_p6t
    int nkb;          // ceil(H7 / 32)
    int SV;           // V ring stages
    int bstride, NB;  // TMEM accumulator buffers (columns per buffer, count)
    int nks;          // 8-k MMA steps: ceil(H7 / 8)
    int a_col;        // TMEM column of A (hi at a_col + 16 ks, lo at + 8)
    int v_kb_bytes;   // NV * 128
    int v_stage;      // 2 * nkb * v_kb_bytes
    int x_bytes;      // t3 tile of a unit: Th2*Th1*Tp6*Tp5*Tp4*4
    int x_stage;      // x_bytes rounded up to 1 KB
    int XB;           // t3 tile buffers per epilogue group (2: the next owned unit is prefetched)
    int XS;           // XB = 1: the tile moves as XS slices (one TMA box and barrier each; 0 = whole tiles), so
                      // the next owned unit's slice s is requested as soon as slice s has been processed
    int sph, p6s;     // slices per h2 plane and p6 columns per slice (XS = Th2 * sph, p6s = Tp6 / sph)
    int order;        // 1: A tiles round-robin over CTAs (concurrent CTAs sweep whole t3 blocks)
    int dbg;          // development only (EATSS_CCSD_TC_DBG): 1 no MMA, 2 no t3 traffic, 4 no v2 loads
    unsigned long long *prof;  // development only (EATSS_CCSD_TC_PROF): cycles per wait site
};

struct Unit {
    int a, hh, p6t;
};
__device__ __forceinline__ float lo_of(float x) {
    const float hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
    uint32_t lb;
    asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(lb) : "f"(x - hi));
    return __uint_as_float(lb);
}
__device__ __forceinline__ Unit decode(const Args &p, int64_t u) {
    Unit w;
    w.p6t = (int)(u % p.n_p6t);
    const int64_t r = u / p.n_p6t;
    w.hh = p.hh0 + (int)(r % p.nhh);
    w.a = (int)(r / p.nhh);
    return w;
}
// The units of CTA c.  Every A tile owns R = nhh * n_p6t units (all (h3,h2) for fixed
// (h1,p5,p4) rows).  order 1: A tiles c, c+G, c+2G, ... whole, then an even share of the
// remaining n_a mod G tiles' units -- so at any moment the G CTAs update adjacent row blocks
// of the same (h3,h2,h1) t3 blocks (DRAM page locality) while each keeps its A tile resident.
// order 0: one contiguous range of the unit space per CTA.
struct Sched {
    int64_t n1, lo, n, R;
    int c, G, K1;
};
__device__ __forceinline__ Sched sched_of(const Args &p, int c, int G) {
    Sched sc;
    sc.c = c;
    sc.G = G;
    sc.R = (int64_t)p.nhh * p.n_p6t;
    const int n_a = p.n_h1t * p.n_p5t * p.n_p4t;
    if (p.order == 1) {
        sc.K1 = n_a / G;
        sc.n1 = (int64_t)sc.K1 * sc.R;
        const int64_t rem = (int64_t)(n_a - sc.K1 * G) * sc.R;
        sc.lo = rem * c / G;
        sc.n = sc.n1 + rem * (c + 1) / G - sc.lo;
    } else {
        sc.K1 = 0;
        sc.n1 = 0;
        sc.lo = p.units * c / G;
        sc.n = p.units * (c + 1) / G - sc.lo;
    }
    return sc;
}
__device__ __forceinline__ Unit unit_at(const Args &p, const Sched &sc, int64_t i) {
    if (i < sc.n1) {
        const int64_t k = i / sc.R, r2 = i % sc.R;
        Unit w;
        w.a = sc.c + (int)k * sc.G;
        w.hh = p.hh0 + (int)(r2 / p.n_p6t);
        w.p6t = (int)(r2 % p.n_p6t);
        return w;
    }
    return decode(p, (int64_t)sc.K1 * sc.G * sc.R + sc.lo + (i - sc.n1));
}
__device__ __forceinline__ void a_coords(const Args &p, int a, int &h1_0, int &p5_0, int &p4_0) {
    const int p4t = a % p.n_p4t;
    a /= p.n_p4t;
    const int p5t = a % p.n_p5t;
    const int h1t = a / p.n_p5t;
    h1_0 = h1t * p.Th1;
    p5_0 = p5t * p.Tp5;
    p4_0 = p4t * p.Tp4;
}

// t3 tile coordinates of a unit in the 5-D tensor map: Th2 = 1 -> dims (p4, p5, p6, h1, (h3,h2));
// Th2 > 1 -> dims ((p5,p4), p6, h1, h2, h3) (Tp4 = P4), so a tile never straddles two h3
__device__ __forceinline__ void x_coords(const Args &p, int hb, int p6t, int h1_0, int p5_0, int p4_0, int (&c)[5]) {
    if (p.Th2 == 1) {
        c[0] = p4_0; c[1] = p5_0; c[2] = p6t * p.Tp6; c[3] = h1_0; c[4] = hb;
    } else {
        const int h3 = hb / p.n_h2t, h2_0 = (hb - h3 * p.n_h2t) * p.Th2;
        c[0] = p5_0 * p.P4 + p4_0; c[1] = p6t * p.Tp6; c[2] = h1_0; c[3] = h2_0; c[4] = h3;
    }
}
// first row of the unit's v2 tile in v2 viewed as [(h3, h2, p6)][h7]
__device__ __forceinline__ int v_row(const Args &p, int hb, int p6t) {
    if (p.Th2 == 1) return hb * p.P6 + p6t * p.Tp6;
    const int h3 = hb / p.n_h2t, h2_0 = (hb - h3 * p.n_h2t) * p.Th2;
    return (h3 * p.H2 + h2_0) * p.P6 + p6t * p.Tp6;
}

// Incremental walk over a CTA's units (no 64-bit divisions in the loops): region 1 = whole A
// tiles c, c+G, ..., region 2 = the CTA's share of the remainder in plain unit order.
struct UnitIter {
    int a, hh, p6t;
    int64_t left1;
    bool r1;
};
__device__ __forceinline__ void iter_region2(const Args &p, const Sched &sc, UnitIter &w) {
    const Unit u = decode(p, (int64_t)sc.K1 * sc.G * sc.R + sc.lo);
    w.a = u.a;
    w.hh = u.hh;
    w.p6t = u.p6t;
    w.r1 = false;
}
__device__ __forceinline__ UnitIter iter_begin(const Args &p, const Sched &sc) {
    UnitIter w;
    w.left1 = sc.n1;
    if (sc.n1 > 0) {
        w.a = sc.c;
        w.hh = p.hh0;
        w.p6t = 0;
        w.r1 = true;
    } else {
        iter_region2(p, sc, w);
    }
    return w;
}
__device__ __forceinline__ void iter_next(const Args &p, const Sched &sc, UnitIter &w) {
    if (++w.p6t == p.n_p6t) {
        w.p6t = 0;
        if (++w.hh == p.hh0 + p.nhh) {
            w.hh = p.hh0;
            w.a += w.r1 ? sc.G : 1;
        }
    }
    if (w.r1 && --w.left1 == 0) iter_region2(p, sc, w);
}
// ring position: stage index and the parity of the current round
struct Ring {
    int s = 0;
    unsigned ph = 0;
    __device__ __forceinline__ void next(int S) {
        if (++s == S) {
            s = 0;
            ph ^= 1u;
        }
    }
};

// development instrumentation: cycles a role's lane 0 spends in each wait site (p.prof != nullptr)
#define TWAIT(site, bar, par)                                                   \
    do {                                                                        \
        if (p.prof) {                                                           \
            const long long t0_ = clock64();                                    \
            mbar_wait_sleep(bar, par);                                          \
            if (lane == 0) atomicAdd(p.prof + (site), (unsigned long long)(clock64() - t0_)); \
        } else {                                                                \
            mbar_wait_sleep(bar, par);                                          \
        }                                                                       \
    } while (0)

// warps: 0 v2-tile producer (TMA), 1 MMA issuer, 2 TMEM owner, 3 idle, 4..4+NEPI-1 epilogue
// (NGRP groups of four warps; warp % 4 = TMEM lane quarter; group g takes units u % NGRP == g)
template <int SP6>  // compile-time t3 column (p6) stride P5*P4 in elements, 0 = runtime
__global__ void __launch_bounds__(NTHREADS, 1)
    ccsd_tc_kernel(const float *__restrict__ t2, float *__restrict__ t3, const __grid_constant__ CUtensorMap mV,
                   const __grid_constant__ CUtensorMap mVlo, const __grid_constant__ CUtensorMap mX, const Args p) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    // align by pointer arithmetic on the shared array (an integer round trip would make every
    // access through `smem` a generic-address access)
    unsigned char *smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    // layout: V ring [SV] {hi [nkb], lo [nkb]}, t3 tiles [NGRP][XB], barriers
    unsigned char *vring = smem;
    unsigned char *xring = vring + (size_t)p.SV * p.v_stage;
    uint64_t *xbar = reinterpret_cast<uint64_t *>(xring + (size_t)NGRP * p.XB * p.x_stage);  // [NGRP][XSMAX]
    uint64_t *vfull = xbar + XSMAX * NGRP;
    uint64_t *vempty = vfull + p.SV;
    uint64_t *dfull = vempty + p.SV;
    uint64_t *dempty = dfull + 4;
    uint64_t *afull = dempty + 4;
    uint64_t *aempty = afull + 1;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(aempty + 1);
    const Sched sc = sched_of(p, (int)blockIdx.x, (int)gridDim.x);

    if (tid == 0) {
        for (int s = 0; s < p.SV; s++) {
            mbar_init(vfull + s, 1);
            mbar_init(vempty + s, 1);
        }
        for (int b = 0; b < 4; b++) {
            mbar_init(dfull + b, 1);
            mbar_init(dempty + b, 4);
        }
        for (int b = 0; b < XSMAX * NGRP; b++) mbar_init(xbar + b, 1);
        mbar_init(afull, 4);  // the owning epilogue group writes A into TMEM
        mbar_init(aempty, 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&mV)) : "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&mVlo)) : "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&mX)) : "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(su32(tmem_slot)),
                     "r"(512)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::: "memory");
    }
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {  // ------------------------------------ v2 tile producer (L2-resident)
            UnitIter w = iter_begin(p, sc);
            Ring r;
            for (int64_t u = 0; u < sc.n; u++, iter_next(p, sc, w), r.next(p.SV)) {
                if (u >= p.SV) TWAIT(0, vempty + r.s, r.ph ^ 1u);
                unsigned char *st = vring + (size_t)r.s * p.v_stage;
                if (p.dbg & 4) { mbar_arrive(vfull + r.s); continue; }
                mbar_expect_tx(vfull + r.s, p.v_stage);
                const int vrow = v_row(p, w.hh, w.p6t);
                for (int kb = 0; kb < p.nkb; kb++) {
                    tma_2d<1>(st + kb * p.v_kb_bytes, &mV, kb * 32, vrow, su32(vfull + r.s));
                    tma_2d<1>(st + (p.nkb + kb) * p.v_kb_bytes, &mVlo, kb * 32, vrow, su32(vfull + r.s));
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {  // ------------------------------------------------ MMA issuer
            const uint32_t ID = idesc(p.NV, 1, true);  // M = 128, N = NV = Th2 * Tp6, A and B K-major
            const long long tmma = p.prof ? clock64() : 0;
            int a_prev = -1, na = 0;
            UnitIter w = iter_begin(p, sc);
            Ring rv, rd;
            for (int64_t u = 0; u < sc.n; u++, iter_next(p, sc, w), rv.next(p.SV), rd.next(p.NB)) {
                if (w.a != a_prev) {
                    if (na > 0) mma_commit<1>(aempty);  // fires when every MMA on the old A is done
                    mbar_wait_sleep(afull, (unsigned)(na & 1));
                    a_prev = w.a;
                    na++;
                }
                if (u >= p.NB) TWAIT(1, dempty + rd.s, rd.ph ^ 1u);
                TWAIT(2, vfull + rv.s, rv.ph);
                fence_after();
                unsigned char *st = vring + (size_t)rv.s * p.v_stage;
                const uint32_t d = tmem + (uint32_t)(rd.s * p.bstride);
                const uint64_t vh0 = desc_sw128(st, 16u, 1024u), vl0 = desc_sw128(st + p.nkb * p.v_kb_bytes, 16u, 1024u);
                bool first = true;
                for (int k8 = 0; k8 < (p.dbg & 1 ? 0 : p.nks); k8++) {
                    // descriptor start address advances by (kb * v_kb_bytes + ks * 32) >> 4
                    const uint64_t off = (uint64_t)(((k8 >> 2) * p.v_kb_bytes + (k8 & 3) * 32) >> 4);
                    const uint32_t ah = tmem + (uint32_t)(p.a_col + 16 * k8), al = ah + 8;
                    mma_ts(d, ah, vh0 + off, ID, first ? 0u : 1u);
                    mma_ts(d, ah, vl0 + off, ID, 1u);
                    mma_ts(d, al, vh0 + off, ID, 1u);
                    first = false;
                }
                mma_commit<1>(dfull + rd.s);
                mma_commit<1>(vempty + rv.s);
            }
            if (p.prof) atomicAdd(p.prof + 6, (unsigned long long)(clock64() - tmma));
        }
    } else if (warp >= 4) {  // ------------------------------------------------ epilogue
        // Group g owns the units u = g, g + NGRP, ...  Its t3 tiles come from HBM by TMA into XB
        // group-private shared buffers, the next owned unit's tile being requested before the
        // current one is processed, so the HBM latency is hidden behind a whole unit; the updated
        // values go straight back to global memory (row m = (h1l, p5l, p4l): with Tp4 = P4 a warp's
        // 32 rows are 128 contiguous bytes, one coalesced streaming store per column).
        const int q = warp & 3, g = (warp - 4) >> 2, m = q * 32 + lane;
        const int Mrows = p.Th1 * p.Tp5 * p.Tp4;
        const int p4l = m % p.Tp4, p5l = (m / p.Tp4) % p.Tp5, h1l = m / (p.Tp4 * p.Tp5);
        const bool live = m < Mrows;
        const uint32_t trow = tmem + ((uint32_t)(q * 32) << 16);
        const int sp6 = SP6 > 0 ? SP6 : p.P5 * p.P4;
        const int64_t s_h1 = (int64_t)p.P6 * sp6, s_hh = p.H1 * s_h1;
        const int xstep = p.Tp5 * p.Tp4;                                 // smem column (p6) stride
        const int xrow0 = h1l * p.Tp6 * xstep + p5l * p.Tp4 + p4l;       // smem offset of row m
        const int xh2 = p.Th1 * p.Tp6 * xstep;                           // smem stride of h2l
        const int xslice = p.Th1 * p.p6s * xstep;                        // smem floats per slice
        const int xrow0s = h1l * p.p6s * xstep + p5l * p.Tp4 + p4l;      // row m inside a slice
        unsigned char *xbuf = xring + (size_t)g * p.XB * p.x_stage;
        uint64_t *xb = xbar + XSMAX * g;
        const bool leader = q == 0 && lane == 0;
        const uint64_t pol = policy_evict_first();  // t3 is touched once: keep v2 / t2 in L2
        auto fetch = [&](const UnitIter &wn, int buf) {  // t3 tile of unit wn -> xbuf[buf]
            int h1_0, p5_0, p4_0, c[5];
            a_coords(p, wn.a, h1_0, p5_0, p4_0);
            x_coords(p, wn.hh, wn.p6t, h1_0, p5_0, p4_0, c);
            if (p.XS) {  // XS slices (h2 plane q / sph, p6 part q % sph), barriers xb[0 .. XS-1]
                const int sb = p.x_bytes / p.XS;
                for (int q = 0; q < p.XS; q++) {
                    mbar_expect_tx(xb + q, sb);
                    tma_5d_hint(xbuf + (size_t)q * sb, &mX, c[0], c[1] + (q % p.sph) * p.p6s, c[2], c[3] + q / p.sph,
                                c[4], xb + q, pol);
                }
                return;
            }
            mbar_expect_tx(xb + buf, p.x_bytes);
            tma_5d_hint(xbuf + (size_t)buf * p.x_stage, &mX, c[0], c[1], c[2], c[3], c[4], xb + buf, pol);
        };
        auto fetch_slice = [&](const UnitIter &wn, int q) {  // slice q of unit wn -> its part of xbuf
            int h1_0, p5_0, p4_0, c[5];
            a_coords(p, wn.a, h1_0, p5_0, p4_0);
            x_coords(p, wn.hh, wn.p6t, h1_0, p5_0, p4_0, c);
            const int sb = p.x_bytes / p.XS;
            mbar_expect_tx(xb + q, sb);
            tma_5d_hint(xbuf + (size_t)q * sb, &mX, c[0], c[1] + (q % p.sph) * p.p6s, c[2], c[3] + q / p.sph, c[4],
                        xb + q, pol);
        };
        UnitIter w = iter_begin(p, sc), wn = w;  // wn: this group's next unit to prefetch
        for (int i = 0; i < g && i < sc.n; i++) iter_next(p, sc, wn);
        int64_t un = g;  // unit index of wn
        int a_prev = -1, na = 0, own = g, k = 0;  // own: units until this group's next unit; k: owned count
        bool rin = false;
        int64_t rowoff = 0;  // t3 offset of row m for hh = 0, p6 = 0
        // XB = 2: the first owned tile now; XS: its two slices now; XB = 1: at unit start
        if ((p.XB == 2 || p.XS) && leader && !(p.dbg & 2) && un < sc.n) fetch(wn, 0);
        Ring rd;
        for (int64_t u = 0; u < sc.n; u++, iter_next(p, sc, w), rd.next(p.NB), own--) {
            const bool mine = own == 0;
            if (mine) own = NGRP;
            if (w.a != a_prev) {  // new A tile: row coordinates; the owning group writes A into TMEM
                int h1_0, p5_0, p4_0;
                a_coords(p, w.a, h1_0, p5_0, p4_0);
                const int h1 = h1_0 + h1l, p5 = p5_0 + p5l, p4 = p4_0 + p4l;
                rin = live && h1 < p.H1 && p5 < p.P5 && p4 < p.P4;
                rowoff = (int64_t)h1 * s_h1 + (int64_t)p5 * p.P4 + p4;
                if (mine) {
                    const float *src = t2 + (((int64_t)p4 * p.P5 + p5) * p.H1 + h1);
                    const int64_t hstride = (int64_t)p.P4 * p.P5 * p.H1;
                    if (na > 0) mbar_wait_sleep(aempty, (unsigned)((na - 1) & 1));  // MMAs on the old A are done
                    for (int k8 = 0; k8 < p.nks; k8++) {
                        uint32_t hi[8], lo[8];
#pragma unroll
                        for (int c = 0; c < 8; c++) {
                            const int h7 = 8 * k8 + c;
                            const float x = (rin && h7 < p.H7) ? __ldg(src + h7 * hstride) : 0.f;
                            hi[c] = __float_as_uint(x);
                            lo[c] = __float_as_uint(lo_of(x));
                        }
                        tmem_st8(trow + (uint32_t)(p.a_col + 16 * k8), hi);
                        tmem_st8(trow + (uint32_t)(p.a_col + 16 * k8 + 8), lo);
                    }
                    wait_st();
                    fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(afull);
                }
                a_prev = w.a;
                na++;
            }
            if (!mine) continue;
            const int buf = p.XB == 2 ? (k & 1) : 0;
            const unsigned xph = (unsigned)((p.XB == 2 ? (k >> 1) : k) & 1);
            // next owned unit: its buffer was last read for unit k - 1 (XB = 2) -- the group barrier
            // orders those reads before the TMA overwrites it; XB = 1 fetches the current unit here
            for (int i = 0; i < NGRP && un < sc.n; i++, un++) iter_next(p, sc, wn);
            if (!p.XS) {
                named_bar(1 + g, 128);
                if (p.XB == 2) {
                    if (leader && !(p.dbg & 2) && un < sc.n) fetch(wn, buf ^ 1);
                } else if (leader && !(p.dbg & 2)) {
                    fetch(w, 0);
                }
            }
            // columns of this unit: hh = hhb + h2l (h2l < nh valid), p6 = p6b + c6 (c6 < np6 valid)
            int hhb, nh;
            if (p.Th2 == 1) {
                hhb = w.hh;
                nh = 1;
            } else {
                const int h3 = w.hh / p.n_h2t, h2_0 = (w.hh - h3 * p.n_h2t) * p.Th2;
                hhb = h3 * p.H2 + h2_0;
                nh = min(p.Th2, p.H2 - h2_0);
            }
            const int p6b = w.p6t * p.Tp6, np6 = min(p.Tp6, p.P6 - p6b);
            float *const rowp = t3 + rowoff + (int64_t)hhb * s_hh + (int64_t)p6b * sp6;
            const float *xs = reinterpret_cast<const float *>(xbuf + (size_t)buf * p.x_stage) + xrow0;
            const float *xsl = reinterpret_cast<const float *>(xbuf) + xrow0s;  // slices (XB = 1)
            const bool io = rin && !(p.dbg & 2);
            if (!(p.dbg & 2) && !p.XS) TWAIT(7, xb + buf, xph);
            if (p.prof && leader) atomicAdd(p.prof + 5, 1ull);
            TWAIT(3, dfull + rd.s, rd.ph);
            const long long tproc = p.prof ? clock64() : 0;
            fence_after();
            // chunks of 16 columns (Tp6 % 16 == 0: never two h2 in a chunk), walked without divisions
            constexpr int CH = 16;
            int h2l = 0, c6 = 0, q = 0, cq = 0;  // q: slice of this chunk, cq: column within the slice
            for (int c0 = 0; c0 < p.NV; c0 += CH) {
                if (p.XS && cq == 0) {  // a new slice: its t3 rows have landed (slice q, phase of unit k)
                    if (q >= 1) {  // slice q-1 fully read by the group: request the next owned unit's slice q-1
                        named_bar(1 + g, 128);
                        if (leader && !(p.dbg & 2) && un < sc.n) fetch_slice(wn, q - 1);
                    }
                    if (!(p.dbg & 2)) TWAIT(7, xb + q, (unsigned)(k & 1));
                }
                uint32_t v[CH];
                tmem_ld8(trow + (uint32_t)(rd.s * p.bstride + c0), *reinterpret_cast<uint32_t(*)[8]>(v));
                tmem_ld8(trow + (uint32_t)(rd.s * p.bstride + c0 + 8), *reinterpret_cast<uint32_t(*)[8]>(v + 8));
                // slice layout [q][h1l][p6 within the slice][(p5, p4)]; without slices q = h2l, p6s = Tp6
                const float *xc = p.XS ? xsl + q * xslice + cq * xstep : xs + h2l * xh2 + c6 * xstep;
                float x[CH];  // rows m >= Th1*Tp5*Tp4 lie outside the tile (and possibly the window)
#pragma unroll
                for (int c = 0; c < CH; c++) x[c] = live ? xc[c * xstep] : 0.f;
                wait_ld();
                const int nok = (io && h2l < nh) ? min(CH, np6 - c6) : 0;
                float *gp = rowp + (int64_t)h2l * s_hh + (int64_t)c6 * sp6;
                if (nok == CH) {
#pragma unroll
                    for (int c = 0; c < CH; c++) __stcs(gp + c * sp6, x[c] - __uint_as_float(v[c]));
                } else {
#pragma unroll
                    for (int c = 0; c < CH; c++)
                        if (c < nok) __stcs(gp + c * sp6, x[c] - __uint_as_float(v[c]));
                }
                c6 += CH;
                if (c6 == p.Tp6) { c6 = 0; h2l++; }
                cq += CH;
                if (cq == p.p6s) { cq = 0; q++; }
            }
            if (p.XS) {  // the last slice read: request the next owned unit's last slice
                named_bar(1 + g, 128);
                if (leader && !(p.dbg & 2) && un < sc.n) fetch_slice(wn, p.XS - 1);
            }
            fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(dempty + rd.s);
            if (p.prof && leader) atomicAdd(p.prof + 4, (unsigned long long)(clock64() - tproc));
            k++;
        }
    }
    fence_before();
    __syncthreads();
    if (warp == 2) {
        fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(512) : "memory");
    }
}

// v2lo = lo(v2)  (raw-hi split: v2 itself is the hi half)
__global__ void prep_kernel(const float *__restrict__ v2, float *__restrict__ v2_lo, int64_t n_v2) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n_v2; e += stride) v2_lo[e] = lo_of(v2[e]);
}

// n-D fp32 tensor map, dims/strides innermost first (strides in bytes for dims 1..n-1)
static bool make_map_nd(CUtensorMap *m, const float *base, int rank, const uint64_t *dims, const uint64_t *strides,
                        const uint32_t *box, CUtensorMapSwizzle sw) {
    EncodeTiled enc = encode_fn();
    if (!enc) return false;
    cuuint64_t d[5], st[4];
    cuuint32_t b[5], es[5];
    for (int i = 0; i < rank; i++) {
        d[i] = dims[i];
        b[i] = box[i];
        es[i] = 1;
        if (i > 0) st[i - 1] = strides[i - 1];
    }
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, (cuuint32_t)rank, const_cast<float *>(base), d, st, b, es,
               CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace ccsdtc

namespace {
struct CcsdTcPlan {
    bool ok = false;
    ccsdtc::Args a{};
    int smem = 0;
};

CcsdTcPlan plan_ccsd_tc(const int64_t *dims, const int64_t *tiles) {
    CcsdTcPlan pl;
    int64_t T[7];
    for (int i = 0; i < 7; i++) T[i] = std::min(tiles[i], dims[i]);
    const int64_t H3 = dims[0], H2 = dims[1], H1 = dims[2], P6 = dims[3], P5 = dims[4], P4 = dims[5], H7 = dims[6];
    if (T[0] != 1 || T[6] < H7) return pl;  // one h3 per unit, whole h7 reduction
    // Th2 > 1: Th2 consecutive h2 per unit (MMA N = Th2 * P6: their v2 rows are contiguous)
    // and whole p4 (the t3 tile's TMA box flattens (p5, p4))
    if (T[1] > 1 && (T[3] != P6 || T[5] != P4 || T[1] * P6 > 256 || (T[1] * P6) % 16)) return pl;
    if (H7 > 64 || (H7 % 4) || (P4 % 4) || (T[5] % 4)) return pl;  // 16-byte TMA strides / boxes
    if (T[2] * T[4] * T[5] > ccsdtc::MROWS || (T[3] % 16) || T[3] > 256) return pl;
    if (H3 * H2 > INT32_MAX || H3 * H2 * P6 > INT32_MAX || H1 * P5 * P4 * H7 > INT32_MAX) return pl;
    ccsdtc::Args &a = pl.a;
    a.H3 = (int)H3; a.H2 = (int)H2; a.H1 = (int)H1; a.P6 = (int)P6; a.P5 = (int)P5; a.P4 = (int)P4; a.H7 = (int)H7;
    a.Th1 = (int)T[2]; a.Tp6 = (int)T[3]; a.Tp5 = (int)T[4]; a.Tp4 = (int)T[5];
    a.Th2 = (int)T[1]; a.n_h2t = (int)((H2 + a.Th2 - 1) / a.Th2); a.NV = a.Th2 * a.Tp6;
    a.n_h1t = (int)((H1 + a.Th1 - 1) / a.Th1); a.n_p5t = (int)((P5 + a.Tp5 - 1) / a.Tp5);
    a.n_p4t = (int)((P4 + a.Tp4 - 1) / a.Tp4); a.n_p6t = (int)((P6 + a.Tp6 - 1) / a.Tp6);
    a.nkb = (int)((H7 + 31) / 32);
    static const int order_env = getenv("EATSS_CCSD_TC_ORDER") ? atoi(getenv("EATSS_CCSD_TC_ORDER")) : 1;
    a.order = order_env;
#ifdef EATSS_DEVTOOLS  // component switches for cost isolation (results then wrong): never in the product build
    a.dbg = getenv("EATSS_CCSD_TC_DBG") ? atoi(getenv("EATSS_CCSD_TC_DBG")) : 0;
#else
    a.dbg = 0;
#endif
    a.nks = (int)((H7 + 7) / 8);
    a.bstride = 32;
    while (a.bstride < a.NV) a.bstride *= 2;
    a.a_col = 384;                            // TMEM: D buffers in [0, 384), A in [384, 512)
    a.NB = std::min(4, 384 / a.bstride);
    if (a.NB < 1) return pl;
    a.v_kb_bytes = a.NV * 128;
    a.v_stage = 2 * a.nkb * a.v_kb_bytes;
    a.x_bytes = a.Th2 * a.Th1 * a.Tp6 * a.Tp5 * a.Tp4 * 4;
    a.x_stage = (a.x_bytes + 1023) / 1024 * 1024;
    const int fixed = 1024 /*align*/ + 512 /*barriers*/;
    const int budget = 232448 - fixed;
    a.XB = 2;
    if (budget - ccsdtc::NGRP * a.XB * a.x_stage < 3 * a.v_stage) a.XB = 1;  // keep >= 3 v2 stages if possible
    static const int xb_env = getenv("EATSS_CCSD_TC_XB") ? atoi(getenv("EATSS_CCSD_TC_XB")) : 0;  // development
    if (xb_env > 0) a.XB = std::min(2, xb_env);
    a.SV = std::min(6, (budget - ccsdtc::NGRP * a.XB * a.x_stage) / a.v_stage);
    // t3 slices (XB = 1, Th2 > 1 layout): one per h2 plane by default; finer (h2 plane, p6 part of >= 16 columns)
    // slices measured slower at dims 48 (6 slices 24.2 ms, 2 slices 19.0-20.1 ms, none 22.0 ms:
    // profiles/r02/experiments/gpu41_ccsd_slices.log); EATSS_CCSD_TC_SLICES = 0 / XS overrides (development)
    static const int xs_env = getenv("EATSS_CCSD_TC_SLICES") ? atoi(getenv("EATSS_CCSD_TC_SLICES")) : -1;
    a.XS = 0; a.sph = 1; a.p6s = a.Tp6;
    if (a.XB == 1 && a.Th2 > 1 && xs_env != 0) {
        for (int sph = xs_env > 0 ? a.Tp6 / 16 : 1; sph >= 1; sph--) {
            const int xs = a.Th2 * sph;
            if (a.Tp6 % sph || (a.Tp6 / sph) % 16 || xs > ccsdtc::XSMAX) continue;
            if (xs_env > 0 && xs != xs_env) continue;
            a.XS = xs; a.sph = sph; a.p6s = a.Tp6 / sph;
            break;
        }
    }
    static const int sv_env = getenv("EATSS_CCSD_TC_VSTAGES") ? atoi(getenv("EATSS_CCSD_TC_VSTAGES")) : 0;
    if (sv_env > 0) a.SV = std::min(a.SV, sv_env);
    if (a.SV < 2) return pl;
    pl.smem = fixed + a.SV * a.v_stage + ccsdtc::NGRP * a.XB * a.x_stage;
    pl.ok = true;
    return pl;
}
}  // namespace

bool ccsd_tc_applicable(const int64_t *dims, const int64_t *tiles) {
    return plan_ccsd_tc(dims, tiles).ok && tcm::encode_fn() != nullptr;
}

size_t ccsd_tc_ws_floats(const int64_t *dims) {  // v2's tf32 lo half (descriptor-owned scratch)
    return (size_t)(dims[0] * dims[1] * dims[3] * dims[6] + 64);
}

cudaError_t launch_ccsd_tc(float *t3, const float *t2, const float *v2, const int64_t *dims, const int64_t *tiles,
                           int64_t h3_begin, int64_t h3_count, float *ws, size_t ws_floats, cudaStream_t s,
                           cudaEvent_t *ev) {
    CcsdTcPlan pl = plan_ccsd_tc(dims, tiles);
    if (!pl.ok || !tcm::encode_fn()) return cudaErrorNotSupported;
    ccsdtc::Args a = pl.a;
    const int64_t H2 = dims[1], H1 = dims[2], P6 = dims[3], P5 = dims[4], P4 = dims[5], H7 = dims[6];
    a.hh0 = (int)(h3_begin * (a.Th2 == 1 ? H2 : a.n_h2t));
    a.nhh = (int)(h3_count * (a.Th2 == 1 ? H2 : a.n_h2t));
    a.units = (int64_t)a.n_h1t * a.n_p5t * a.n_p4t * a.nhh * a.n_p6t;
    if (a.units == 0) return cudaSuccess;
    const int64_t n_v2 = (int64_t)a.H3 * H2 * P6 * H7;
    float *v2_lo = ws;
    if (!v2_lo || ws_floats < (size_t)(n_v2 + 64)) return cudaErrorInvalidValue;
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    ccsdtc::prep_kernel<<<nsm * 4, 256, 0, s>>>(v2, v2_lo, n_v2);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    CUtensorMap mV, mVlo;
    // V: v2 as [(h3,h2,p6)][h7], box {32, NV}, SWIZZLE_128B (K-major UMMA operand)
    const uint64_t vdims[2] = {(uint64_t)H7, (uint64_t)((int64_t)a.H3 * H2 * P6)};
    const uint64_t vstr[1] = {(uint64_t)H7 * 4};
    const uint32_t vbox[2] = {32, (uint32_t)a.NV};
    // X: t3 as [(h3,h2)][h1][p6][p5][p4], box {Tp4, Tp5, Tp6, Th1, 1}; Th2 > 1: ((p5,p4), p6, h1, h2, h3)
    uint64_t xdims[5] = {(uint64_t)P4, (uint64_t)P5, (uint64_t)P6, (uint64_t)H1, (uint64_t)((int64_t)a.H3 * H2)};
    uint64_t xstr[4] = {(uint64_t)P4 * 4, (uint64_t)(P5 * P4) * 4, (uint64_t)(P6 * P5 * P4) * 4,
                        (uint64_t)(H1 * P6 * P5 * P4) * 4};
    uint32_t xbox[5] = {(uint32_t)a.Tp4, (uint32_t)a.Tp5, (uint32_t)a.Tp6, (uint32_t)a.Th1, 1};
    if (a.Th2 > 1) {
        const uint64_t d2[5] = {(uint64_t)(P5 * P4), (uint64_t)P6, (uint64_t)H1, (uint64_t)H2, (uint64_t)a.H3};
        const uint64_t s2[4] = {(uint64_t)(P5 * P4) * 4, (uint64_t)(P6 * P5 * P4) * 4, (uint64_t)(H1 * P6 * P5 * P4) * 4,
                                (uint64_t)(H2 * H1 * P6 * P5 * P4) * 4};
        const uint32_t b2[5] = {(uint32_t)(a.Tp5 * a.Tp4), (uint32_t)(a.XS ? a.p6s : a.Tp6), (uint32_t)a.Th1,
                                (uint32_t)(a.XS ? 1 : a.Th2), 1};  // XS: one (h2, p6 part) slice per box
        for (int i = 0; i < 5; i++) { xdims[i] = d2[i]; xbox[i] = b2[i]; }
        for (int i = 0; i < 4; i++) xstr[i] = s2[i];
    }
    CUtensorMap mX;
    if (!ccsdtc::make_map_nd(&mV, v2, 2, vdims, vstr, vbox, CU_TENSOR_MAP_SWIZZLE_128B) ||
        !ccsdtc::make_map_nd(&mVlo, v2_lo, 2, vdims, vstr, vbox, CU_TENSOR_MAP_SWIZZLE_128B) ||
        !ccsdtc::make_map_nd(&mX, t3, 5, xdims, xstr, xbox, CU_TENSOR_MAP_SWIZZLE_NONE))
        return cudaErrorInvalidValue;
    static std::mutex mu;
    static int smem_set = -1;
    {
        std::lock_guard<std::mutex> lk(mu);
        if (smem_set < pl.smem) {
            e = cudaFuncSetAttribute(ccsdtc::ccsd_tc_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem);
            if (e == cudaSuccess)
                e = cudaFuncSetAttribute(ccsdtc::ccsd_tc_kernel<48 * 48>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         pl.smem);
            if (e != cudaSuccess) return e;
            smem_set = pl.smem;
        }
    }
    const int grid = (int)std::min<int64_t>(nsm, a.units);
    static unsigned long long *prof = nullptr;
    static const bool prof_on = getenv("EATSS_CCSD_TC_PROF") != nullptr;  // development: wait profile
    if (prof_on) {
        if (!prof) cudaMalloc(&prof, 16 * sizeof(unsigned long long));
        cudaMemsetAsync(prof, 0, 16 * sizeof(unsigned long long), s);
        a.prof = prof;
    }
    if (ev) cudaEventRecord(ev[0], s);
    if (a.P5 * a.P4 == 48 * 48)  // the BASELINE dims-48 stride: immediate-offset accesses
        ccsdtc::ccsd_tc_kernel<48 * 48><<<grid, ccsdtc::NTHREADS, pl.smem, s>>>(t2, t3, mV, mVlo, mX, a);
    else
        ccsdtc::ccsd_tc_kernel<0><<<grid, ccsdtc::NTHREADS, pl.smem, s>>>(t2, t3, mV, mVlo, mX, a);
    e = cudaGetLastError();
    if (a.prof) {  // development: per-site average cycles (per CTA role lane / per unit)
        unsigned long long h[16];
        cudaMemcpyAsync(h, prof, sizeof(h), cudaMemcpyDeviceToHost, s);
        cudaStreamSynchronize(s);
        const double units = (double)h[5];
        fprintf(stderr,
                "ccsd_tc prof: units %.0f | per unit: V wait vempty %.0f, MMA wait dempty %.0f, MMA wait vfull "
                "%.0f, EPI wait dfull %.0f, EPI process %.0f, EPI wait t3 %.0f | MMA loop per CTA %.0f cyc (%d CTAs)\n",
                units, h[0] / units, h[1] / units, h[2] / units, h[3] / units / 4, h[4] / units, h[7] / units / 4, h[6] / (double)grid,
                grid);
    }
    if (ev) cudaEventRecord(ev[1], s);
    return e;
}

}  // namespace eatss
