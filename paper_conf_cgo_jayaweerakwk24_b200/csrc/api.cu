// api.cu -- the C ABI of libeatss.so (include/eatss.h): descriptors, GPU
// parameters, launch plans and execution.  The tile model lives in model.cpp,
// the kernels in contract.cu / stencil.cu / ccsd.cu, energy in energy.cpp.
#include <cuda_runtime.h>

#include <algorithm>
#include <map>
#include <mutex>
#include <cstring>
#include <string>
#include <vector>

#include "contract.cuh"
#include "desc.hpp"

namespace eatss {

static thread_local std::string g_err;
void set_error(const std::string &m) { g_err = m; }
eatss_status fail(eatss_status s, const std::string &m) {
    g_err = m;
    return s;
}
static eatss_status cuda_fail(cudaError_t e, const char *where) {
    return fail(EATSS_E_CUDA, std::string(where) + ": " + cudaGetErrorName(e) + " (" +
                                  cudaGetErrorString(e) + ")");
}

// stencil.cu / ccsd.cu entry points
cudaError_t launch_jacobi2d_sweep(void *dst, const void *src, const void *bsrc, int64_t n, int64_t Ti,
                                  int64_t Tj, bool f64, int carveout, int32_t *counts, cudaStream_t s, int waf);
cudaError_t launch_interior_copy2d(void *dst, const void *src, int64_t n, bool f64, cudaStream_t s);
// stencil_untiled.cu: the untiled baseline (engine EATSS_ENGINE_UNTILED; tile vector ignored)
cudaError_t launch_jacobi2d_untiled(void *dst, const void *src, const void *bsrc, int64_t n, bool f64, cudaStream_t s);
cudaError_t launch_heat3d_untiled(void *dst, const void *src, int64_t n, bool f64, cudaStream_t s);
cudaError_t launch_heat3d_sweep(void *dst, const void *src, int64_t n, int64_t Ti, int64_t Tj,
                                int64_t Tk, bool f64, int carveout, int32_t *counts, cudaStream_t s, int waf);
int stencil_simt_x(bool heat, int64_t n, const int64_t *t, bool f64, int waf);
void stencil_plan_dims(bool heat, int64_t n, const int64_t *t, bool f64, int64_t *gx, int64_t *gy,
                       int *bx, int *by, int *vec);
cudaError_t launch_ccsd_d1(float *t3, const float *t2, const float *v2, const int64_t *dims,
                           const int64_t *tiles, int64_t h3_begin, int64_t h3_count, int carveout,
                           int32_t *counts, cudaStream_t s);
bool ccsd_tc_applicable(const int64_t *dims, const int64_t *tiles);
size_t ccsd_tc_ws_floats(const int64_t *dims);
cudaError_t launch_ccsd_tc(float *t3, const float *t2, const float *v2, const int64_t *dims, const int64_t *tiles,
                           int64_t h3_begin, int64_t h3_count, float *ws, size_t ws_floats, cudaStream_t s,
                           cudaEvent_t *ev);
void ccsd_plan_dims(const int64_t *dims, const int64_t *tiles, int64_t *gx, int64_t *gy, int *bx,
                    int *by, int *rm, int *rn, int *passes, int *smem);

// lowdim.cu entry points (mvt, atax, bicg, gemver)
struct LowdimArgs {
    const float *A;
    float *Aout;
    int64_t nx, ny;
    int Ti, Tj;
    float *rowout;
    const float *vr;
    float ar;
    float *colout;
    const float *vc;
    float ac;
    const float *u1, *v1, *u2, *v2;
};
cudaError_t launch_lowdim(const LowdimArgs &a, bool row, bool col, bool upd, cudaStream_t s, int64_t *launched);
cudaError_t launch_lowdim_axpy(float *out, const float *add, float scale, int64_t n, cudaStream_t s,
                               int64_t *launched);

// mttkrp.cu / conv2d.cu entry points (non-PolyBench 4-D kernels)
bool mttkrp_plan(const int64_t *dims, const int64_t *tiles, int64_t *gx, int64_t *gy, int64_t *gz, int *bx, int *by,
                 int *rm, int *smem, int *splits, int *sw_out = nullptr, int *ks_out = nullptr);
cudaError_t launch_mttkrp(float *A, const float *B, const float *C, const float *D, const int64_t *dims,
                          const int64_t *tiles, float *ws, int32_t *counts, cudaStream_t s, int64_t *launched);
bool mttkrp_tc_applicable(const int64_t *dims, const int64_t *tiles);
size_t mttkrp_tc_ws_floats(const int64_t *dims);
cudaError_t launch_mttkrp_tc(float *A, const float *B, const float *C, const float *D, const int64_t *dims, float *ws,
                             cudaStream_t s, cudaEvent_t *ev, int64_t *launched);
bool conv2d_plan(int64_t n, int64_t f, const int64_t *tiles, int64_t *gx, int64_t *gy, int *threads, int *smem,
                 int *rc, int *wc, int *groups, int *segs);
cudaError_t launch_conv2d(float *out, const float *inp, const float *W, int64_t n, int64_t f, const int64_t *tiles,
                          int32_t *counts, cudaStream_t s, int64_t *launched);

// ------------------------------------------------------------------ builtin nests
// Loop positions are bits: the model only needs which loops a subscript uses.
static Sub S(uint32_t iters, int off = 0) {
    Sub s;
    s.iters = iters;
    s.off = off;
    return s;
}
static Ref R(int array, std::vector<Sub> subs, bool write = false) {
    Ref r;
    r.array = array;
    r.subs = std::move(subs);
    r.write = write;
    return r;
}
static Nest N3(int64_t e0, int64_t e1, int64_t e2, bool p2, std::vector<Ref> refs) {
    Nest n;
    n.loops = {{e0, true}, {e1, true}, {e2, p2}};
    n.refs = std::move(refs);
    return n;
}

enum : uint32_t { I = 1u, J = 2u, K = 4u };

// gemm-like nest Out[i][j] (+)= In[i][k] * Ker[k][j]   (Fig. 4)
static Nest mm_nest(int64_t ni, int64_t nj, int64_t nk, int out, int in, int ker, bool out_read) {
    std::vector<Ref> refs{R(out, {S(I), S(J)}, true)};
    if (out_read) refs.push_back(R(out, {S(I), S(J)}));
    refs.push_back(R(in, {S(I), S(K)}));
    refs.push_back(R(ker, {S(K), S(J)}));
    return N3(ni, nj, nk, false, refs);
}

static eatss_status build(eatss_kernel_desc *d) {
    const auto &x = d->dims;
    switch (d->kind) {
        case EATSS_GEMM:  // C A B
            d->nests = {mm_nest(x[0], x[1], x[2], 0, 1, 2, true)};
            d->buffer_elems = {x[0] * x[1], x[0] * x[2], x[2] * x[1]};
            break;
        case EATSS_2MM:  // tmp A B C D ; dims ni nj nk nl
            d->nests = {mm_nest(x[0], x[1], x[2], 0, 1, 2, false), mm_nest(x[0], x[3], x[1], 4, 0, 3, true)};
            d->buffer_elems = {x[0] * x[1], x[0] * x[2], x[2] * x[1], x[1] * x[3], x[0] * x[3]};
            break;
        case EATSS_3MM:  // E A B F C D G ; dims ni nj nk nl nm
            d->nests = {mm_nest(x[0], x[1], x[2], 0, 1, 2, false), mm_nest(x[1], x[3], x[4], 3, 4, 5, false),
                        mm_nest(x[0], x[3], x[1], 6, 0, 3, false)};
            d->buffer_elems = {x[0] * x[1], x[0] * x[2], x[2] * x[1], x[1] * x[3],
                               x[1] * x[4], x[4] * x[3], x[0] * x[3]};
            break;
        case EATSS_SYRK: {  // C A ; dims (ni, nj) or (ni, nj, r0, rows): rows [r0, r0+rows) of C
            const int64_t rows = x.size() == 4 ? x[3] : x[0];
            d->nests = {N3(rows, x[0], x[1], false,
                           {R(0, {S(I), S(J)}, true), R(0, {S(I), S(J)}), R(1, {S(I), S(K)}), R(1, {S(J), S(K)})})};
            d->buffer_elems = {rows * x[0], x[0] * x[1]};
            break;
        }
        case EATSS_JACOBI2D: {  // A B ; dims n ; interior extent n-2, time loop excluded
            const int64_t m = x[0] - 2;
            Nest c, cp;
            c.loops = {{m, true}, {m, true}};
            c.refs = {R(1, {S(I), S(J)}, true), R(0, {S(I), S(J)}), R(0, {S(I), S(J, -1)}),
                      R(0, {S(I), S(J, 1)}), R(0, {S(I, 1), S(J)}), R(0, {S(I, -1), S(J)})};
            cp.loops = c.loops;
            cp.refs = {R(0, {S(I), S(J)}, true), R(1, {S(I), S(J)})};
            d->nests = {c, cp};
            d->buffer_elems = {x[0] * x[0], x[0] * x[0]};
            break;
        }
        case EATSS_HEAT3D: {  // A B ; dims n
            const int64_t m = x[0] - 2;
            auto sweep = [&](int dst, int src) {
                Nest n;
                n.loops = {{m, true}, {m, true}, {m, true}};
                n.refs = {R(dst, {S(I), S(J), S(K)}, true),
                          R(src, {S(I, 1), S(J), S(K)}), R(src, {S(I), S(J), S(K)}), R(src, {S(I, -1), S(J), S(K)}),
                          R(src, {S(I), S(J, 1), S(K)}), R(src, {S(I), S(J, -1), S(K)}),
                          R(src, {S(I), S(J), S(K, 1)}), R(src, {S(I), S(J), S(K, -1)})};
                return n;
            };
            d->nests = {sweep(1, 0), sweep(0, 1)};
            d->buffer_elems = {x[0] * x[0] * x[0], x[0] * x[0] * x[0]};
            break;
        }
        case EATSS_CCSD_T_D1: {  // t3 t2 v2 ; loops h3 h2 h1 p6 p5 p4 h7
            Nest n;
            for (int p = 0; p < 7; p++) n.loops.push_back({x[p], p != 6});
            const uint32_t h3 = 1, h2 = 2, h1 = 4, p6 = 8, p5 = 16, p4 = 32, h7 = 64;
            n.refs = {R(0, {S(h3), S(h2), S(h1), S(p6), S(p5), S(p4)}, true),
                      R(0, {S(h3), S(h2), S(h1), S(p6), S(p5), S(p4)}),
                      R(1, {S(h7), S(p4), S(p5), S(h1)}), R(2, {S(h3), S(h2), S(p6), S(h7)})};
            d->nests = {n};
            d->buffer_elems = {x[0] * x[1] * x[2] * x[3] * x[4] * x[5], x[6] * x[5] * x[4] * x[2],
                               x[0] * x[1] * x[3] * x[6]};
            break;
        }
        // low-dimensional PolyBench 3.2 kernels (reading R-N7): 2-deep nests
        // (i, j); a reduction loop is marked not parallel
        case EATSS_MVT: {  // x1 x2 y_1 y_2 A ; dims n
            const int64_t n = x[0];
            Nest a, b;
            a.loops = b.loops = {{n, true}, {n, false}};
            a.refs = {R(0, {S(I)}, true), R(0, {S(I)}), R(4, {S(I), S(J)}), R(2, {S(J)})};
            b.refs = {R(1, {S(I)}, true), R(1, {S(I)}), R(4, {S(J), S(I)}), R(3, {S(J)})};
            d->nests = {a, b};
            d->buffer_elems = {n, n, n, n, n * n};
            break;
        }
        case EATSS_ATAX: {  // y tmp A x ; dims (nx, ny)
            Nest a, b;
            a.loops = {{x[0], true}, {x[1], false}};
            a.refs = {R(1, {S(I)}, true), R(1, {S(I)}), R(2, {S(I), S(J)}), R(3, {S(J)})};
            b.loops = {{x[0], false}, {x[1], true}};
            b.refs = {R(0, {S(J)}, true), R(0, {S(J)}), R(2, {S(I), S(J)}), R(1, {S(I)})};
            d->nests = {a, b};
            d->buffer_elems = {x[1], x[0], x[0] * x[1], x[1]};
            break;
        }
        case EATSS_BICG: {  // s q A r p ; dims (nx, ny)
            Nest a, b;
            a.loops = {{x[0], false}, {x[1], true}};
            a.refs = {R(0, {S(J)}, true), R(0, {S(J)}), R(3, {S(I)}), R(2, {S(I), S(J)})};
            b.loops = {{x[0], true}, {x[1], false}};
            b.refs = {R(1, {S(I)}, true), R(1, {S(I)}), R(2, {S(I), S(J)}), R(4, {S(J)})};
            d->nests = {a, b};
            d->buffer_elems = {x[1], x[0], x[0] * x[1], x[0], x[1]};
            break;
        }
        case EATSS_GEMVER: {  // A x w u1 v1 u2 v2 y z ; dims n
            const int64_t n = x[0];
            Nest a, b, c, e;
            a.loops = {{n, true}, {n, true}};
            a.refs = {R(0, {S(I), S(J)}, true), R(0, {S(I), S(J)}), R(3, {S(I)}), R(4, {S(J)}), R(5, {S(I)}),
                      R(6, {S(J)})};
            b.loops = {{n, true}, {n, false}};
            b.refs = {R(1, {S(I)}, true), R(1, {S(I)}), R(0, {S(J), S(I)}), R(7, {S(J)})};
            c.loops = {{n, true}};
            c.refs = {R(1, {S(I)}, true), R(1, {S(I)}), R(8, {S(I)})};
            e.loops = {{n, true}, {n, false}};
            e.refs = {R(2, {S(I)}, true), R(2, {S(I)}), R(0, {S(I), S(J)}), R(1, {S(J)})};
            d->nests = {a, b, c, e};
            d->buffer_elems = {n * n, n, n, n, n, n, n, n, n};
            break;
        }
        // non-PolyBench 4-D kernels (readings R-N8, R-N9): reduction loops serial
        case EATSS_MTTKRP: {  // A B C D ; dims (ni, nj, nk, nl) ; loops i j k l
            Nest n;
            n.loops = {{x[0], true}, {x[1], true}, {x[2], false}, {x[3], false}};
            const uint32_t i = 1, j = 2, k = 4, l = 8;
            n.refs = {R(0, {S(i), S(j)}, true), R(0, {S(i), S(j)}), R(1, {S(i), S(k), S(l)}), R(2, {S(k), S(j)}),
                      R(3, {S(l), S(j)})};
            d->nests = {n};
            d->buffer_elems = {x[0] * x[1], x[0] * x[2] * x[3], x[2] * x[1], x[3] * x[1]};
            break;
        }
        case EATSS_CONV2D: {  // out inp W ; dims (n, f) ; loops i j p q over out[m][m], m = n - f + 1
            const int64_t m = x[0] - x[1] + 1;
            Nest n;
            n.loops = {{m, true}, {m, true}, {x[1], false}, {x[1], false}};
            const uint32_t i = 1, j = 2, p = 4, q = 8;
            n.refs = {R(0, {S(i), S(j)}, true), R(0, {S(i), S(j)}), R(1, {S(i | p), S(j | q)}), R(2, {S(p), S(q)})};
            d->nests = {n};
            d->buffer_elems = {m * m, x[0] * x[0], x[1] * x[1]};
            break;
        }
        default:
            return fail(EATSS_E_INVALID, "eatss_desc_builtin: unknown builtin");
    }
    d->num_buffers = (int)d->buffer_elems.size();
    return EATSS_OK;
}

// Library-owned scratch of a descriptor (grown on demand, on the current device).
static void free_ws(eatss_kernel_desc *d) {
    if (!d->ws) return;
    int cur = 0;
    cudaGetDevice(&cur);
    if (d->ws_dev >= 0 && d->ws_dev != cur) cudaSetDevice(d->ws_dev);  // free on the owning device
    cudaFree(d->ws);  // synchronises that device: no queued launch still uses the old scratch
    if (d->ws_dev >= 0 && d->ws_dev != cur) cudaSetDevice(cur);
    d->ws = nullptr;
    d->ws_bytes = 0;
}
static eatss_status ensure_ws(eatss_kernel_desc *d, size_t need) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (d->ws && d->ws_dev == dev && d->ws_bytes >= need) return EATSS_OK;
    free_ws(d);
    d->ws_bytes = 0;
    cudaError_t e = cudaMalloc(&d->ws, need);
    if (e != cudaSuccess) return cuda_fail(e, "eatss_run(workspace)");
    d->ws_bytes = need;
    d->ws_dev = dev;
    return EATSS_OK;
}

// Stream-ordered scratch of ONE run (tensor engines' split operands): allocated from a library-owned
// pool of the current device on the run's stream and freed on it after the run's launches, so runs on
// different streams, devices or host threads never share it and nothing synchronises (the pool keeps
// its memory: release threshold = max).
static cudaMemPool_t scratch_pool() {
    static std::mutex mu;
    static std::map<int, cudaMemPool_t> pools;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(mu);
    auto it = pools.find(dev);
    if (it != pools.end()) return it->second;
    cudaMemPoolProps props{};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t pool = nullptr;
    if (cudaMemPoolCreate(&pool, &props) != cudaSuccess) return nullptr;
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    pools[dev] = pool;
    return pool;
}
struct RunScratch {  // freed (stream-ordered) when the run's launches have been issued
    void *p = nullptr;
    size_t bytes = 0;
    cudaStream_t s = nullptr;
    cudaError_t alloc(size_t n, cudaStream_t st) {
        s = st;
        cudaMemPool_t pool = scratch_pool();
        if (!pool) return cudaErrorMemoryAllocation;
        cudaError_t e = cudaMallocFromPoolAsync(&p, n, pool, st);
        if (e == cudaSuccess) bytes = n;
        else p = nullptr;
        return e;
    }
    ~RunScratch() {
        if (p) cudaFreeAsync(p, s);
    }
};

// SIMT syrk: its transposed operand B(k, j) = A[j][k] is laid out as A^T once per run (a layout pass
// into the descriptor's workspace, ~2 x 64 MB of traffic at N = 4000) so the executor runs its
// non-transposed staged path; every element keeps the same k-ascending sum.  EATSS_SYRK_TRANSB=1
// keeps the strided transposed-operand path (for comparison).
static bool simt_untranspose(const eatss_kernel_desc *d) {
    static const bool off = [] {
        const char *e = getenv("EATSS_SYRK_TRANSB");
        return e && atoi(e) != 0;
    }();
    return d->kind == EATSS_SYRK && d->dtype == EATSS_F32 && d->exec.engine != EATSS_ENGINE_TENSOR &&
           d->exec.engine != EATSS_ENGINE_TENSOR_F16 && !off;
}
static void untranspose_nests(const eatss_kernel_desc *d, std::vector<ContractNest> &cn, const void *at) {
    for (auto &n : cn) {
        n.B = at;
        n.ldb = d->dims[0];  // A^T is nj x ni
        n.transB = false;
    }
}

static const int kDimsPerBuiltin[] = {3, 4, 5, 2, 1, 1, 7, 1, 2, 2, 1, 4, 2};

static bool is_lowdim(eatss_builtin k) {
    return k == EATSS_MVT || k == EATSS_ATAX || k == EATSS_BICG || k == EATSS_GEMVER;
}

// ------------------------------------------------------------------ execution helpers
static int smem_limit_bytes() {
    int dev = 0, v = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return 232448;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) return 232448;
    return v;
}

// The gemm-family nests of a program as executor arguments.
static std::vector<ContractNest> contraction_nests(const eatss_kernel_desc *d, void *const *b) {
    const auto &x = d->dims;
    const bool f64 = d->dtype == EATSS_F64;
    auto mk = [&](int64_t M, int64_t Nn, int64_t Kk, const void *A, int64_t lda, const void *B, int64_t ldb,
                  bool tB, void *C, int64_t ldc, double al, double be, bool z) {
        ContractNest n;
        n.M = M; n.N = Nn; n.K = Kk; n.A = A; n.lda = lda; n.B = B; n.ldb = ldb; n.transB = tB;
        n.C = C; n.ldc = ldc; n.alpha = al; n.beta = be; n.init_zero = z; n.f64 = f64;
        return n;
    };
    std::vector<ContractNest> v;
    switch (d->kind) {
        case EATSS_GEMM:
            v.push_back(mk(x[0], x[1], x[2], b[1], x[2], b[2], x[1], false, b[0], x[1], d->alpha, d->beta, false));
            break;
        case EATSS_2MM:
            v.push_back(mk(x[0], x[1], x[2], b[1], x[2], b[2], x[1], false, b[0], x[1], d->alpha, 0.0, true));
            v.push_back(mk(x[0], x[3], x[1], b[0], x[1], b[3], x[3], false, b[4], x[3], 1.0, d->beta, false));
            break;
        case EATSS_3MM:
            v.push_back(mk(x[0], x[1], x[2], b[1], x[2], b[2], x[1], false, b[0], x[1], 1.0, 0.0, true));
            v.push_back(mk(x[1], x[3], x[4], b[4], x[4], b[5], x[3], false, b[3], x[3], 1.0, 0.0, true));
            v.push_back(mk(x[0], x[3], x[1], b[0], x[1], b[3], x[3], false, b[6], x[3], 1.0, 0.0, true));
            break;
        case EATSS_SYRK: {
            const int64_t r0 = x.size() == 4 ? x[2] : 0, rows = x.size() == 4 ? x[3] : x[0];
            const void *Ar = static_cast<const char *>(b[1]) + r0 * x[1] * (f64 ? 8 : 4);
            v.push_back(mk(rows, x[0], x[1], Ar, x[1], b[1], x[1], true, b[0], x[0], d->alpha, d->beta, false));
            break;
        }
        default:
            break;
    }
    return v;
}

static bool is_contraction(eatss_builtin k) {
    return k == EATSS_GEMM || k == EATSS_2MM || k == EATSS_3MM || k == EATSS_SYRK;
}

static eatss_status check_tiles(const eatss_kernel_desc *d, const int64_t *tiles) {
    if (!tiles) return fail(EATSS_E_INVALID, "tiles is null");
    const int L = eatss_desc_num_loops(d);
    for (int p = 0; p < L; p++)
        if (tiles[p] <= 0) return fail(EATSS_E_INVALID, "tile entries must be >= 1");
    return EATSS_OK;
}

static eatss_status check_bufs(const eatss_kernel_desc *d, void *const *b) {
    if (!b) return fail(EATSS_E_INVALID, "buffers is null");
    for (int i = 0; i < d->num_buffers; i++)
        if (!b[i] && d->buffer_elems[i] > 0) return fail(EATSS_E_INVALID, "buffer pointer is null");
    return EATSS_OK;
}

// The carve-out request of a descriptor's launches (sigma and exec.carveout_exact).
static int exec_cv(const eatss_kernel_desc *d) { return cv_make(d->exec.split_pct, d->exec.carveout_exact != 0); }

// Issue the stencil time loop on stream s (no graph).
static cudaError_t stencil_issue(const eatss_kernel_desc *d, const int64_t *t, void *const *b, cudaStream_t s) {
    const bool f64 = d->dtype == EATSS_F64;
    const int64_t n = d->dims[0];
    const int cv = exec_cv(d);
    cudaError_t e = cudaSuccess;
    if (n < 3) return cudaSuccess;
    const bool untiled = d->exec.engine == EATSS_ENGINE_UNTILED;
    if (d->kind == EATSS_JACOBI2D) {
        void *A = b[0], *B = b[1];
        for (int64_t step = 0; step < d->tsteps && e == cudaSuccess; step++) {
            void *dst = step % 2 == 0 ? B : A, *src = step % 2 == 0 ? A : B;
            e = untiled ? launch_jacobi2d_untiled(dst, src, A, n, f64, s)
                        : launch_jacobi2d_sweep(dst, src, A, n, t[0], t[1], f64, cv, nullptr, s, d->exec.warp_align);
        }
        if (e == cudaSuccess && d->tsteps > 0) {
            // the literal copy nest of the last step (both interiors end equal to X_T)
            if (d->tsteps % 2 == 1) e = launch_interior_copy2d(A, B, n, f64, s);
            else e = launch_interior_copy2d(B, A, n, f64, s);
        }
    } else {
        void *A = b[0], *B = b[1];
        for (int64_t step = 0; step < d->tsteps && e == cudaSuccess; step++) {
            e = untiled ? launch_heat3d_untiled(B, A, n, f64, s)
                        : launch_heat3d_sweep(B, A, n, t[0], t[1], t[2], f64, cv, nullptr, s, d->exec.warp_align);
            if (e == cudaSuccess)
                e = untiled ? launch_heat3d_untiled(A, B, n, f64, s)
                            : launch_heat3d_sweep(A, B, n, t[0], t[1], t[2], f64, cv, nullptr, s, d->exec.warp_align);
        }
    }
    return e;
}

static eatss_status stencil_run(eatss_kernel_desc *d, const int64_t *t, void *const *b, cudaStream_t s) {
    if (!d->exec.use_graph || d->tsteps <= 1) {
        take_carveout();
        cudaError_t e = stencil_issue(d, t, b, s);
        d->graph_cv = take_carveout();
        return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_run(stencil)");
    }
    GraphKey key;
    key.tiles.assign(t, t + eatss_desc_num_loops(d));
    key.tiles.push_back(d->exec.engine);  // a tiled and an untiled time loop are different graphs
    key.tiles.push_back(d->exec.split_pct);  // the carve-out is captured with each launch
    key.tiles.push_back(d->exec.carveout_exact);
    key.tiles.push_back(d->exec.warp_align);  // the lane layout is a kernel argument of every captured sweep
    int gdev = 0;
    cudaGetDevice(&gdev);
    key.tiles.push_back(gdev);  // a graph is instantiated for one device
    for (int i = 0; i < d->num_buffers; i++) key.bufs.push_back((uintptr_t)b[i]);
    key.stream = 0;  // graphs are stream-independent; launched on the caller's stream
    cudaGraphExec_t exec = nullptr;
    {
        std::lock_guard<std::mutex> lk(d->graph_mu);
        auto it = d->graphs.find(key);
        if (it != d->graphs.end()) {
            exec = (cudaGraphExec_t)it->second;
            d->graph_cv = d->graph_cvs[key];
        }
    }
    if (!exec) {
        // set function attributes outside capture by issuing nothing: attributes are
        // set inside the launchers, which is legal during thread-local capture.
        cudaStream_t cs;
        cudaError_t e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
        if (e != cudaSuccess) return cuda_fail(e, "cudaStreamCreate");
        e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
        if (e != cudaSuccess) {
            cudaStreamDestroy(cs);
            return cuda_fail(e, "cudaStreamBeginCapture");
        }
        take_carveout();
        cudaError_t ei = stencil_issue(d, t, b, cs);
        const int cap_cv = take_carveout();
        cudaGraph_t g = nullptr;
        e = cudaStreamEndCapture(cs, &g);
        cudaStreamDestroy(cs);
        if (ei != cudaSuccess) {
            if (g) cudaGraphDestroy(g);
            return cuda_fail(ei, "stencil capture");
        }
        if (e != cudaSuccess) return cuda_fail(e, "cudaStreamEndCapture");
        e = cudaGraphInstantiate(&exec, g, 0);
        cudaGraphDestroy(g);
        if (e != cudaSuccess) return cuda_fail(e, "cudaGraphInstantiate");
        std::lock_guard<std::mutex> lk(d->graph_mu);
        d->graphs[key] = exec;
        d->graph_cvs[key] = cap_cv;
        d->graph_cv = cap_cv;
    }
    cudaError_t e = cudaGraphLaunch(exec, s);
    return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "cudaGraphLaunch");
}

}  // namespace eatss

using namespace eatss;

eatss_kernel_desc::~eatss_kernel_desc() {
    for (auto &kv : graphs) cudaGraphExecDestroy((cudaGraphExec_t)kv.second);
    for (void *e : kev) cudaEventDestroy((cudaEvent_t)e);
    for (void *b : hbuf) cudaFree(b);
    for (void *e : hev) cudaEventDestroy((cudaEvent_t)e);
    for (void *st : hstream)
        if (st) cudaStreamDestroy((cudaStream_t)st);
    free_ws(this);
}

// exec.time_kernels: a {start, stop} event pair per nest on the current device (nullptr if off)
static cudaEvent_t *kernel_events(eatss_kernel_desc *d, int nest) {
    if (!d->exec.time_kernels) return nullptr;
    int dev = 0;
    cudaGetDevice(&dev);
    if (d->kev_dev != dev) {
        for (void *e : d->kev) cudaEventDestroy((cudaEvent_t)e);
        d->kev.clear();
        d->kev_dev = dev;
    }
    while ((int)d->kev.size() < 2 * (int)d->nests.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
        d->kev.push_back(e);
    }
    d->kev_valid = (int)d->nests.size();
    return reinterpret_cast<cudaEvent_t *>(&d->kev[2 * nest]);
}

extern "C" {

const char *eatss_last_error(void) { return g_err.c_str(); }
int eatss_abi_version(void) { return EATSS_ABI_VERSION; }

eatss_status eatss_desc_builtin(eatss_builtin k, const int64_t *dims, int ndims, eatss_dtype dt,
                                int64_t tsteps, eatss_kernel_desc **out) {
    if (!out) return fail(EATSS_E_INVALID, "eatss_desc_builtin: out is null");
    *out = nullptr;
    if ((int)k < 0 || (int)k > (int)EATSS_CONV2D) return fail(EATSS_E_INVALID, "eatss_desc_builtin: bad builtin");
    if (dt != EATSS_F32 && dt != EATSS_F64) return fail(EATSS_E_INVALID, "eatss_desc_builtin: bad dtype");
    if (!dims) return fail(EATSS_E_INVALID, "eatss_desc_builtin: dims is null");
    const int want = kDimsPerBuiltin[k];
    std::vector<int64_t> dv;
    if (k == EATSS_CCSD_T_D1 && ndims == 1) dv.assign(7, dims[0]);
    else if (ndims == want || (k == EATSS_SYRK && ndims == 4)) dv.assign(dims, dims + ndims);
    else return fail(EATSS_E_INVALID, "eatss_desc_builtin: wrong number of dims");
    for (size_t i = 0; i < dv.size(); i++)
        if (dv[i] <= 0 && !(k == EATSS_SYRK && i == 2 && dv[i] == 0))
            return fail(EATSS_E_INVALID, "eatss_desc_builtin: dims must be >= 1");
    if (k == EATSS_SYRK && dv.size() == 4 && dv[2] + dv[3] > dv[0])
        return fail(EATSS_E_INVALID, "eatss_desc_builtin: syrk row block exceeds ni");
    if ((k == EATSS_JACOBI2D || k == EATSS_HEAT3D) && (dv[0] < 3 || tsteps < 0))
        return fail(EATSS_E_INVALID, "eatss_desc_builtin: stencils need n >= 3 and tsteps >= 0");
    if (k == EATSS_CONV2D && dv[1] > dv[0])
        return fail(EATSS_E_INVALID, "eatss_desc_builtin: conv-2d needs f <= n");
    if (k == EATSS_CCSD_T_D1 && dt != EATSS_F32)
        return fail(EATSS_E_UNSUPPORTED, "eatss_desc_builtin: ccsd_t_d1 is fp32 only in this build");
    auto *d = new (std::nothrow) eatss_kernel_desc();
    if (!d) return fail(EATSS_E_NOMEM, "eatss_desc_builtin: out of memory");
    d->kind = k;
    d->dtype = dt;
    d->dims = dv;
    d->tsteps = tsteps;
    eatss_status st = build(d);
    if (st != EATSS_OK) {
        delete d;
        return st;
    }
    *out = d;
    return EATSS_OK;
}

void eatss_desc_destroy(eatss_kernel_desc *d) { delete d; }

int eatss_desc_num_loops(const eatss_kernel_desc *d) {
    if (!d) return -1;
    size_t L = 0;
    for (const Nest &n : d->nests) L = std::max(L, n.loops.size());
    return (int)L;
}
int eatss_desc_num_nests(const eatss_kernel_desc *d) { return d ? (int)d->nests.size() : -1; }
int eatss_desc_num_buffers(const eatss_kernel_desc *d) { return d ? d->num_buffers : -1; }
int64_t eatss_desc_buffer_elems(const eatss_kernel_desc *d, int i) {
    if (!d || i < 0 || i >= d->num_buffers) return -1;
    return d->buffer_elems[i];
}

double eatss_desc_flops(const eatss_kernel_desc *d) {
    if (!d) return 0;
    const auto &x = d->dims;
    auto D = [](int64_t v) { return (double)v; };
    switch (d->kind) {
        case EATSS_GEMM: return 2 * D(x[0]) * D(x[1]) * D(x[2]);
        case EATSS_2MM: return 2 * D(x[0]) * D(x[1]) * D(x[2]) + 2 * D(x[0]) * D(x[3]) * D(x[1]);
        case EATSS_3MM:
            return 2 * (D(x[0]) * D(x[1]) * D(x[2]) + D(x[1]) * D(x[3]) * D(x[4]) + D(x[0]) * D(x[3]) * D(x[1]));
        case EATSS_SYRK: return 2 * D(x.size() == 4 ? x[3] : x[0]) * D(x[0]) * D(x[1]);
        case EATSS_JACOBI2D: return 5 * D(x[0] - 2) * D(x[0] - 2) * D(d->tsteps);
        case EATSS_HEAT3D: return 15 * D(x[0] - 2) * D(x[0] - 2) * D(x[0] - 2) * 2 * D(d->tsteps);
        case EATSS_CCSD_T_D1: return 2 * D(x[0]) * D(x[1]) * D(x[2]) * D(x[3]) * D(x[4]) * D(x[5]) * D(x[6]);
        case EATSS_MVT: return 4 * D(x[0]) * D(x[0]);
        case EATSS_ATAX: case EATSS_BICG: return 4 * D(x[0]) * D(x[1]);
        case EATSS_GEMVER: return 10 * D(x[0]) * D(x[0]) + D(x[0]);  // 4 + 3 + 3 per (i, j), + per i
        // one multiply-add per iteration point (the Khatri-Rao factor C[k][j]*D[l][j] formed once per
        // (k, l, j), not per point)
        case EATSS_MTTKRP: return 2 * D(x[0]) * D(x[1]) * D(x[2]) * D(x[3]);
        case EATSS_CONV2D: return 2 * D(x[1]) * D(x[1]) * D(x[0] - x[1] + 1) * D(x[0] - x[1] + 1);
    }
    return 0;
}

double eatss_desc_bytes(const eatss_kernel_desc *d) {
    if (!d) return 0;
    const double e = dtype_bytes(d->dtype);
    const auto &x = d->dims;
    auto D = [](int64_t v) { return (double)v; };
    switch (d->kind) {
        case EATSS_GEMM: return e * (D(x[0]) * D(x[2]) + D(x[2]) * D(x[1]) + 2 * D(x[0]) * D(x[1]));
        case EATSS_2MM:  // A B read, tmp written; tmp C read, D read+written
            return e * (D(x[0]) * D(x[2]) + D(x[2]) * D(x[1]) + D(x[0]) * D(x[1]) + D(x[0]) * D(x[1]) +
                        D(x[1]) * D(x[3]) + 2 * D(x[0]) * D(x[3]));
        case EATSS_3MM: {
            double s = 0;
            for (int i = 0; i < 7; i++) s += D(d->buffer_elems[i]);
            return e * (s + D(d->buffer_elems[0]) + D(d->buffer_elems[3]));  // E, F re-read by G
        }
        case EATSS_SYRK: return e * (D(x[0]) * D(x[1]) + 2 * D(x.size() == 4 ? x[3] : x[0]) * D(x[0]));
        case EATSS_JACOBI2D:  // per sweep (no time tiling): read src + write dst; + final copy
            return e * 2 * D(x[0]) * D(x[0]) * (D(d->tsteps) + (d->tsteps > 0 ? 1 : 0));
        case EATSS_HEAT3D: return e * 2 * D(x[0]) * D(x[0]) * D(x[0]) * 2 * D(d->tsteps);
        case EATSS_CCSD_T_D1:
            return e * (2 * D(d->buffer_elems[0]) + D(d->buffer_elems[1]) + D(d->buffer_elems[2]));
        // the matrix once (mvt, bicg: both products from one read -- the fused pass) or twice (atax:
        // tmp = A x must be complete before y = A^T tmp); gemver: A read + written by the update,
        // read again by w = A' x; vectors once each (read, + write for outputs)
        case EATSS_MVT: return e * (D(x[0]) * D(x[0]) + 6 * D(x[0]));
        case EATSS_ATAX: return e * (2 * D(x[0]) * D(x[1]) + 2 * D(x[1]) + D(x[0]));
        case EATSS_BICG: return e * (D(x[0]) * D(x[1]) + 2 * D(x[0]) + 2 * D(x[1]));
        case EATSS_GEMVER: return e * (3 * D(x[0]) * D(x[0]) + 11 * D(x[0]));
        case EATSS_MTTKRP:  // A read + written, B, C, D read once
            return e * (2 * D(x[0]) * D(x[1]) + D(x[0]) * D(x[2]) * D(x[3]) + D(x[2]) * D(x[1]) + D(x[3]) * D(x[1]));
        case EATSS_CONV2D:  // inp, W read once, out written once
            return e * (D(x[0]) * D(x[0]) + D(x[1]) * D(x[1]) + D(x[0] - x[1] + 1) * D(x[0] - x[1] + 1));
    }
    return 0;
}

eatss_status eatss_desc_set_scalars(eatss_kernel_desc *d, double alpha, double beta) {
    if (!d) return fail(EATSS_E_INVALID, "eatss_desc_set_scalars: null descriptor");
    d->alpha = alpha;
    d->beta = beta;
    return EATSS_OK;
}

eatss_status eatss_desc_set_exec(eatss_kernel_desc *d, const eatss_exec_opts *o) {
    if (!d || !o) return fail(EATSS_E_INVALID, "eatss_desc_set_exec: null argument");
    if (o->split_pct < 0 || o->split_pct > 100) return fail(EATSS_E_INVALID, "split_pct must be 0..100");
    if (o->engine < 0 || o->engine > 4) return fail(EATSS_E_INVALID, "bad engine");
    if (o->warp_align != 0 && o->warp_align != 4 && o->warp_align != 8 && o->warp_align != 16 && o->warp_align != 32)
        return fail(EATSS_E_INVALID, "warp_align must be 0, 4, 8, 16 or 32");
    if (o->carveout_exact != 0 && o->carveout_exact != 1) return fail(EATSS_E_INVALID, "carveout_exact must be 0 or 1");
    d->exec = *o;
    return EATSS_OK;
}

eatss_status eatss_gpu_params_b200(eatss_gpu_params *o) {
    if (!o) return fail(EATSS_E_INVALID, "null");
    *o = {1024, 32, 255, 65536, 65536, 256 * 1024, 126LL * 1024 * 1024, 148, 232448};
    return EATSS_OK;
}

eatss_status eatss_gpu_params_ga100(eatss_gpu_params *o) {
    if (!o) return fail(EATSS_E_INVALID, "null");
    // Table I: KB/MB read as KiB/MiB (reading Q2); SMs from Table III
    *o = {1024, 32, 255, 65536, 65536, 192 * 1024, 40LL * 1024 * 1024, 108, 48 * 1024};
    return EATSS_OK;
}

eatss_status eatss_gpu_params_query(int device, eatss_gpu_params *o) {
    if (!o) return fail(EATSS_E_INVALID, "null");
    int v[8];
    cudaDeviceAttr a[8] = {cudaDevAttrMaxThreadsPerBlock, cudaDevAttrWarpSize, cudaDevAttrMaxRegistersPerMultiprocessor,
                           cudaDevAttrMaxRegistersPerBlock, cudaDevAttrL2CacheSize, cudaDevAttrMultiProcessorCount,
                           cudaDevAttrMaxSharedMemoryPerBlockOptin, cudaDevAttrMaxSharedMemoryPerMultiprocessor};
    for (int i = 0; i < 8; i++) {
        cudaError_t e = cudaDeviceGetAttribute(&v[i], a[i], device);
        if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceGetAttribute");
    }
    o->threads_per_block = v[0];
    o->threads_per_warp = v[1];
    o->regs_per_thread = 255;
    o->regs_per_sm = v[2];
    o->regs_per_block = v[3];
    // combined L1 + shared memory per SM is not queryable: datasheet 256 KiB on sm_100
    o->l1_shared_bytes = 256 * 1024;
    o->l2_bytes = v[4];
    o->num_sms = v[5];
    o->max_smem_per_block = v[6];
    return EATSS_OK;
}

eatss_status eatss_plan(const eatss_kernel_desc *d, const int64_t *tiles, eatss_launch_plan *plans,
                        int max_plans, int *n_plans) {
    if (!d || !plans || !n_plans) return fail(EATSS_E_INVALID, "eatss_plan: null argument");
    eatss_status st = check_tiles(d, tiles);
    if (st != EATSS_OK) return st;
    const int nn = (int)d->nests.size();
    if (max_plans < nn) return fail(EATSS_E_INVALID, "eatss_plan: max_plans < number of nests");
    const int L = eatss_desc_num_loops(d);
    const bool f64 = d->dtype == EATSS_F64;
    *n_plans = 0;
    if (is_contraction(d->kind)) {
        // alignment-dependent choices assume 256-byte aligned buffers (cudaMalloc / torch)
        std::vector<char> fake(16);
        void *b[EATSS_MAX_BUFFERS];
        for (int i = 0; i < EATSS_MAX_BUFFERS; i++) b[i] = (void *)(uintptr_t)(256 * (i + 1));
        auto cn = contraction_nests(d, b);
        if (simt_untranspose(d)) untranspose_nests(d, cn, b[EATSS_MAX_BUFFERS - 1]);
        for (int i = 0; i < (int)cn.size(); i++) {
            ContractPlan p = plan_contraction(cn[i], tiles, 232448, d->exec.warp_align);
            eatss_launch_plan &o = plans[i];
            std::memset(&o, 0, sizeof(o));
            o.nest = i; o.engine = 1;
            o.grid_x = p.grid_x; o.grid_y = p.grid_y; o.grid_z = 1;
            o.block_x = p.bx; o.block_y = p.by; o.rm = p.rm; o.rn = p.rn; o.vec = p.vec;
            o.passes = p.passes_i * p.passes_j; o.smem_bytes = p.smem_bytes;
            o.a_in_smem = p.a_smem; o.b_in_smem = p.b_smem; o.carveout_pct = d->exec.split_pct;
            o.simt_x = plan_simt_x(p);
            o.tile[0] = p.Ti; o.tile[1] = p.Tj; o.tile[2] = p.Tk;
        }
        *n_plans = (int)cn.size();
    } else if (d->kind == EATSS_JACOBI2D || d->kind == EATSS_HEAT3D) {
        for (int i = 0; i < nn; i++) {
            eatss_launch_plan &o = plans[i];
            std::memset(&o, 0, sizeof(o));
            o.nest = i; o.engine = 1;
            int64_t t[3];
            for (int p = 0; p < L; p++) t[p] = std::min(tiles[p], d->dims[0]);
            stencil_plan_dims(d->kind == EATSS_HEAT3D, d->dims[0], t, f64, &o.grid_x, &o.grid_y, &o.block_x,
                              &o.block_y, &o.vec);
            o.grid_z = 1; o.rm = 1; o.rn = o.vec; o.passes = 1; o.carveout_pct = d->exec.split_pct;
            o.simt_x = stencil_simt_x(d->kind == EATSS_HEAT3D, d->dims[0], t, f64, d->exec.warp_align);
            for (int p = 0; p < L; p++) o.tile[p] = t[p];
        }
        *n_plans = nn;
    } else if (is_lowdim(d->kind)) {  // one CTA per (Ti, Tj) block of the matrix, 256 threads
        const int64_t nx = d->dims[0], ny = d->kind == EATSS_ATAX || d->kind == EATSS_BICG ? d->dims[1] : d->dims[0];
        for (int i = 0; i < nn; i++) {
            eatss_launch_plan &o = plans[i];
            std::memset(&o, 0, sizeof(o));
            o.nest = i; o.engine = 1;
            const int64_t ti = std::min(tiles[0], nx), tj = std::min(tiles[1], ny);
            o.grid_x = (ny + tj - 1) / tj; o.grid_y = (nx + ti - 1) / ti; o.grid_z = 1;
            o.block_x = 256; o.block_y = 1; o.rm = 1; o.rn = 4; o.vec = (ny % 4 == 0 && tj % 4 == 0) ? 4 : 1;
            o.passes = 1; o.carveout_pct = d->exec.split_pct; o.simt_x = 32;
            o.tile[0] = ti; o.tile[1] = tj;
        }
        *n_plans = nn;
    } else if (d->kind == EATSS_MTTKRP || d->kind == EATSS_CONV2D) {
        eatss_launch_plan &o = plans[0];
        std::memset(&o, 0, sizeof(o));
        o.engine = 1;
        o.carveout_pct = d->exec.split_pct;
        if (d->kind == EATSS_MTTKRP) {
            int bx, by, rm, smem, sp;
            const bool fast = mttkrp_plan(d->dims.data(), tiles, &o.grid_x, &o.grid_y, &o.grid_z, &bx, &by, &rm, &smem, &sp);
            o.block_x = bx; o.block_y = by; o.rm = rm; o.rn = fast ? 4 : 1; o.vec = fast ? 4 : 1;
            o.passes = sp;  // split-k factor (grid.z)
            o.smem_bytes = smem; o.a_in_smem = 0; o.b_in_smem = fast;
        } else {
            int threads, smem, rc, wc, groups, segs;
            const bool fast = conv2d_plan(d->dims[0], d->dims[1], tiles, &o.grid_x, &o.grid_y, &threads, &smem, &rc,
                                          &wc, &groups, &segs);
            o.grid_z = 1; o.block_x = threads; o.block_y = 1; o.rm = rc; o.rn = 4; o.vec = fast ? 4 : 1;
            o.passes = 1; o.smem_bytes = smem; o.a_in_smem = fast; o.b_in_smem = 0;
        }
        o.simt_x = std::min(32, o.block_x);
        const int64_t ex[4] = {d->nests[0].loops[0].extent, d->nests[0].loops[1].extent, d->nests[0].loops[2].extent,
                               d->nests[0].loops[3].extent};
        for (int p = 0; p < 4; p++) o.tile[p] = std::min(tiles[p], ex[p]);
        *n_plans = 1;
    } else {
        eatss_launch_plan &o = plans[0];
        std::memset(&o, 0, sizeof(o));
        o.engine = 1;
        ccsd_plan_dims(d->dims.data(), tiles, &o.grid_x, &o.grid_y, &o.block_x, &o.block_y, &o.rm, &o.rn,
                       &o.passes, &o.smem_bytes);
        o.grid_z = 1; o.vec = 1; o.a_in_smem = 1; o.b_in_smem = 1; o.carveout_pct = d->exec.split_pct;
        o.simt_x = std::min(32, o.block_x);
        for (int p = 0; p < 7; p++) o.tile[p] = std::min(tiles[p], d->dims[p]);
        *n_plans = 1;
    }
    return EATSS_OK;
}

// mvt / atax / bicg / gemver as passes of the tiled matrix-vector executor (lowdim.cu); the tile
// (Ti, Tj) maps rows x columns of the matrix for every pass.  `launched` counts kernels (may be null).
static cudaError_t lowdim_run(const eatss_kernel_desc *d, const int64_t *t, void *const *b, cudaStream_t s,
                              int64_t *launched) {
    auto F = [&](int i) { return static_cast<float *>(b[i]); };
    const auto &x = d->dims;
    LowdimArgs a{};
    a.Ti = (int)std::min<int64_t>(t[0], INT32_MAX);
    a.Tj = (int)std::min<int64_t>(t[1], INT32_MAX);
    cudaError_t e;
    auto zero = [&](int i) { return cudaMemsetAsync(b[i], 0, (size_t)d->buffer_elems[i] * 4, s); };
    switch (d->kind) {
        case EATSS_MVT:  // x1 += A y_1 (row form), x2 += A^T y_2 (col form): one pass over A
            a.A = F(4); a.nx = a.ny = x[0];
            a.rowout = F(0); a.vr = F(2); a.ar = 1.f;
            a.colout = F(1); a.vc = F(3); a.ac = 1.f;
            return launch_lowdim(a, true, true, false, s, launched);
        case EATSS_ATAX:  // tmp = A x; y = A^T tmp (tmp complete first)
            if ((e = zero(0)) != cudaSuccess || (e = zero(1)) != cudaSuccess) return e;
            a.A = F(2); a.nx = x[0]; a.ny = x[1];
            a.rowout = F(1); a.vr = F(3); a.ar = 1.f;
            if ((e = launch_lowdim(a, true, false, false, s, launched)) != cudaSuccess) return e;
            a.colout = F(0); a.vc = F(1); a.ac = 1.f;
            return launch_lowdim(a, false, true, false, s, launched);
        case EATSS_BICG:  // s = A^T r (col form), q = A p (row form): one pass over A
            if ((e = zero(0)) != cudaSuccess || (e = zero(1)) != cudaSuccess) return e;
            a.A = F(2); a.nx = x[0]; a.ny = x[1];
            a.colout = F(0); a.vc = F(3); a.ac = 1.f;
            a.rowout = F(1); a.vr = F(4); a.ar = 1.f;
            return launch_lowdim(a, true, true, false, s, launched);
        case EATSS_GEMVER: {  // A' = A + u1 v1^T + u2 v2^T fused with x += beta A'^T y; x += z; w += alpha A' x
            // the fused pass carries nest 2 (x[i] += beta A[j][i] y[j]): its loop i runs along A's
            // columns, so that pass maps tile position 0 to columns and position 1 to rows
            a.Ti = (int)std::min<int64_t>(t[1], INT32_MAX);
            a.Tj = (int)std::min<int64_t>(t[0], INT32_MAX);
            a.A = F(0); a.Aout = F(0); a.nx = a.ny = x[0];
            a.u1 = F(3); a.v1 = F(4); a.u2 = F(5); a.v2 = F(6);
            a.colout = F(1); a.vc = F(7); a.ac = (float)d->beta;
            if ((e = launch_lowdim(a, false, true, true, s, launched)) != cudaSuccess) return e;
            if ((e = launch_lowdim_axpy(F(1), F(8), 1.f, x[0], s, launched)) != cudaSuccess) return e;
            LowdimArgs w{};
            w.A = F(0); w.nx = w.ny = x[0];
            w.Ti = (int)std::min<int64_t>(t[0], INT32_MAX);  // nest 4: i rows, j columns
            w.Tj = (int)std::min<int64_t>(t[1], INT32_MAX);
            w.rowout = F(2); w.vr = F(1); w.ar = (float)d->alpha;
            return launch_lowdim(w, true, false, false, s, launched);
        }
        default:
            return cudaErrorInvalidValue;
    }
}

static eatss_status run_body(eatss_kernel_desc *d, int only_nest, const int64_t *tiles, void *const *buffers,
                             void *stream);
static eatss_status run_impl(const eatss_kernel_desc *cd, int only_nest, const int64_t *tiles,
                             void *const *buffers, void *stream) {
    auto *d = const_cast<eatss_kernel_desc *>(cd);
    if (!d) return fail(EATSS_E_INVALID, "eatss_run: null descriptor");
    d->last_cv.assign(d->nests.size(), -1);
    take_carveout();
    return run_body(d, only_nest, tiles, buffers, stream);
}

static eatss_status run_body(eatss_kernel_desc *d, int only_nest, const int64_t *tiles, void *const *buffers,
                             void *stream) {
    eatss_status st = check_tiles(d, tiles);
    if (st != EATSS_OK) return st;
    st = check_bufs(d, buffers);
    if (st != EATSS_OK) return st;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return fail(EATSS_E_CUDA, "eatss_run: no CUDA device (there is no CPU fallback)");
    cudaStream_t s = (cudaStream_t)stream;
    if (d->exec.engine == EATSS_ENGINE_UNTILED && d->kind != EATSS_JACOBI2D && d->kind != EATSS_HEAT3D)
        return fail(EATSS_E_UNSUPPORTED, "eatss_run: the untiled engine is the stencils' baseline only");
    if (d->exec.engine == EATSS_ENGINE_TENSOR_F16 && (!is_contraction(d->kind) || d->dtype != EATSS_F32))
        return fail(EATSS_E_UNSUPPORTED, "eatss_run: the 3xFP16 tensor engine runs the fp32 gemm family only");
    if (is_contraction(d->kind)) {
        auto cn = contraction_nests(d, buffers);
        const int sl = smem_limit_bytes();
        if (simt_untranspose(d)) {
            const int64_t ni = d->dims[0], nj = d->dims[1];
            if ((st = ensure_ws(d, (size_t)ni * nj * 4)) != EATSS_OK) return st;
            cudaError_t e = launch_transpose((const float *)buffers[1], ni, nj, nj, (float *)d->ws, s);
            if (e != cudaSuccess) return cuda_fail(e, "eatss_run(syrk layout pass)");
            untranspose_nests(d, cn, d->ws);
        }
        RunScratch scratch;  // split-operand scratch of the tcgen05 GEMMs (stream-ordered, this run only)
        const bool f16 = d->exec.engine == EATSS_ENGINE_TENSOR_F16;
        if (d->exec.engine == EATSS_ENGINE_TENSOR || f16) {
            size_t need = 0;
            for (int i = 0; i < (int)cn.size(); i++) {
                ContractPlan p = plan_contraction(cn[i], tiles, sl, d->exec.warp_align);
                if (f16 && tcf_applicable(cn[i], p)) need = std::max(need, tcf_ws_floats(cn[i], p));
                if (!f16 && tcm_applicable(cn[i], p)) need = std::max(need, tcm_ws_floats(cn[i], p));
            }
            if (need) {
                cudaError_t e = scratch.alloc(need * 4, s);
                if (e != cudaSuccess) return cuda_fail(e, "eatss_run(tensor scratch)");
            }
        }
        for (int i = 0; i < (int)cn.size(); i++) {
            if (only_nest >= 0 && i != only_nest) continue;
            ContractPlan p = plan_contraction(cn[i], tiles, sl, d->exec.warp_align);
            int tsm = 0, tcols = 0;
            const bool want_tc = d->exec.engine == EATSS_ENGINE_TENSOR;
            // MMA-legal tiles (Ti = 128/256) take the TMA/SS-UMMA GEMM; narrow tiles the transposed TS kernel
            const bool tcm = want_tc && tcm_applicable(cn[i], p);
            const bool tc = want_tc && !tcm && tc_plan(cn[i], p, &tsm, &tcols);
            const bool tcf = f16 && tcf_applicable(cn[i], p);
            if (want_tc && !tc && !tcm)
                return fail(EATSS_E_UNSUPPORTED, "eatss_run: tensor engine not applicable to this tile/operand layout");
            if (f16 && !tcf)
                return fail(EATSS_E_UNSUPPORTED, "eatss_run: the 3xFP16 tensor engine needs Ti in {128, 256}, Tj in "
                                                 "16..256 step 16, Tk in {16, 32, 64, 128} fitting two stages");
            cudaEvent_t *ev = kernel_events(d, i);
            if (ev && !tcm && !tcf) cudaEventRecord(ev[0], s);
            cudaError_t e = tcf   ? launch_tcf_contraction(cn[i], p, (float *)scratch.p, scratch.bytes / 4, s, ev)
                            : tcm ? launch_tcm_contraction(cn[i], p, (float *)scratch.p, scratch.bytes / 4, s, ev)
                            : tc  ? launch_tc_contraction(cn[i], p, exec_cv(d), s)
                                  : launch_contraction(cn[i], p, exec_cv(d), nullptr, s);
            if (ev && !tcm && !tcf) cudaEventRecord(ev[1], s);
            d->last_cv[i] = take_carveout();
            if (e != cudaSuccess) return cuda_fail(e, "eatss_run(contraction)");
        }
        return EATSS_OK;
    }
    if (is_lowdim(d->kind)) {
        if (only_nest >= 0) return fail(EATSS_E_UNSUPPORTED, "eatss_run_nest: low-dimensional kernels run whole");
        if (d->dtype != EATSS_F32)  // fp64 descriptors serve the model (paper-mode tables) only
            return fail(EATSS_E_UNSUPPORTED, "eatss_run: the low-dimensional executor is fp32 only");
        cudaEvent_t *ev = kernel_events(d, 0);
        if (ev) cudaEventRecord(ev[0], s);
        const cudaError_t e = lowdim_run(d, tiles, buffers, s, nullptr);
        if (ev) cudaEventRecord(ev[1], s);
        return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_run(low-dimensional kernel)");
    }
    if (d->kind == EATSS_MTTKRP || d->kind == EATSS_CONV2D) {
        if (d->dtype != EATSS_F32)  // fp64 descriptors serve the model (paper-mode tables) only
            return fail(EATSS_E_UNSUPPORTED, "eatss_run: the mttkrp / conv-2d executors are fp32 only");
        cudaEvent_t *ev = kernel_events(d, 0);
        cudaError_t e = cudaSuccess;
        if (d->kind == EATSS_MTTKRP) {
            const bool tc = d->exec.engine == EATSS_ENGINE_TENSOR;
            if (tc && !mttkrp_tc_applicable(d->dims.data(), tiles))
                return fail(EATSS_E_UNSUPPORTED, "eatss_run: the mttkrp tensor engine needs the tile (1, nj, 128, 32) "
                                                 "with nj in {32, 64, 128}, nk % 128 == 0, nl % 32 == 0");
            int64_t gx, gy, gz;
            int bx, by, rm, smem, sp;
            mttkrp_plan(d->dims.data(), tiles, &gx, &gy, &gz, &bx, &by, &rm, &smem, &sp);
            if (tc || sp > 1) {  // split partials (SIMT) / D lo + block partials (tensor): library-owned
                const size_t need = tc ? mttkrp_tc_ws_floats(d->dims.data()) * 4
                                       : (size_t)sp * (size_t)d->buffer_elems[0] * 4;
                eatss_status ws_st = ensure_ws(d, need);
                if (ws_st != EATSS_OK) return ws_st;
            }
            if (tc) {  // events around the tcgen05 kernel alone (the D split and the block reduction outside)
                e = launch_mttkrp_tc((float *)buffers[0], (const float *)buffers[1], (const float *)buffers[2],
                                     (const float *)buffers[3], d->dims.data(), (float *)d->ws, s, ev, nullptr);
                return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_run(mttkrp, tensor)");
            }
            if (ev) cudaEventRecord(ev[0], s);
            e = launch_mttkrp((float *)buffers[0], (const float *)buffers[1], (const float *)buffers[2],
                              (const float *)buffers[3], d->dims.data(), tiles, (float *)d->ws, nullptr, s, nullptr);
        } else {
            if (ev) cudaEventRecord(ev[0], s);
            e = launch_conv2d((float *)buffers[0], (const float *)buffers[1], (const float *)buffers[2], d->dims[0],
                              d->dims[1], tiles, nullptr, s, nullptr);
        }
        if (ev) cudaEventRecord(ev[1], s);
        return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_run(mttkrp / conv-2d)");
    }
    if (d->kind == EATSS_JACOBI2D || d->kind == EATSS_HEAT3D) {
        if (only_nest >= 0) return fail(EATSS_E_UNSUPPORTED, "eatss_run_nest: stencils run whole time loops");
        cudaEvent_t *ev = kernel_events(d, 0);
        if (ev) cudaEventRecord(ev[0], s);
        const eatss_status r = stencil_run(d, tiles, buffers, s);
        if (ev) cudaEventRecord(ev[1], s);
        for (auto &v : d->last_cv) v = d->graph_cv;  // set by the capture / direct issue
        return r;
    }
    cudaEvent_t *ev = kernel_events(d, 0);
    if (d->exec.engine == EATSS_ENGINE_TENSOR) {  // tcgen05 3xTF32 with TMA-streamed t3 (ccsd_tc.cu)
        if (!ccsd_tc_applicable(d->dims.data(), tiles))
            return fail(EATSS_E_UNSUPPORTED, "eatss_run: tensor engine needs a ccsd tile (1,1,Th1,Tp6,Tp5,Tp4,>=H7) "
                                             "with Th1*Tp5*Tp4 <= 128, Tp6 % 16 == 0, Tp4 % 4 == 0, "
                                             "P4 % 4 == 0, H7 % 4 == 0, H7 <= 64");
        RunScratch scratch;  // v2's lo half (stream-ordered, this run only)
        cudaError_t e = scratch.alloc(ccsd_tc_ws_floats(d->dims.data()) * 4, s);
        if (e != cudaSuccess) return cuda_fail(e, "eatss_run(ccsd tensor scratch)");
        e = launch_ccsd_tc((float *)buffers[0], (const float *)buffers[1], (const float *)buffers[2], d->dims.data(),
                           tiles, 0, d->dims[0], (float *)scratch.p, scratch.bytes / 4, s, ev);
        return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_run(ccsd_t_d1, tensor)");
    }
    if (ev) cudaEventRecord(ev[0], s);
    cudaError_t e = launch_ccsd_d1((float *)buffers[0], (const float *)buffers[1], (const float *)buffers[2],
                                   d->dims.data(), tiles, 0, d->dims[0], exec_cv(d), nullptr, s);
    if (ev) cudaEventRecord(ev[1], s);
    d->last_cv[0] = take_carveout();
    return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_run(ccsd_t_d1)");
}

eatss_status eatss_run(const eatss_kernel_desc *d, const int64_t *tiles, void *const *buffers, void *stream) {
    return run_impl(d, -1, tiles, buffers, stream);
}

eatss_status eatss_run_nest(const eatss_kernel_desc *d, int nest, const int64_t *tiles, void *const *buffers,
                            void *stream) {
    if (!d || nest < 0 || nest >= (int)d->nests.size()) return fail(EATSS_E_INVALID, "eatss_run_nest: bad nest");
    return run_impl(d, nest, tiles, buffers, stream);
}

// ------------------------------------------------------------------ host-buffer execution
// Which buffers a builtin reads (copied host->device) and writes (copied device->host).
static void buffer_io(const eatss_kernel_desc *d, int i, bool *in, bool *out) {
    *in = true;
    *out = false;
    switch (d->kind) {
        case EATSS_GEMM: case EATSS_SYRK: case EATSS_CCSD_T_D1: *out = i == 0; break;
        case EATSS_2MM: *in = i != 0; *out = i == 0 || i == 4; break;
        case EATSS_3MM: *in = !(i == 0 || i == 3 || i == 6); *out = !*in; break;
        case EATSS_JACOBI2D: case EATSS_HEAT3D: *out = true; break;
        case EATSS_MVT: *out = i <= 1; break;
        case EATSS_ATAX: *in = i >= 2; *out = i <= 1; break;
        case EATSS_BICG: *in = i >= 2; *out = i <= 1; break;
        case EATSS_GEMVER: *out = i <= 2; break;
        case EATSS_MTTKRP: *out = i == 0; break;
        case EATSS_CONV2D: *in = i != 0; *out = i == 0; break;
    }
}

eatss_status eatss_run_host(const eatss_kernel_desc *cd, const int64_t *tiles, void *const *host_buffers,
                            int64_t row_blocks, void *stream) {
    auto *d = const_cast<eatss_kernel_desc *>(cd);
    if (!d || !host_buffers) return fail(EATSS_E_INVALID, "eatss_run_host: null argument");
    for (int i = 0; i < d->num_buffers; i++)
        if (!host_buffers[i]) return fail(EATSS_E_INVALID, "eatss_run_host: null host buffer");
    eatss_status st = check_tiles(d, tiles);
    if (st != EATSS_OK) return st;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return fail(EATSS_E_CUDA, "eatss_run_host: no CUDA device (there is no CPU fallback)");
    int dev = 0;
    cudaGetDevice(&dev);
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e = cudaSuccess;
    // library-owned device buffers, streams and events (per descriptor, re-created on a device change)
    if (d->hdev != dev) {
        for (void *b : d->hbuf) cudaFree(b);
        for (void *ev : d->hev) cudaEventDestroy((cudaEvent_t)ev);
        for (void *&hs : d->hstream)
            if (hs) { cudaStreamDestroy((cudaStream_t)hs); hs = nullptr; }
        d->hbuf.assign(d->num_buffers, nullptr);
        d->hbuf_bytes.assign(d->num_buffers, 0);
        d->hev.clear();
        d->hdev = dev;
    }
    const size_t esz = (size_t)dtype_bytes(d->dtype);
    for (int i = 0; i < d->num_buffers; i++) {
        const size_t bytes = (size_t)d->buffer_elems[i] * esz;
        if (d->hbuf_bytes[i] < bytes) {
            if (d->hbuf[i]) cudaFree(d->hbuf[i]);
            d->hbuf[i] = nullptr;
            if ((e = cudaMalloc(&d->hbuf[i], bytes)) != cudaSuccess) {
                d->hbuf_bytes[i] = 0;
                return cuda_fail(e, "eatss_run_host: device buffer");
            }
            d->hbuf_bytes[i] = bytes;
        }
    }
    for (void *&hs : d->hstream)
        if (!hs) {
            cudaStream_t t;
            if ((e = cudaStreamCreateWithFlags(&t, cudaStreamNonBlocking)) != cudaSuccess)
                return cuda_fail(e, "eatss_run_host: stream");
            hs = t;
        }
    cudaStream_t sin = (cudaStream_t)d->hstream[0], sout = (cudaStream_t)d->hstream[1];
    auto event = [&](size_t k) -> cudaEvent_t {
        while (d->hev.size() <= k) {
            cudaEvent_t ev;
            if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) return nullptr;
            d->hev.push_back(ev);
        }
        return (cudaEvent_t)d->hev[k];
    };
    // event slots: 0 = start, 1 = end, 2.. = pipeline
    // previous work on s (an earlier call's kernels may still read the device copies) before copies
    cudaEvent_t e0 = event(0);
    if (!e0) return fail(EATSS_E_CUDA, "eatss_run_host: event");
    cudaEventRecord(e0, s);
    cudaStreamWaitEvent(sin, e0, 0);
    cudaStreamWaitEvent(sout, e0, 0);
    void *dev_bufs[EATSS_MAX_BUFFERS];
    for (int i = 0; i < d->num_buffers; i++) dev_bufs[i] = d->hbuf[i];
    const bool f64 = d->dtype == EATSS_F64;
    // gemm: row blocks of whole i-tiles pipelined -- B first, then per block A_r, C_r host->device,
    // the block's gemm, and C_r device->host, the three on separate streams so copies in both
    // directions overlap the compute (each block sees the single-launch operation order: its
    // tiles are whole i-tiles of the full problem)
    if (d->kind == EATSS_GEMM && row_blocks > 1) {
        auto cn = contraction_nests(d, dev_bufs);
        ContractNest full = cn[0];
        const int64_t M = full.M, Ti = std::max<int64_t>(1, std::min(tiles[0], M));
        const bool f16 = d->exec.engine == EATSS_ENGINE_TENSOR_F16;
        const int64_t unit = d->exec.engine == EATSS_ENGINE_TENSOR || f16 ? std::max<int64_t>(Ti, 256) : Ti;
        int64_t rb = (M + row_blocks - 1) / row_blocks;
        rb = (rb + unit - 1) / unit * unit;
        const int nblk = (int)((M + rb - 1) / rb);
        const size_t rowA = (size_t)full.lda * esz, rowC = (size_t)full.ldc * esz;
        char *hA = (char *)host_buffers[1], *hB = (char *)host_buffers[2], *hC = (char *)host_buffers[0];
        char *dA = (char *)dev_bufs[1], *dC = (char *)dev_bufs[0];
        cudaMemcpyAsync(dev_bufs[2], hB, d->hbuf_bytes[2], cudaMemcpyHostToDevice, sin);
        const int sl = smem_limit_bytes();
        RunScratch scratch;  // tensor engine: split operands of the largest block (blocks run in order on s)
        if (d->exec.engine == EATSS_ENGINE_TENSOR || f16) {
            ContractNest b0 = full;
            b0.M = std::min(rb, M);
            ContractPlan p0 = plan_contraction(b0, tiles, sl, d->exec.warp_align);
            const size_t need = f16 ? (tcf_applicable(b0, p0) ? tcf_ws_floats(b0, p0) : 0)
                                    : (tcm_applicable(b0, p0) ? tcm_ws_floats(b0, p0) : 0);
            if (need) {
                const cudaError_t ea = scratch.alloc(need * 4, s);
                if (ea != cudaSuccess) return cuda_fail(ea, "eatss_run_host(tensor scratch)");
            }
        }
        for (int r = 0; r < nblk; r++) {
            const int64_t r0 = (int64_t)r * rb, rows = std::min(rb, M - r0);
            cudaMemcpyAsync(dA + r0 * rowA, hA + r0 * rowA, rows * rowA, cudaMemcpyHostToDevice, sin);
            cudaMemcpyAsync(dC + r0 * rowC, hC + r0 * rowC, rows * rowC, cudaMemcpyHostToDevice, sin);
            cudaEvent_t ein = event(2 + 2 * r), ecomp = event(3 + 2 * r);
            if (!ein || !ecomp) return fail(EATSS_E_CUDA, "eatss_run_host: event");
            cudaEventRecord(ein, sin);
            cudaStreamWaitEvent(s, ein, 0);
            ContractNest blk = full;
            blk.M = rows;
            blk.A = dA + r0 * rowA;
            blk.C = dC + r0 * rowC;
            ContractPlan p = plan_contraction(blk, tiles, sl, d->exec.warp_align);
            const bool want_tc = d->exec.engine == EATSS_ENGINE_TENSOR;
            int tsm = 0, tcols = 0;
            const bool tcm = want_tc && tcm_applicable(blk, p);
            const bool tc = want_tc && !tcm && tc_plan(blk, p, &tsm, &tcols);
            const bool tcf = f16 && tcf_applicable(blk, p);
            if ((want_tc && !tc && !tcm) || (f16 && !tcf))
                return fail(EATSS_E_UNSUPPORTED, "eatss_run_host: tensor engine not applicable to this tile");
            e = tcf   ? launch_tcf_contraction(blk, p, (float *)scratch.p, scratch.bytes / 4, s, nullptr)
                : tcm ? launch_tcm_contraction(blk, p, (float *)scratch.p, scratch.bytes / 4, s, nullptr)
                : tc  ? launch_tc_contraction(blk, p, exec_cv(d), s)
                      : launch_contraction(blk, p, exec_cv(d), nullptr, s);
            if (e != cudaSuccess) return cuda_fail(e, "eatss_run_host(gemm block)");
            cudaEventRecord(ecomp, s);
            cudaStreamWaitEvent(sout, ecomp, 0);
            cudaMemcpyAsync(hC + r0 * rowC, dC + r0 * rowC, rows * rowC, cudaMemcpyDeviceToHost, sout);
        }
        (void)f64;
    } else {
        for (int i = 0; i < d->num_buffers; i++) {
            bool in, out;
            buffer_io(d, i, &in, &out);
            if (in) cudaMemcpyAsync(dev_bufs[i], host_buffers[i], d->hbuf_bytes[i], cudaMemcpyHostToDevice, sin);
        }
        cudaEvent_t ein = event(2);
        if (!ein) return fail(EATSS_E_CUDA, "eatss_run_host: event");
        cudaEventRecord(ein, sin);
        cudaStreamWaitEvent(s, ein, 0);
        st = run_impl(d, -1, tiles, dev_bufs, s);
        if (st != EATSS_OK) return st;
        cudaEvent_t ecomp = event(3);
        cudaEventRecord(ecomp, s);
        cudaStreamWaitEvent(sout, ecomp, 0);
        for (int i = 0; i < d->num_buffers; i++) {
            bool in, out;
            buffer_io(d, i, &in, &out);
            if (out) cudaMemcpyAsync(host_buffers[i], dev_bufs[i], d->hbuf_bytes[i], cudaMemcpyDeviceToHost, sout);
        }
    }
    // the call is complete on `stream` once the device->host copies are
    cudaEvent_t eend = event(1);
    if (!eend) return fail(EATSS_E_CUDA, "eatss_run_host: event");
    cudaEventRecord(eend, sout);
    cudaStreamWaitEvent(s, eend, 0);
    e = cudaGetLastError();
    return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_run_host");
}

eatss_status eatss_coverage(const eatss_kernel_desc *d, int nest, const int64_t *tiles, int32_t *counts,
                            void *stream) {
    if (!d || !counts || nest < 0 || nest >= (int)d->nests.size())
        return fail(EATSS_E_INVALID, "eatss_coverage: bad argument");
    eatss_status st = check_tiles(d, tiles);
    if (st != EATSS_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    const bool f64 = d->dtype == EATSS_F64;
    if (is_contraction(d->kind)) {
        // operand pointers are never dereferenced in coverage mode; use aligned dummies
        void *b[EATSS_MAX_BUFFERS];
        for (int i = 0; i < EATSS_MAX_BUFFERS; i++) b[i] = (void *)(uintptr_t)(256 * (i + 1));
        auto cn = contraction_nests(d, b);
        ContractPlan p = plan_contraction(cn[nest], tiles, smem_limit_bytes(), d->exec.warp_align);
        p.a_smem = false;  // no operand traffic in coverage mode
        p.b_smem = false;
        p.smem_bytes = 0;
        cudaError_t e = launch_contraction(cn[nest], p, exec_cv(d), counts, s);
        return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_coverage");
    }
    if (is_lowdim(d->kind))
        return fail(EATSS_E_UNSUPPORTED, "eatss_coverage: the low-dimensional kernels have no visit-count mode");
    if (d->kind == EATSS_MTTKRP) {
        cudaError_t e = launch_mttkrp(nullptr, nullptr, nullptr, nullptr, d->dims.data(), tiles, nullptr, counts, s,
                                      nullptr);
        return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_coverage");
    }
    if (d->kind == EATSS_CONV2D) {
        cudaError_t e = launch_conv2d(nullptr, nullptr, nullptr, d->dims[0], d->dims[1], tiles, counts, s, nullptr);
        return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_coverage");
    }
    const int64_t n = d->dims[0];
    cudaError_t e;
    if (d->kind == EATSS_JACOBI2D)
        e = launch_jacobi2d_sweep(nullptr, nullptr, nullptr, n, tiles[0], tiles[1], f64, exec_cv(d), counts, s,
                                  d->exec.warp_align);
    else if (d->kind == EATSS_HEAT3D)
        e = launch_heat3d_sweep(nullptr, nullptr, n, tiles[0], tiles[1], tiles[2], f64, exec_cv(d), counts, s,
                                d->exec.warp_align);
    else
        e = launch_ccsd_d1(nullptr, nullptr, nullptr, d->dims.data(), tiles, 0, d->dims[0], exec_cv(d),
                           counts, s);
    return e == cudaSuccess ? EATSS_OK : cuda_fail(e, "eatss_coverage");
}

int64_t eatss_launches_per_run(const eatss_kernel_desc *d, const int64_t *tiles) {
    if (!d) return -1;
    if (is_contraction(d->kind) && d->exec.engine == EATSS_ENGINE_TENSOR_F16) {
        if (!tiles || check_tiles(d, tiles) != EATSS_OK) return -1;
        void *b[EATSS_MAX_BUFFERS];
        for (int i = 0; i < EATSS_MAX_BUFFERS; i++) b[i] = (void *)((uintptr_t)(1 << 20) * (uintptr_t)(i + 1));
        int64_t total = 0;
        for (auto &n : contraction_nests(d, b)) {
            ContractPlan p = plan_contraction(n, tiles, smem_limit_bytes(), d->exec.warp_align);
            if (!tcf_applicable(n, p)) return -1;
            total += 3;  // row / column maxima, split + tail pre-pass, GEMM
        }
        return total;
    }
    if (is_contraction(d->kind) && d->exec.engine == EATSS_ENGINE_TENSOR) {
        if (!tiles || check_tiles(d, tiles) != EATSS_OK) return -1;
        void *b[EATSS_MAX_BUFFERS];  // layout only: aligned dummies, never dereferenced
        for (int i = 0; i < EATSS_MAX_BUFFERS; i++) b[i] = (void *)((uintptr_t)(1 << 20) * (uintptr_t)(i + 1));
        auto cn = contraction_nests(d, b);
        const int sl = smem_limit_bytes();
        int64_t total = 0;
        for (auto &n : cn) {
            ContractPlan p = plan_contraction(n, tiles, sl, d->exec.warp_align);
            int tsm = 0, tcols = 0;
            total += tcm_applicable(n, p) ? tcm_launches(n, p) : tc_plan(n, p, &tsm, &tcols) ? 1 : 0;
        }
        return total;
    }
    if (d->kind == EATSS_CCSD_T_D1 && d->exec.engine == EATSS_ENGINE_TENSOR) return 2;  // prep + contraction
    if (is_contraction(d->kind)) {  // SIMT: one kernel per nest (+ the tail pre-pass when it splits)
        if (!tiles || check_tiles(d, tiles) != EATSS_OK) return -1;
        void *b[EATSS_MAX_BUFFERS];
        for (int i = 0; i < EATSS_MAX_BUFFERS; i++) b[i] = (void *)((uintptr_t)(1 << 20) * (uintptr_t)(i + 1));
        int64_t total = 0;
        const int sl = smem_limit_bytes();
        auto cn = contraction_nests(d, b);
        if (simt_untranspose(d)) {
            untranspose_nests(d, cn, b[EATSS_MAX_BUFFERS - 1]);
            total += 1;  // the layout pass
        }
        for (auto &n : cn) total += contraction_launches(n, plan_contraction(n, tiles, sl, d->exec.warp_align));
        return total;
    }
    switch (d->kind) {
        case EATSS_CCSD_T_D1: return 1;
        case EATSS_JACOBI2D: return d->tsteps + (d->tsteps > 0 ? 1 : 0);
        case EATSS_HEAT3D: return 2 * d->tsteps;
        case EATSS_MVT: case EATSS_BICG: return 1;  // one fused pass over the matrix
        case EATSS_ATAX: return 2;
        case EATSS_GEMVER: return 3;
        case EATSS_CONV2D: return 1;
        case EATSS_MTTKRP: {  // the kernel, + the split-order reduction when k is split across CTAs
            if (!tiles || check_tiles(d, tiles) != EATSS_OK) return -1;
            if (d->exec.engine == EATSS_ENGINE_TENSOR)  // D lo split, tcgen05 kernel, block reduction
                return mttkrp_tc_applicable(d->dims.data(), tiles) ? 3 : -1;
            int64_t gx, gy, gz;
            int bx, by, rm, smem, sp;
            mttkrp_plan(d->dims.data(), tiles, &gx, &gy, &gz, &bx, &by, &rm, &smem, &sp);
            return sp > 1 ? 2 : 1;
        }
    }
    return -1;
}

eatss_status eatss_last_carveout(const eatss_kernel_desc *d, int32_t *pct, int32_t cap, int32_t *n) {
    if (!d || !n || (cap > 0 && !pct)) return fail(EATSS_E_INVALID, "eatss_last_carveout: bad argument");
    const int cnt = (int)d->last_cv.size();
    for (int i = 0; i < cnt && i < cap; i++) pct[i] = d->last_cv[i];
    *n = cnt;
    return EATSS_OK;
}

eatss_status eatss_last_kernel_ms(const eatss_kernel_desc *cd, float *ms, int32_t cap, int32_t *n) {
    auto *d = const_cast<eatss_kernel_desc *>(cd);
    if (!d || !n || (cap > 0 && !ms)) return fail(EATSS_E_INVALID, "eatss_last_kernel_ms: bad argument");
    if (!d->kev_valid) return fail(EATSS_E_INVALID, "eatss_last_kernel_ms: no run with exec.time_kernels = 1");
    int cnt = 0;
    for (int i = 0; i < d->kev_valid; i++) {
        cudaEvent_t a = (cudaEvent_t)d->kev[2 * i], b = (cudaEvent_t)d->kev[2 * i + 1];
        float t = 0.f;
        cudaError_t e = cudaEventSynchronize(b);
        if (e == cudaSuccess) e = cudaEventElapsedTime(&t, a, b);
        if (e == cudaErrorNotReady || e == cudaErrorInvalidResourceHandle) t = -1.f, e = cudaSuccess;
        if (e != cudaSuccess) return cuda_fail(e, "eatss_last_kernel_ms");
        if (cnt < cap) ms[cnt] = t;
        cnt++;
    }
    *n = cnt;
    return EATSS_OK;
}

}  // extern "C"
