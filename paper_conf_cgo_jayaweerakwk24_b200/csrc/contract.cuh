// contract.cuh -- internal interface of the tiled contraction executors.
#pragma once
#include <cstdint>

#include <cuda_runtime.h>

namespace eatss {

// Carve-out request handed to the SIMT launchers: the model's split sigma in percent,
// bit 8 set when it must be honoured exactly (exec.carveout_exact); otherwise it is a lower bound
// the launcher raises as far as its register-limited resident CTAs need.  The
// launchers report what they requested through note_carveout (read back per nest by the API).
inline int cv_make(int pct, bool exact) { return pct | (exact ? 0x100 : 0); }
inline int cv_resolve(int cv, int need) {
    const int pct = cv & 0xff;
    return (cv & 0x100) ? pct : (pct > need ? pct : need);
}
void note_carveout(int pct);  // thread-local: the last carve-out a launcher requested
int take_carveout();          // read and reset (-1 when none was requested)

// One gemm-like nest of the gemm family (gemm, 2mm, 3mm, syrk):
//   C(i,j) = [init_zero ? 0 : beta*C(i,j)] + alpha * sum_k A(i,k) * B(k,j)
//   A(i,k) = A[i*lda + k];  B(k,j) = transB ? B[j*ldb + k] : B[k*ldb + j];  C(i,j) = C[i*ldc + j]
struct ContractNest {
    int64_t M = 0, N = 0, K = 0;
    const void *A = nullptr;
    int64_t lda = 0;
    const void *B = nullptr;
    int64_t ldb = 0;
    bool transB = false;
    void *C = nullptr;
    int64_t ldc = 0;
    double alpha = 1.0, beta = 1.0;
    bool init_zero = false;
    bool f64 = false;
};

struct ContractPlan {
    int64_t Ti = 0, Tj = 0, Tk = 0;  // clipped tile
    int64_t rTi = 0, rTj = 0, rTk = 0;  // tile as requested (the tensor engine's MMA-legal shape)
    int rm = 1, rn = 1, vec = 1;
    int bx = 1, by = 1;
    int passes_i = 1, passes_j = 1;
    bool stream = false;  // accumulators not resident: RMW of C per k-tile through L1
    bool staged = false;  // resident fast path: both operand slices staged via cp.async ring (nbuf stages)
    bool a_smem = true, b_smem = false;
    int nbuf = 1;
    int kst = 0;  // staged path: k-rows per ring stage
    int tkp = 0, tjp = 0;  // shared-memory pitches (elements)
    int bkp = 0;           // staged transposed operand kept as [j][k] rows of this k-pitch (0 = [k][j])
    int smem_bytes = 0;
    int64_t grid_x = 1, grid_y = 1;
    int waf = 0;  // lanes of each warp along j (exec.warp_align; 0 = linear thread layout)
};

ContractPlan plan_contraction(const ContractNest &n, const int64_t *tiles, int smem_limit, int waf = 0);
// lanes of one warp laid along j by a plan (the executor's SIMT length)
int plan_simt_x(const ContractPlan &p);
// tensor-core (tcgen05, 3xTF32) executor: applicability / launch (tc_gemm.cu)
bool tc_plan(const ContractNest &n, const ContractPlan &p, int *smem_bytes, int *tmem_cols);
cudaError_t launch_tc_contraction(const ContractNest &n, const ContractPlan &p, int carveout, cudaStream_t s);
// tcgen05 3xTF32 GEMM for MMA-legal tiles (tc_mma.cu): Ti in {128, 256} (one CTA / a CTA pair),
// Tj in 16..256 step 16, Tk in {8, 16, 32, 64}
bool tcm_applicable(const ContractNest &n, const ContractPlan &p, bool f16 = false);
// Split-operand workspace (floats) one launch needs: owned by the caller's descriptor, so
// concurrent descriptors (streams, devices, host threads) never share it.
size_t tcm_ws_floats(const ContractNest &n, const ContractPlan &p);
// ws: >= tcm_ws_floats() floats on the current device, used in stream order by this launch;
// ev: optional {start, stop} events recorded around the GEMM kernel alone
cudaError_t launch_tcm_contraction(const ContractNest &n, const ContractPlan &p, float *ws, size_t ws_floats,
                                   cudaStream_t s, cudaEvent_t *ev = nullptr);
int tcm_launches(const ContractNest &n, const ContractPlan &p);  // kernels one launch_tcm_contraction issues
// 3xFP16 variant of the same GEMM (engine TENSOR_F16): operands split into fp16 hi / lo after a per-row (A)
// / per-column (B) power-of-two scaling that keeps them inside fp16's range; same tiles, Tk in fp16 elements
// (16, 32, 64, 128: 32..256 bytes per stage row); B always K-major (the split transposes a row-major B)
bool tcf_applicable(const ContractNest &n, const ContractPlan &p);
size_t tcf_ws_floats(const ContractNest &n, const ContractPlan &p);
cudaError_t launch_tcf_contraction(const ContractNest &n, const ContractPlan &p, float *ws, size_t ws_floats,
                                   cudaStream_t s, cudaEvent_t *ev = nullptr);
cudaError_t launch_contraction(const ContractNest &n, const ContractPlan &p, int carveout_pct,
                               int32_t *coverage_counts, cudaStream_t s);
// kernels one launch_contraction issues (the SIMT staged path adds a pre-pass when it splits the
// wave tail along k)
int contraction_launches(const ContractNest &n, const ContractPlan &p);
// dst[c][r] = src[r][c]: fp32, rows x cols with row pitch lds -> cols x rows dense
cudaError_t launch_transpose(const float *src, int64_t rows, int64_t cols, int64_t lds, float *dst, cudaStream_t s);

}  // namespace eatss
