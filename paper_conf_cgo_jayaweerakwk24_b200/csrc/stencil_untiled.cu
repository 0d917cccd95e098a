// stencil_untiled.cu -- the UNTILED stencil baseline of BASELINE config 4 ("jacobi-2d / heat-3d
// stencils, 500 timesteps, EATSS tiles vs untiled").
//
// The plain loop nest mapped onto the GPU without tiling: one thread per interior point, a fixed
// 32 x 8 thread block, every neighbour read from global memory through L1 (no shared-memory staging,
// no register reuse along a walk).  The tile vector is ignored (exec engine EATSS_ENGINE_UNTILED).
// Same time loop (ping-pong, jacobi's final copy nest, CUDA-graph replay) and the same per-point
// arithmetic as stencil.cu / stencil_staged.cu, so results agree with the tiled executors within
// rounding (identical association; FMA contraction may differ).
#include <cuda_runtime.h>

#include <cstdint>

namespace eatss {

namespace {

template <typename T>
__global__ void __launch_bounds__(256) jacobi2d_untiled(T *__restrict__ dst, const T *__restrict__ src,
                                                        const T *__restrict__ bsrc, int64_t n) {
    const int64_t j = 1 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t i = 1 + (int64_t)blockIdx.y * blockDim.y + threadIdx.y;
    if (i >= n - 1 || j >= n - 1) return;
    // boundary cells of the ping-pong sweep that reads B come from A (stencil.cu)
    auto S = [&](int64_t r, int64_t c) -> T {
        const bool b = (r == 0) | (r == n - 1) | (c == 0) | (c == n - 1);
        return b ? bsrc[r * n + c] : src[r * n + c];
    };
    const T c02 = T(0.2);
    dst[i * n + j] = c02 * ((((S(i, j) + S(i, j - 1)) + S(i, j + 1)) + S(i + 1, j)) + S(i - 1, j));
}

template <typename T>
__global__ void __launch_bounds__(256) heat3d_untiled(T *__restrict__ dst, const T *__restrict__ src, int64_t n) {
    const int64_t k = 1 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t j = 1 + (int64_t)blockIdx.y * blockDim.y + threadIdx.y;
    const int64_t i = 1 + (int64_t)blockIdx.z;
    if (i >= n - 1 || j >= n - 1 || k >= n - 1) return;
    const int64_t nn = n * n, o = i * nn + j * n + k;
    const T c = T(0.125), two = T(2.0);
    const T x = src[o];
    dst[o] = c * (src[o + nn] - two * x + src[o - nn]) + c * (src[o + n] - two * x + src[o - n]) +
             c * (src[o + 1] - two * x + src[o - 1]) + x;
}

}  // namespace

cudaError_t launch_jacobi2d_untiled(void *dst, const void *src, const void *bsrc, int64_t n, bool f64, cudaStream_t s) {
    const int64_t m = n - 2;
    if (m <= 0) return cudaSuccess;
    dim3 block(32, 8), grid((unsigned)((m + 31) / 32), (unsigned)((m + 7) / 8));
    if (grid.y > 65535) return cudaErrorInvalidConfiguration;
    if (f64) jacobi2d_untiled<double><<<grid, block, 0, s>>>((double *)dst, (const double *)src, (const double *)bsrc, n);
    else jacobi2d_untiled<float><<<grid, block, 0, s>>>((float *)dst, (const float *)src, (const float *)bsrc, n);
    return cudaGetLastError();
}

cudaError_t launch_heat3d_untiled(void *dst, const void *src, int64_t n, bool f64, cudaStream_t s) {
    const int64_t m = n - 2;
    if (m <= 0) return cudaSuccess;
    dim3 block(32, 8), grid((unsigned)((m + 31) / 32), (unsigned)((m + 7) / 8), (unsigned)m);
    if (grid.y > 65535 || grid.z > 65535) return cudaErrorInvalidConfiguration;
    if (f64) heat3d_untiled<double><<<grid, block, 0, s>>>((double *)dst, (const double *)src, n);
    else heat3d_untiled<float><<<grid, block, 0, s>>>((float *)dst, (const float *)src, n);
    return cudaGetLastError();
}

}  // namespace eatss
