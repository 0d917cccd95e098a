/*
 * eatss.h -- C ABI of libeatss.so, the B200-native EATSS hot path.
 *
 * EATSS = Energy-Aware Tile Size Selection for affine programs on GPUs
 * (Jayaweera, Kong, Wang, Kaeli, CGO 2024).  Citations "P:<line>" refer to the
 * paper text line numbers; the section / table / equation is added.
 *
 * The library does four things, one group of calls each:
 *   1. describe an affine loop nest          eatss_desc_*
 *   2. select its tile-size vector           eatss_select_tiles     (Eq. 1-2)
 *   3. execute the tiled nest on a B200      eatss_plan, eatss_run  (Fig. 4)
 *   4. sweep / measure time and energy       eatss_sweep, eatss_energy_*
 *
 * Conventions (all calls):
 *   - Plain C types only.  Sizes are int64_t.  No exceptions cross the ABI.
 *   - Every call returns an eatss_status; on failure a thread-local message is
 *     available from eatss_last_error() until the next failing call on that thread.
 *   - Host arrays (dims, tiles, variants, results, plans) are caller-owned and only
 *     read/written during the call.
 *   - Device buffers are caller-owned device pointers (e.g. torch.Tensor.data_ptr()),
 *     row-major, contiguous, 16-byte aligned, non-aliasing, in the order documented
 *     per builtin below.  The library never frees them.
 *   - Descriptors are library-owned (create / destroy); a descriptor may be used by
 *     one thread at a time (eatss_run caches CUDA graphs inside it).  A descriptor may also
 *     own device scratch, allocated on the first run that needs it and freed with the
 *     descriptor: mttkrp's split partials / tensor-path block partials, SIMT syrk's A^T
 *     layout copy, eatss_run_host's device buffers.  Runs of ONE descriptor on different
 *     streams must therefore be ordered by the caller (they share that scratch).  The tensor
 *     engines' split operands (3xTF32 lo halves) are per-run scratch instead: allocated on the
 *     run's stream from a library-owned pool of the current device (cudaMallocFromPoolAsync) and
 *     freed on it after the run's launches, so they are never shared between runs.
 *   - eatss_run is asynchronous on `stream`: argument and launch-configuration
 *     errors are returned synchronously; device faults surface on the stream.
 *   - No CPU fallback exists: without a CUDA device eatss_run returns EATSS_E_CUDA.
 */
#ifndef EATSS_H
#define EATSS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define EATSS_API __attribute__((visibility("default")))
#else
#define EATSS_API
#endif

#define EATSS_ABI_VERSION 2
#define EATSS_MAX_LOOPS 8
#define EATSS_MAX_NESTS 4
#define EATSS_MAX_BUFFERS 16

typedef enum {
    EATSS_OK = 0,
    EATSS_E_INVALID = -1,     /* null pointer, bad dimension, tile entry <= 0, bad enum */
    EATSS_E_INFEASIBLE = -2,  /* select_tiles: the constrained tile space is empty */
    EATSS_E_CUDA = -3,        /* CUDA runtime error (message in eatss_last_error) */
    EATSS_E_NVML = -4,        /* NVML unavailable or failed */
    EATSS_E_UNSUPPORTED = -5, /* valid request this build does not implement */
    EATSS_E_NOMEM = -6
} eatss_status;

typedef enum { EATSS_F32 = 1, EATSS_F64 = 2 } eatss_dtype;

/*
 * Builtin affine programs.  dims / buffers per builtin (buffers in this order):
 *   EATSS_GEMM      dims (ni, nj, nk)          buffers {C[ni][nj] (in/out), A[ni][nk], B[nk][nj]}
 *                   C := alpha*A*B + beta*C  (PolyBench 3.2 gemm; Fig. 4)
 *   EATSS_2MM       dims (ni, nj, nk, nl)      buffers {tmp[ni][nj] (out), A[ni][nk], B[nk][nj],
 *                                                       C[nj][nl], D[ni][nl] (in/out)}
 *                   tmp := alpha*A*B; D := tmp*C + beta*D
 *   EATSS_3MM       dims (ni, nj, nk, nl, nm)  buffers {E[ni][nj] (out), A[ni][nk], B[nk][nj],
 *                                                       F[nj][nl] (out), C[nj][nm], D[nm][nl],
 *                                                       G[ni][nl] (out)}
 *                   E := A*B; F := C*D; G := E*F
 *   EATSS_SYRK      dims (ni, nj)              buffers {C[ni][ni] (in/out), A[ni][nj]}
 *                   C := alpha*A*A^T + beta*C (full square, PolyBench 3.2)
 *                   or dims (ni, nj, r0, rows): only rows [r0, r0+rows) of C (a row-block shard,
 *                   SURVEY §8(e)); buffers {C rows x ni (in/out), the full A[ni][nj]}
 *   EATSS_JACOBI2D  dims (n), tsteps           buffers {A[n][n] (in/out), B[n][n] (in/out)}
 *                   tsteps x { B = 0.2*(5-point of A); A = B } on the interior (PolyBench 3.2)
 *   EATSS_HEAT3D    dims (n), tsteps           buffers {A[n][n][n] (in/out), B[n][n][n] (in/out)}
 *                   tsteps x { B = f(A); A = f(B) } on the interior (PolyBench 4.x heat-3d)
 *   EATSS_CCSD_T_D1 dims (h3,h2,h1,p6,p5,p4,h7) or (d) buffers {t3 (in/out), t2[h7][p4][p5][h1],
 *                                                              v2[h3][h2][p6][h7]}
 *                   t3[h3][h2][h1][p6][p5][p4] -= sum_h7 t2[h7][p4][p5][h1]*v2[h3][h2][p6][h7]
 * Low-dimensional PolyBench 3.2 kernels (Fig. 7, Fig. 9),
 * fp32; one executor pass streams the matrix once and may serve two products (reading R-N7):
 *   EATSS_MVT       dims (n)                   buffers {x1[n] (in/out), x2[n] (in/out), y_1[n], y_2[n], A[n][n]}
 *                   x1[i] += A[i][j]*y_1[j];  x2[i] += A[j][i]*y_2[j]
 *   EATSS_ATAX      dims (nx, ny)              buffers {y[ny] (out), tmp[nx] (out), A[nx][ny], x[ny]}
 *                   tmp = A x;  y = A^T tmp
 *   EATSS_BICG      dims (nx, ny)              buffers {s[ny] (out), q[nx] (out), A[nx][ny], r[nx], p[ny]}
 *                   s = A^T r;  q = A p
 *   EATSS_GEMVER    dims (n)                   buffers {A[n][n] (in/out), x (in/out), w (in/out),
 *                                                       u1, v1, u2, v2, y, z} (vectors of n)
 *                   A += u1 v1^T + u2 v2^T;  x += beta A^T y;  x += z;  w += alpha A x
 * Non-PolyBench 4-D kernels (Figs. 10-11, 13), fp32; bodies and
 * sizes are our restatement (readings R-N8, R-N9):
 *   EATSS_MTTKRP    dims (ni, nj, nk, nl)      buffers {A[ni][nj] (in/out), B[ni][nk][nl], C[nk][nj], D[nl][nj]}
 *                   A[i][j] += sum_k sum_l B[i][k][l]*C[k][j]*D[l][j]  (mode-1 MTTKRP, loops i, j, k, l)
 *   EATSS_CONV2D    dims (n, f)                buffers {out[m][m] (out), inp[n][n], W[f][f]}, m = n - f + 1
 *                   out[i][j] = sum_p sum_q inp[i+p][j+q]*W[p][q]  (valid cross-correlation, loops i, j, p, q)
 * The tile vector has one entry per loop depth position (reading Q15): 3 for the
 * gemm family, 2 for jacobi-2d and the low-dimensional kernels, 3 for heat-3d, 7 for ccsd_t_d1
 * (h3,h2,h1,p6,p5,p4,h7), 4 for mttkrp (i,j,k,l) and conv-2d (i,j,p,q).  Stencil time loops are not
 * tiled.
 */
typedef enum {
    EATSS_GEMM = 0,
    EATSS_2MM = 1,
    EATSS_3MM = 2,
    EATSS_SYRK = 3,
    EATSS_JACOBI2D = 4,
    EATSS_HEAT3D = 5,
    EATSS_CCSD_T_D1 = 6,
    EATSS_MVT = 7,
    EATSS_ATAX = 8,
    EATSS_BICG = 9,
    EATSS_GEMVER = 10,
    EATSS_MTTKRP = 11,
    EATSS_CONV2D = 12
} eatss_builtin;

/* GPU parameters of the model: Table I + SM count + the
 * opt-in shared memory per block used by the B200-mode clamp (reading Q18). */
typedef struct {
    int64_t threads_per_block;  /* T_P_B */
    int64_t threads_per_warp;   /* T_P_W */
    int64_t regs_per_thread;    /* R_P_T (carried, unused by the model: reading Q24) */
    int64_t regs_per_sm;        /* R_P_S */
    int64_t regs_per_block;     /* R_P_B (carried, unused by the model) */
    int64_t l1_shared_bytes;    /* L1_SH: combined L1 + shared memory per SM, bytes */
    int64_t l2_bytes;           /* L2 */
    int64_t num_sms;
    int64_t max_smem_per_block; /* opt-in dynamic shared memory per block, bytes */
} eatss_gpu_params;

/* Model options (P:165-169 split factor, P:125/P:282 warp fraction). */
typedef struct {
    int32_t split_pct;  /* SPLIT_FACTOR as an integer percent 0..100 */
    int32_t warp_align; /* WARP_ALIGNMENT_FACTOR = warp_frac * T_P_W, in {4, 8, 16, 32} */
    int32_t mode;       /* 0 = paper mode, 1 = B200 mode (clamp M_SH at max_smem_per_block),
                           2 = tensor-core mode (reading T: MMA-legal tiles of the
                           tcgen05 executors under their TMEM / shared-memory capacities -- depth-3
                           contraction nests: Ti in {128, 256} (one CTA / a CTA pair), Tj in 16..256
                           step 16, Tk in {32, 64}; the 6-D contraction (ccsd_t_d1, T4): rows
                           Th1*Tp5*Tp4 <= 128, columns Th2*Tp6 <= 256, whole reduction; anything
                           else EATSS_E_UNSUPPORTED) */
} eatss_model_opts;

/* Optional report of eatss_select_tiles (values of the first nest unless noted). */
typedef struct {
    int32_t ls1_loop;   /* depth position of the CMA loop l_s1 */
    int32_t nrefs;      /* no.references, max over nests */
    int64_t obj;        /* OBJ at the optimum (Eq. 2, summed over nests) */
    int64_t n_feasible; /* number of feasible tile vectors */
    int64_t n_ties;     /* number of feasible vectors with OBJ == obj */
    int64_t m_l1, m_sh; /* M_L1, M_SH at the optimum (Eq. 1), max over nests */
    int64_t b_size;     /* B_size, max over nests */
    int64_t reg_sm;     /* REG_SM, max over nests */
    double solve_seconds;
} eatss_model_report;

/* Execution options stored in a descriptor (eatss_desc_set_exec). */
/* EATSS_ENGINE_UNTILED (jacobi-2d / heat-3d only; others return EATSS_E_UNSUPPORTED): the plain loop
 * nest without tiling -- one thread per interior point, neighbours from global memory, the tile
 * vector ignored -- the "untiled" baseline of BASELINE config 4 (same time loop and arithmetic). */
/* EATSS_ENGINE_TENSOR_F16 (fp32 gemm family): the tcgen05 GEMM with 3xFP16 operands -- each row of A and
 * column of B scaled by a power of two so its largest magnitude lies in [2^14, 2^15), split into fp16
 * hi + lo (22 significant bits, like 3xTF32), hi*hi + hi*lo + lo*hi accumulated in fp32 and the scales undone
 * exactly in the epilogue: fp32-level accuracy at fp16 MMA rate.  Same tile vector as EATSS_ENGINE_TENSOR
 * with Tk counted in fp16 elements: Ti in {128, 256}, Tj in 16..256 step 16, Tk in {16, 32, 64, 128}
 * (model mode 3).  Other builtins / fp64 descriptors: EATSS_E_UNSUPPORTED. */
typedef enum { EATSS_ENGINE_AUTO = 0, EATSS_ENGINE_SIMT = 1, EATSS_ENGINE_TENSOR = 2, EATSS_ENGINE_UNTILED = 3,
               EATSS_ENGINE_TENSOR_F16 = 4 } eatss_engine;
typedef struct {
    int32_t split_pct;  /* shared-memory carve-out preference, percent of max (sigma) */
    int32_t engine;     /* eatss_engine; AUTO = SIMT unless the tensor-core path applies; UNTILED: stencils */
    int32_t use_graph;  /* stencils: replay the time loop as one CUDA graph (default 1) */
    int32_t time_kernels; /* 1: record CUDA events around each nest's main compute kernel on the
                             run's stream (read back with eatss_last_kernel_ms); default 0.  The tensor
                             engines chain their split launch(es) and GEMM with programmatic dependent
                             launch, except under time_kernels = 1 (the events bracket the GEMM alone) */
    int32_t warp_align; /* SIMT contraction executor: lanes of every warp laid contiguously along the
                           CMA loop l_s1 -- the "SIMT length as a fraction of the warp size" (P:25,
                           P:125): WAF in {4, 8, 16, 32}, the remaining 32/WAF lanes of the warp
                           on consecutive rows of the tile; 0 (default) = the executor's own layout
                           (reported as eatss_launch_plan.simt_x).  Other values: EATSS_E_INVALID */
    int32_t carveout_exact; /* 1: request exactly split_pct as the L1/shared carve-out (the model's
                           sigma); 0 (default): split_pct is a lower bound that the SIMT
                           executors raise as far as their register-limited resident CTAs need.  The
                           value actually requested is reported by eatss_last_carveout */
} eatss_exec_opts;

/* Launch plan of one nest (tile -> GPU mapping, Fig. 4). */
typedef struct {
    int32_t nest;
    int32_t engine;        /* 1 SIMT, 2 tensor */
    int64_t grid_x, grid_y, grid_z;
    int32_t block_x, block_y;
    int32_t rm, rn, vec;   /* register micro-tile rows x cols, vector width along l_s1 */
    int32_t passes;        /* output passes per k-tile (1 = accumulators resident) */
    int32_t smem_bytes;    /* dynamic shared memory per CTA */
    int32_t a_in_smem;     /* SH_set operand staged in shared memory */
    int32_t b_in_smem;
    int32_t carveout_pct;  /* exec.split_pct (the request; the effective value: eatss_last_carveout) */
    int32_t simt_x;        /* lanes of a warp laid along l_s1 (= exec.warp_align when set) */
    int64_t tile[EATSS_MAX_LOOPS]; /* tile vector clipped to the extents */
} eatss_launch_plan;

/* One measured variant (energy = P_avg * t; PPW). */
typedef struct {
    double ms_per_run;
    double joules_per_run;
    double avg_watts;
    double tflops;
    double gflops_per_watt;
    double sm_mhz_median;
    int64_t runs;
    int32_t status;        /* eatss_status of this variant */
    int32_t reserved;
} eatss_measurement;

typedef struct eatss_kernel_desc eatss_kernel_desc;

/* ------------------------------------------------------------ descriptors */
EATSS_API eatss_status eatss_desc_builtin(eatss_builtin k, const int64_t *dims, int ndims, eatss_dtype dt,
                                int64_t tsteps, eatss_kernel_desc **out);
EATSS_API void eatss_desc_destroy(eatss_kernel_desc *d);
EATSS_API int eatss_desc_num_loops(const eatss_kernel_desc *d);   /* L = tile vector length */
EATSS_API int eatss_desc_num_nests(const eatss_kernel_desc *d);
EATSS_API int eatss_desc_num_buffers(const eatss_kernel_desc *d);
/* Element count of buffer i (documented order above); -1 on bad index. */
EATSS_API int64_t eatss_desc_buffer_elems(const eatss_kernel_desc *d, int i);
/* Algorithmic flop count of one run (2 per multiply-add; stencils: adds+muls as written). */
EATSS_API double eatss_desc_flops(const eatss_kernel_desc *d);
/* Algorithmic compulsory DRAM bytes of one run (each input read once, each output written once). */
EATSS_API double eatss_desc_bytes(const eatss_kernel_desc *d);
/* Scalars alpha, beta of gemm / 2mm / syrk (defaults 1.5, 1.2). */
EATSS_API eatss_status eatss_desc_set_scalars(eatss_kernel_desc *d, double alpha, double beta);
EATSS_API eatss_status eatss_desc_set_exec(eatss_kernel_desc *d, const eatss_exec_opts *o);
/* Derived model quantities of nest `nest` for warp alignment `waf`:
 * l_s1 position, nrefs, H weights [num_loops of that nest].  Any out pointer may be NULL. */
EATSS_API eatss_status eatss_desc_model_info(const eatss_kernel_desc *d, int nest, int waf, int32_t *ls1,
                                   int32_t *nrefs, int64_t *H);

/* ------------------------------------------------------------ GPU params */
EATSS_API eatss_status eatss_gpu_params_query(int device, eatss_gpu_params *out); /* cudaDeviceGetAttribute */
EATSS_API eatss_status eatss_gpu_params_b200(eatss_gpu_params *out);              /* B200 nominal */
EATSS_API eatss_status eatss_gpu_params_ga100(eatss_gpu_params *out);             /* Table I + III */

/* ------------------------------------------------------------ tile model */
/* Exact argmax of OBJ (Eq. 2) over the WAF-aligned domain subject to the
 * resource constraints with the deterministic tie-break of
 * DESIGN.md §2.2 rule 13.  Pure host code, deterministic, thread-safe.
 * tiles: caller array of eatss_desc_num_loops(d) entries.  rep may be NULL.
 * Returns EATSS_E_INFEASIBLE (tiles untouched) when no vector satisfies the constraints. */
EATSS_API eatss_status eatss_select_tiles(const eatss_kernel_desc *d, const eatss_gpu_params *g,
                                const eatss_model_opts *o, int64_t *tiles,
                                eatss_model_report *rep);

/* ------------------------------------------------------------ execution */
/* Launch plan for `tiles` (any entries >= 1 are accepted).  plans: caller
 * array of at least eatss_desc_num_nests(d) entries; *n_plans receives the count. */
EATSS_API eatss_status eatss_plan(const eatss_kernel_desc *d, const int64_t *tiles, eatss_launch_plan *plans,
                        int max_plans, int *n_plans);
/* Execute the program with tile vector `tiles` on `stream` (cudaStream_t as void*;
 * NULL = legacy default stream).  buffers: eatss_desc_num_buffers(d) device pointers. */
EATSS_API eatss_status eatss_run(const eatss_kernel_desc *d, const int64_t *tiles, void *const *buffers,
                       void *stream);
/* Execute only nest `nest` (0-based) -- used by the multi-GPU 3mm path between nests. */
EATSS_API eatss_status eatss_run_nest(const eatss_kernel_desc *d, int nest, const int64_t *tiles,
                            void *const *buffers, void *stream);
/* Execute the program on HOST buffers (the end-to-end path: host->device copies, the run, and
 * device->host copies of the outputs, all ordered on `stream`).  host_buffers: the
 * eatss_desc_num_buffers(d) arrays in the documented order, caller-owned host memory (page-locked
 * -- cudaHostAlloc / torch pin_memory -- for the copies to run asynchronously; pageable memory
 * works but serialises).  Inputs are read and outputs written per builtin (gemm: C in/out, A, B
 * in; 2mm: tmp out, D in/out; 3mm: E, F, G out; stencils: both arrays in/out; ccsd: t3 in/out).
 * The library keeps device copies per descriptor (allocated on first use, freed with the
 * descriptor).  row_blocks > 1 (gemm): the rows of C are processed in that many blocks of whole
 * i-tiles (CTA-pair rows on the tensor engine), B copied first, then each block's A and C rows
 * copied in, computed and copied out on separate streams, so copies in both directions overlap
 * the compute; every element sees the same operation order as one eatss_run.  Asynchronous:
 * the outputs are in host memory once `stream` has reached the end of the call (synchronize on
 * it); host buffers must stay valid until then.  Errors as eatss_run. */
EATSS_API eatss_status eatss_run_host(const eatss_kernel_desc *d, const int64_t *tiles, void *const *host_buffers,
                                      int64_t row_blocks, void *stream);
/* Indexing oracle: run the executor's exact point mapping of nest
 * `nest`, adding 1 to counts[point] (int32, row-major over the nest's loops) for every
 * iteration point executed.  Contraction nests and stencil sweeps only. */
EATSS_API eatss_status eatss_coverage(const eatss_kernel_desc *d, int nest, const int64_t *tiles,
                            int32_t *counts, void *stream);
/* Number of kernel launches one eatss_run issues with the descriptor's current exec options
 * (graph nodes counted individually; tensor engine: one prep launch -- the operand splits and
 * the split-k tail pre-pass -- plus the GEMM).  -1 on a bad argument. */
EATSS_API int64_t eatss_launches_per_run(const eatss_kernel_desc *d, const int64_t *tiles);
/* Device time in ms of the main compute kernel of each nest in the LAST eatss_run on `d`
 * issued with exec.time_kernels = 1 (tensor engine: the tcgen05 GEMM kernel alone, without
 * the prep launch; SIMT / ccsd: the nest's kernel; stencils: the whole time loop).
 * Writes min(cap, #nests) values to ms and the count to *n.  Blocks until those kernels have
 * finished.  E_INVALID if no timed run has been issued on `d`. */
EATSS_API eatss_status eatss_last_kernel_ms(const eatss_kernel_desc *d, float *ms, int32_t cap, int32_t *n);

/* Carve-out (percent) each nest's main kernel requested in the LAST eatss_run on `d` (the effective
 * value under exec.carveout_exact; -1 for kernels that set none, e.g. the tcgen05 engine, whose
 * shared memory is fixed by its stage ring).  Writes min(cap, #nests) values, the count to *n. */
EATSS_API eatss_status eatss_last_carveout(const eatss_kernel_desc *d, int32_t *pct, int32_t cap, int32_t *n);

/* ------------------------------------------------------------ energy */
/* NVML total-energy counter of `device` in millijoules since driver load. */
EATSS_API eatss_status eatss_energy_mj(int device, uint64_t *mj);
/* Instantaneous board power (milliwatts) and SM clock (MHz). */
EATSS_API eatss_status eatss_power_sample(int device, uint32_t *mw, uint32_t *sm_mhz);

/* Measure each variant (tile vector row v of `variants`, n rows of
 * eatss_desc_num_loops(d) entries): `warmup` runs, then back-to-back runs until
 * >= min_window_s, timed with CUDA events and metered with the NVML energy
 * counter; a background thread samples power and SM clock every 10 ms.
 * Synchronous.  A variant that fails is recorded (status) and the sweep goes on. */
EATSS_API eatss_status eatss_sweep(const eatss_kernel_desc *d, const int64_t *variants, int n,
                         void *const *buffers, int device, int warmup, double min_window_s,
                         eatss_measurement *results);

EATSS_API const char *eatss_last_error(void);
EATSS_API int eatss_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* EATSS_H */
