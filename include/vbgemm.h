/*
 * vbgemm.h — C-ABI of the B200-native variable-size batched GEMM
 *            (coordinated tiling + batching, Li et al. PPoPP'19).
 *
 * Operation (PAPER.md P31, §1; P133, §2.2), for every GEMM i of a batch:
 *
 *     C_i <- alpha_i * A_i x B_i + beta_i * C_i,
 *     A_i: M_i x K_i, B_i: K_i x N_i, C_i: M_i x N_i, all ROW-MAJOR with leading
 *     dimensions lda_i / ldb_i / ldc_i in ELEMENTS (reading C-15).
 *
 * BLAS rules (reading C-16): beta_i == 0 -> C_i is not read (NaN in C_i does not
 * propagate); M_i == 0 or N_i == 0 -> GEMM i is a no-op; K_i == 0 -> C_i = beta_i * C_i.
 * alpha/beta are fp32 for every dtype.  bf16/fp16 inputs accumulate in fp32 and round
 * to nearest-even on output; fp32 accumulates in fp32 with FFMA (reading C-17).
 *
 * The method is two host phases and one device kernel (P163 Fig. 4, P167):
 *   plan:  tiling engine (§4.2.3, P245-255, Eq. 1) -> tile enumeration ->
 *          batching engine (§5, P259-270: threshold / binary) -> the five auxiliary
 *          arrays of §6 (P282-284, Fig. 6) packed as device tile descriptors.
 *   exec:  persistent sm_100a kernels walk the descriptors (Fig. 7, P294-312): tcgen05 for
 *          bf16/fp16 (a 2-SM cluster launch for pair tiles, then a 1-SM launch), packed-FFMA2
 *          for fp32.
 * vb_plan_conv maps a batch of 2-D convolutions onto the same engines (implicit GEMM).
 *
 * Conventions
 *  - Every call returns vb_status; nothing throws across the ABI.  On failure a
 *    human-readable reason is available from vb_last_error() (thread-local).
 *  - "HOST" = pointer to host memory, read during the call only.
 *    "DEVICE" = pointer to device memory of the plan's device.
 *  - Streams are passed as void* holding a cudaStream_t (NULL = legacy default stream).
 */
#ifndef VBGEMM_H_
#define VBGEMM_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  VB_OK = 0,
  VB_ERR_INVALID_ARG = 1,   /* bad size, null pointer, inconsistent schedule            */
  VB_ERR_ALIGNMENT = 2,     /* ld * sizeof(elem) not a multiple of 16 bytes              */
  VB_ERR_UNSUPPORTED = 3,   /* not an sm_100 device, dtype/table mismatch, host-only plan */
  VB_ERR_OOM = 4,           /* device or host allocation failed                          */
  VB_ERR_CUDA = 5,          /* a CUDA runtime / driver call failed                       */
  VB_ERR_INTERNAL = 6
} vb_status;

typedef enum { VB_F32 = 0, VB_BF16 = 1, VB_F16 = 2 } vb_dtype;   /* one dtype per batch */

/* Batching policy (§5): THRESHOLD = TLP first (P261), BINARY = ILP first (P263-270),
 * NONE = one tile per block (the un-batched baseline, P259 "a thread block is
 * responsible for a single tile"), AUTO = on-line choice between THRESHOLD and BINARY by
 * the random forest over (mean M, mean N, mean K, batch size) (P272-274), trained offline
 * on B200 (reading C-25); vb_plan_policy reports the choice. */
typedef enum {
  VB_BATCH_THRESHOLD = 0, VB_BATCH_BINARY = 1, VB_BATCH_NONE = 2, VB_BATCH_AUTO = 3
} vb_policy;

/* Strategy tables.
 *  VB_TABLE_V100        PAPER.md Table 2 (P204-214) with the V100 constants (P290):
 *                       TLP threshold 65536, theta 256, versions T = 256 / 128.
 *  VB_TABLE_B200_FFMA   Table 2 shapes without 128x128 (16x16 ... 128x64 / 64x128) with the
 *                       128-thread sub-tiles for the fp32 FFMA kernel, T = 128, B200 constants.
 *  VB_TABLE_B200_TC     tcgen05 table (bf16/fp16): 64x32, 128x32, 64x64, 128x64, 64x128,
 *                       128x128, 64x256, 128x256 C tiles and 2-SM pair tiles 256x{64,128,256,512},
 *                       BK = 64, T = 256; availability tested against max(M, 128) x max(N, 256)
 *                       (reading C-1b).
 *  VB_TABLE_DEFAULT     B200_FFMA for VB_F32, B200_TC for VB_BF16 / VB_F16. */
typedef enum {
  VB_TABLE_DEFAULT = 0, VB_TABLE_V100 = 1, VB_TABLE_B200_FFMA = 2, VB_TABLE_B200_TC = 3
} vb_table;

/* Platform constants, set offline per platform (P253, P290).  0 = table default. */
typedef struct {
  int32_t table_id;        /* vb_table                                                  */
  int64_t tlp_threshold;   /* TLP threshold of the tiling engine (Eq. 1 units: threads) */
  int32_t theta;           /* K-workload threshold theta of the batching engine (P259)  */
} vb_tuning;

typedef struct vb_plan *vb_plan_t;

/* ------------------------------------------------------------------------------------
 * vb_plan_vbatched — run the tiling and batching engines for one batch shape.
 *
 *  device   CUDA device ordinal (must be sm_100), or -1 for a HOST-ONLY plan: planning
 *           and vb_plan_export work, vb_exec_vbatched returns VB_ERR_UNSUPPORTED.
 *  dt       element type of A, B and C.
 *  batch    number of GEMMs (>= 0; 0 gives a valid empty plan).
 *  M,N,K    HOST int32[batch], each >= 0.
 *  lda,ldb,ldc  HOST int32[batch], leading dimensions in elements, row-major:
 *           lda >= K, ldb >= N, ldc >= N, and ld * sizeof(elem) % 16 == 0
 *           (else VB_ERR_ALIGNMENT).
 *  policy   batching policy.   tuning: nullable (all defaults).
 *  out      receives the plan.  The plan owns its device descriptors and workspace.
 * Device plans upload the compact schedule (Tile[], slot order, GEMM segments, per-GEMM
 * parameters, tensor-map templates) in one copy on a private stream, expand it on the device
 * into per-slot tile records and per-GEMM tensor maps, and synchronise that stream before
 * returning.  The workspace comes from a per-device stream-ordered memory pool that keeps
 * freed memory for the next plan (VB_NO_PLAN_POOL=1 in the environment: plain cudaMalloc).
 * ------------------------------------------------------------------------------------ */
vb_status vb_plan_vbatched(int device, vb_dtype dt, int32_t batch,
                           const int32_t *M, const int32_t *N, const int32_t *K,
                           const int32_t *lda, const int32_t *ldb, const int32_t *ldc,
                           vb_policy policy, const vb_tuning *tuning, vb_plan_t *out);

/* ------------------------------------------------------------------------------------
 * vb_plan_from_schedule — build a plan from a caller-supplied tiling + batching scheme
 * ("through the five auxiliary arrays, we can describe any possible batching scheme",
 * P282).  Arrays are HOST:
 *   gemm_row[batch]        table row (strategy shape) per GEMM (Tiling[] of Fig. 7, C-12)
 *   version_T              thread version, must be one of the table's versions
 *   block_ptr[n_blocks+1]  Tile[] of Fig. 6: block b owns slots [block_ptr[b], block_ptr[b+1])
 *   tile_gemm/tile_y/tile_x[n_slots]  GEMM[], Y_Coordinate[], X_Coordinate[] per slot
 * Validated: CSR monotone from 0, every C tile of every GEMM exactly once.
 * ------------------------------------------------------------------------------------ */
vb_status vb_plan_from_schedule(int device, vb_dtype dt, int32_t batch,
                                const int32_t *M, const int32_t *N, const int32_t *K,
                                const int32_t *lda, const int32_t *ldb, const int32_t *ldc,
                                int32_t table_id, const int32_t *gemm_row, int32_t version_T,
                                int32_t n_blocks, const int32_t *block_ptr,
                                const int32_t *tile_gemm, const int32_t *tile_y,
                                const int32_t *tile_x, vb_plan_t *out);

/* ------------------------------------------------------------------------------------
 * vb_plan_conv — a batch of 2-D convolutions run as batched IMPLICIT GEMMs (SURVEY.md §8(f)
 * NEXT-3): "GEMM is the core of convolution ... the im2col approach transforms the
 * convolution into a GEMM" with M = #filters, N = H*W*images, K = Cin*kh*kw (PAPER.md P45,
 * P338-352).  Here the im2col matrix is never materialised: the kernel's A-operand producer
 * loads it tile by tile with TMA im2col-mode copies straight from the NHWC input, so each
 * convolution reads its input, weights and output once.  Orientation (transposed against
 * P45 so that the output is NHWC): the GEMM is
 *     Y[p][co] = alpha * sum_{kh,kw,ci} X[n][h+kh-pad][w+kw-pad][ci] * Wt[kh][kw][ci][co]
 *                + beta * Y[p][co]
 * with p = (n*Hout + h)*Wout + w the output pixel (GEMM row, M = nb*Hout*Wout), co the output
 * channel (GEMM column, N = Cout) and K = KH*KW*Cin ordered (kh, kw, ci); X outside the
 * image reads as 0.  Hout = H + 2*pad - KH + 1, Wout = W + 2*pad - KW + 1 (stride 1,
 * dilation 1; "same" convolution for pad = (KH-1)/2).
 *  dt       VB_BF16 or VB_F16 (tensor-core path; fp32 accumulation).
 *  desc     HOST vb_conv_desc[batch].  Layouts, all row-major, element strides:
 *           X  (exec's A[i]): NHWC, nb x H x W x Cin, dense (pixel stride Cin).
 *           Wt (exec's B[i]): HWIO, the (KH*KW*Cin) x Cout GEMM B matrix, row stride ldb.
 *           Y  (exec's C[i]): NHWC output, (nb*Hout*Wout) x Cout, row stride ldc -- an
 *              inception module's branches write into one concatenated tensor by passing
 *              its channel offset in the pointer and the total channel count as ldc.
 *  Constraints (else VB_ERR_INVALID_ARG / VB_ERR_ALIGNMENT): sizes >= 1, KH == KW <= 8,
 *           0 <= pad < KH, Hout, Wout >= 1, Cin % 8 == 0, ldb >= Cout, ldc >= Cout,
 *           ldb % 8 == 0, ldc % 8 == 0 (16-byte rows), nb*H*W*Cin < 2^31.
 * The tiling and batching engines run on (M, N, K) exactly as vb_plan_vbatched (1-SM
 * strategies only); execution is vb_exec_vbatched / vb_plan_bind + vb_exec_bound with the
 * pointer arrays above.  Ownership and errors as vb_plan_vbatched.
 * ------------------------------------------------------------------------------------ */
typedef struct {
  int32_t nb, H, W, Cin, Cout, KH, KW, pad;
  int32_t ldb, ldc;
} vb_conv_desc;

vb_status vb_plan_conv(int device, vb_dtype dt, int32_t batch, const vb_conv_desc *desc,
                       vb_policy policy, const vb_tuning *tuning, vb_plan_t *out);

/* ------------------------------------------------------------------------------------
 * vb_exec_vbatched — enqueue the batched GEMM on `stream`.
 *  A, B     DEVICE arrays [batch] of DEVICE pointers to the matrices (16-byte aligned).
 *  C        DEVICE array  [batch] of DEVICE pointers (16-byte aligned), read+written.
 *  alpha, beta  DEVICE fp32 arrays [batch].
 *  stream   cudaStream_t as void*.
 * Never allocates, never synchronises.  Enqueues at most three kernels: the descriptor
 * prep kernel (tensor-map address patch and work-counter reset), then the GEMM kernel(s) --
 * fp32: one FFMA kernel; bf16/fp16: the 2-SM pair kernel (if the plan has pair tiles) and
 * the 1-SM kernel.  The GEMM kernels are launched with programmatic stream serialisation
 * (they start their setup while the prep kernel runs and wait for it before touching its
 * output).  All of it may be captured in a CUDA graph.  The caller
 * keeps every buffer alive until the stream work completes.  A plan may be re-executed
 * with new pointers / alpha / beta, but not concurrently on two streams.
 * Returns VB_ERR_CUDA if a launch fails (vb_last_error() has the CUDA message).
 * ------------------------------------------------------------------------------------ */
vb_status vb_exec_vbatched(vb_plan_t plan, const void *const *A, const void *const *B,
                           void *const *C, const float *alpha, const float *beta, void *stream);

/* ------------------------------------------------------------------------------------
 * vb_plan_bind / vb_exec_bound — vb_exec_vbatched split in two for callers that run the
 * same buffers many times (e.g. a fixed batch in DNN training, P272):
 *  vb_plan_bind   records the DEVICE pointer arrays A, B, C in the plan and enqueues the
 *                 descriptor prep kernel (tensor-map address patch) on `stream`.  The arrays
 *                 and matrices must stay valid until the last vb_exec_bound using them ends.
 *  vb_exec_bound  enqueues only the GEMM kernel(s), using the last bound pointers and the
 *                 given alpha/beta (DEVICE fp32 [batch]).  VB_ERR_INVALID_ARG if never bound.
 *                 The GEMM kernels reset their own work-list counters when they finish, so
 *                 vb_exec_bound may be repeated, or captured alone in a CUDA graph and replayed.
 * vb_exec_vbatched(...) == vb_plan_bind(...) + vb_exec_bound(...).
 * ------------------------------------------------------------------------------------ */
vb_status vb_plan_bind(vb_plan_t plan, const void *const *A, const void *const *B, void *const *C,
                       void *stream);
vb_status vb_exec_bound(vb_plan_t plan, const float *alpha, const float *beta, void *stream);

/* ------------------------------------------------------------------------------------
 * vb_plan_info — sizes of the plan (any output pointer may be NULL).
 *   n_tiles, n_blocks   tile slots and blocks (work lists) of the batching scheme
 *   workspace_bytes     device bytes owned by the plan (0 for host-only plans)
 *   version_T           chosen thread version of the tiling engine
 *   launches_per_exec   kernels one vb_exec_vbatched enqueues
 * ------------------------------------------------------------------------------------ */
vb_status vb_plan_info(vb_plan_t plan, int64_t *n_tiles, int64_t *n_blocks,
                       int64_t *workspace_bytes, int32_t *version_T, int32_t *launches_per_exec);

/* vb_plan_policy — the batching policy the plan was built with (VB_BATCH_AUTO resolved to
 * THRESHOLD or BINARY; -1 for a plan from vb_plan_from_schedule). */
vb_status vb_plan_policy(vb_plan_t plan, int32_t *policy);

/* ------------------------------------------------------------------------------------
 * vb_plan_tune — "for the case where the batch size and the size of each matrix are fixed
 * ... we can try both two batching heuristics and choose the better one" (P272).
 * Plans the batch with THRESHOLD and with BINARY batching (same arguments as
 * vb_plan_vbatched), runs each once to warm up and then `reps` times on `stream` with the
 * caller's DEVICE buffers (as vb_exec_vbatched), times them with CUDA events, keeps the
 * faster plan (ties keep THRESHOLD) and destroys the other.  *out is bound to A, B, C.
 *  ms   nullable HOST float[2]: mean ms per run of THRESHOLD and BINARY.
 * SYNCHRONISES `stream`.  C is used as scratch: it is overwritten (1 + reps) times per
 * candidate and holds an unspecified value on return.  Errors as vb_plan_vbatched /
 * vb_exec_vbatched; VB_ERR_UNSUPPORTED for device < 0.
 * ------------------------------------------------------------------------------------ */
vb_status vb_plan_tune(int device, vb_dtype dt, int32_t batch,
                       const int32_t *M, const int32_t *N, const int32_t *K,
                       const int32_t *lda, const int32_t *ldb, const int32_t *ldc,
                       const vb_tuning *tuning, const void *const *A, const void *const *B,
                       void *const *C, const float *alpha, const float *beta, int32_t reps,
                       void *stream, vb_plan_t *out, float *ms);

/* vb_plan_export — the five auxiliary arrays of §6 (HOST outputs, sized by vb_plan_info):
 *   block_ptr[n_blocks+1], tile_gemm/tile_y/tile_x[n_tiles], gemm_strategy[batch]
 *   (strategy id = version_index * table_rows + row, reading C-14).
 * For device plans the arrays are decoded from the DEVICE copy of the descriptors (a
 * synchronous device-to-host read), so the export proves what the kernel walks. */
vb_status vb_plan_export(vb_plan_t plan, int32_t *block_ptr, int32_t *tile_gemm,
                         int32_t *tile_y, int32_t *tile_x, int32_t *gemm_strategy);

/* vb_plan_debug_tmaps — diagnostic: copy the plan's per-GEMM tensor maps (DEVICE copy,
 * batch x 6 x 128 bytes for bf16/fp16 plans, batch x 2 x 128 for fp32) to the HOST buffer `out`
 * of `bytes` bytes; *needed receives the size (0 for host-only plans).  Tests use it to check
 * that maps built on the device from templates equal the host encoder's maps bit for bit
 * (the environment variable VB_TMAPS_HOST=1 makes vb_plan_* encode every map on the host).
 * Errors: VB_ERR_INVALID_ARG (null plan, buffer too small), VB_ERR_CUDA. */
vb_status vb_plan_debug_tmaps(vb_plan_t plan, void *out, int64_t bytes, int64_t *needed);

/* vb_debug_tile_cols — diagnostic: the column range [*n0, *end) that column tile x of a
 * tensor-core GEMM with N columns and strategy width BX covers in the kernels (DESIGN.md reading
 * C-26: the GEMM's ceil(N / G) column chunks, G = min(64, BX), shared as evenly as whole chunks
 * allow among its ceil(N / BX) column tiles), and *x_back = the tile index the plan export
 * decodes from *n0.  Host only, no GPU needed.
 * Errors: VB_ERR_INVALID_ARG (null outputs, N < 1, BX not a multiple of 16 in [16, 512],
 * x outside [0, ceil(N / BX))). */
vb_status vb_debug_tile_cols(int32_t x, int32_t N, int32_t BX, int32_t *n0, int32_t *end, int32_t *x_back);

/* vb_debug_set_coverage — diagnostic, coverage-counter build only (libvbgemm_cov.so, compiled
 * with -DVB_COVERAGE; SURVEY.md §4 "each C element written exactly once"): from now on every
 * element a GEMM kernel's epilogue stores on `device` also adds 1 to the int32 counter at the
 * same element offset from `c_base` in the DEVICE array `counts` (caller-owned, zeroed by the
 * caller, one counter per element of the C arena that starts at `c_base`, element size
 * `elem_bytes`).  counts = NULL switches counting off.  The product build returns
 * VB_ERR_UNSUPPORTED; VB_ERR_INVALID_ARG for a missing base or element size. */
vb_status vb_debug_set_coverage(int device, int32_t *counts, const void *c_base, int32_t elem_bytes);

/* vb_plan_tiler_trace — per round of the tiling engine: TLP (Eq. 1) and version T.
 * Writes min(cap, rounds) entries; *n_rounds receives the total number of rounds. */
vb_status vb_plan_tiler_trace(vb_plan_t plan, int32_t cap, int64_t *tlp, int32_t *version_T,
                              int32_t *n_rounds);

vb_status vb_plan_destroy(vb_plan_t plan);

/* ------------------------------------------------------------------------------------
 * vb_shard_lpt — FLOP-balanced GEMM -> rank assignment for multi-GPU runs (BASELINE.json
 * north_star).  Host only, deterministic: GEMMs in order of (-2*M*N*K, index) each go to
 * the least-loaded rank, ties to the lowest rank.  M,N,K HOST int32[batch];
 * rank_of HOST int32[batch] output.
 * ------------------------------------------------------------------------------------ */
vb_status vb_shard_lpt(int32_t batch, const int32_t *M, const int32_t *N, const int32_t *K,
                       int32_t n_ranks, int32_t *rank_of);

/* ------------------------------------------------------------------------------------
 * vb_fill_uniform_batch — device input generator (the paper artifact's gen_data, P428):
 * for each i < batch, fills the rows[i] x cols[i] matrix at ptrs[i] (leading dimension
 * ld[i] elements; padding untouched) with the counter-hash draw of vbinputs/__init__.py:
 * value(r,c) = ((splitmix64(mkey(seed, gemm_id[i], operand) + r*cols[i] + c) >> 40)
 * * 2^-23 - 1), rounded to nearest-even for bf16/fp16.
 * rows, cols, ld: DEVICE int32[batch]; ptrs: DEVICE void*[batch]; gemm_id: DEVICE
 * int64[batch]; total_elems: sum of rows*cols (host value, sizes the grid).
 * ------------------------------------------------------------------------------------ */
vb_status vb_fill_uniform_batch(vb_dtype dt, int32_t batch, const int32_t *rows,
                                const int32_t *cols, const int32_t *ld, void *const *ptrs,
                                const int64_t *gemm_id, uint64_t seed, int32_t operand,
                                int64_t total_elems, void *stream);

/* vb_fill_alpha_beta — DEVICE fp32 alpha[batch], beta[batch] for GEMM ids gemm_id[i]
 * (DEVICE int64): alpha = 0.5 + u*2^-24, beta = u*2^-23 - 1 (operands 3 and 4). */
vb_status vb_fill_alpha_beta(int32_t batch, const int64_t *gemm_id, uint64_t seed,
                             float *alpha, float *beta, void *stream);

/* Device properties used by the planner: SM count and compute capability. */
vb_status vb_device_info(int device, int32_t *sm_count, int32_t *cc_major, int32_t *cc_minor);

const char *vb_status_str(vb_status s);
const char *vb_last_error(void);       /* thread-local detail of the last failing call */
const char *vb_version(void);

#ifdef __cplusplus
}
#endif
#endif /* VBGEMM_H_ */
