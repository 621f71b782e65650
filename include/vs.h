/*
 * vs.h — C ABI of libvs: column-vector-sparse fp16 SpMM / SDDMM for B200 (sm_100a).
 *
 * Method: Chen, Qu, Liu, Ding, Xie, "Efficient Tensor Core-Based GPU Kernels for
 * Structured Sparsity under Reduced Precision", SC'21.  "P:n" below = line n of the
 * paper text (reference PAPER.md).
 *
 * Column-vector sparse encoding (§4.2, Fig. 8):
 *   A matrix of M rows and K columns is cut into W = ceil(M/V) row windows of V rows.
 *   Inside window w, column k is a "column vector" A[wV .. wV+V-1][k].  Only nonzero
 *   column vectors are stored, CSR-style:
 *     row_ptr[W+1]   int32, row_ptr[0] = 0, non-decreasing; window w owns vectors
 *                    p in [row_ptr[w], row_ptr[w+1]).
 *     col_idx[nnz_v] int32, the column k of vector p (the encoder emits ascending k).
 *     vals[nnz_v*V]  fp16, vector-major: vals[p*V + r] = A[wV + r][col_idx[p]]
 *                    ("elements within each nonzero column vector are stored in
 *                    consecutive addresses, and the consecutive vectors in the same
 *                    row are also consecutive").  Rows wV+r >= M of the last
 *                    window are padding and hold +0.0.
 *   V is 1, 2, 4 or 8 (V=1 is plain scalar CSR).
 *
 * General conventions (apply to every entry point):
 *   - All matrix / index pointers are DEVICE pointers (unless a name ends in _host).
 *     fp16 buffers are IEEE binary16 passed as void*.
 *   - Every call is stream-ordered on `stream` (a cudaStream_t; NULL = legacy default
 *     stream) and asynchronous, except where a phase below says it synchronises.
 *   - Ownership: the caller allocates and frees every buffer.  The library allocates no
 *     device memory and keeps no global mutable state except a once-initialised cache of
 *     device attributes, so calls are thread-safe.
 *   - Errors: argument checks run on the host before anything is enqueued.  Bad V,
 *     negative sizes, a NULL required pointer -> VS_ERROR_INVALID_VALUE; device is not
 *     sm_100 -> VS_ERROR_NOT_SUPPORTED; an fp16 pointer not 2-byte aligned, vals not
 *     2-byte aligned or an int32 pointer not 4-byte aligned -> VS_ERROR_MISALIGNED;
 *     a failed launch -> VS_ERROR_CUDA.  Faults inside kernels surface asynchronously
 *     as in CUDA.  No C++ exception ever crosses this ABI.
 *   - Preconditions not checked (undefined behaviour if violated): row_ptr[0] == 0 and
 *     non-decreasing; 0 <= col_idx < K (SpMM) / < N (SDDMM); output buffers do not
 *     alias inputs.  Kernels do not rely on col_idx order (duplicates sum in SpMM).
 *   - Sizes are int64; indices int32 (so nnz_v < 2^31); all address arithmetic is 64-bit.
 *   - Any M, N, K >= 0 is accepted: the fast path wants 16-byte aligned dense operands
 *     and N % 8 == 0 (SpMM) / K % 8 == 0 (SDDMM); everything else takes a guarded path
 *     that gives the same results.
 *   - Arithmetic: fp16 x fp16 products accumulated in fp32 (HMMA.884.F32.F32),
 *     results rounded to fp16 round-to-nearest-even (output precision is a reading,
 *     DESIGN.md R1).  Results are deterministic (no atomics on outputs).
 */
#ifndef VS_H_
#define VS_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Same type as cudaStream_t (struct CUstream_st*); declared here so this header does
   not need the CUDA headers. */
typedef struct CUstream_st* vs_stream_t;

typedef enum {
  VS_SUCCESS = 0,
  VS_ERROR_INVALID_VALUE = 1,
  VS_ERROR_NOT_SUPPORTED = 2,
  VS_ERROR_CUDA = 3,
  VS_ERROR_MISALIGNED = 4
} vs_status_t;

/* Human-readable name of a status code (static storage, never NULL). */
const char* vs_status_string(vs_status_t s);

/* Library version as MAJOR*10000 + MINOR*100 + PATCH. */
int vs_version(void);

/*
 * vs_encode_colvec — dense matrix or mask [M x K] -> column-vector CSR with grain V.
 * Defined by §4.2 P:622-633 and the worked example of Fig. 8.
 *
 *   dense : fp16 [M x K] row-major (leading dimension K), or NULL.
 *   mask  : uint8 [M x K] row-major, or NULL.  At least one of dense / mask is required.
 *   Keep predicate for window w, column k:
 *     mask != NULL : any_{r<V, wV+r<M} mask[wV+r][k] != 0
 *     mask == NULL : any_{r<V, wV+r<M} bits(dense[wV+r][k]) != 0   (so -0.0 is kept;
 *                    a kept vector may contain zeros, as (0,1) in Fig. 8)
 *   row_ptr : int32 [W+1] output, W = ceil(M/V).  Always written.
 *
 *   Count mode (col_idx == NULL): writes row_ptr only.  If nnz_vec_host != NULL, the call
 *     synchronises `stream` and stores nnz_v = row_ptr[W] into *nnz_vec_host.
 *   Full mode (col_idx != NULL): writes row_ptr, col_idx[nnz_v] (ascending k inside each
 *     window) and, if vals != NULL, vals[nnz_v*V] (requires dense != NULL; rows >= M
 *     padded with +0.0; vals must be 2-byte aligned).  Capacity precondition: col_idx
 *     holds >= nnz_v entries and vals >= nnz_v*V (e.g. from a previous count-mode call,
 *     or the bound W*K).  Asynchronous unless nnz_vec_host != NULL (then it synchronises
 *     and stores nnz_v).
 *   M == 0 or K == 0 gives row_ptr = 0 everywhere and nnz_v = 0.
 *   ceil(M/V) * K >= 2^31 (nnz_v could overflow the int32 row_ptr) -> VS_ERROR_NOT_SUPPORTED,
 *   before anything is enqueued.
 */
vs_status_t vs_encode_colvec(int64_t M, int64_t K, int V,
                             const void* dense, const uint8_t* mask,
                             int32_t* row_ptr, int32_t* col_idx, void* vals,
                             int64_t* nnz_vec_host, vs_stream_t stream);

/*
 * vs_transpose_colvec — column-vector encoding (grain V) of A^T [K x M] from the encoding
 * of A [M x K].  The training-side operand: with Y = W X (SpMM), the
 * backward pass needs dX = W^T dY, "W^T ... encode[d] with our column-vector sparse
 * encoding" (§8 Case 1; the transposed operand of the Discussion).
 *
 *   Window kw of A^T covers columns kw*V .. kw*V+V-1 of A; vector (kw, m) holds
 *   A[m][kw*V + j], j < V (j with kw*V + j >= K is padding, +0.0).  It is kept iff one of
 *   its V fp16 bit patterns is nonzero (vals != NULL; the keep rule of vs_encode_colvec, so
 *   the result is bit-identical to encoding the dense transpose), or iff the A vector it
 *   comes from is stored (vals == NULL: pattern-only transpose of a mask, no valsT).  For
 *   patterns of square V x V blocks each block gives exactly V vectors.
 *
 *   row_ptr[W+1], col_idx[nnz_v], vals[nnz_v*V] (or NULL): A, W = ceil(M/V); col_idx must
 *     not repeat inside a window (the encoder's output satisfies this).
 *   rowT_ptr : int32 [ceil(K/V) + 1] output, always written.
 *   colT_idx : int32 [nnzT] output (ascending m inside each window), or NULL = count mode.
 *   valsT    : fp16 [nnzT * V] output (requires vals), or NULL.
 *   workspace: device buffer of vs_transpose_colvec_workspace(M, K, V) bytes (int32
 *              aligned), scratch for the call: a dense ceil(K/V) x ceil(M/V) int32 table of
 *              per-(column group, window) row masks, i.e. O(M*K/V^2) bytes whatever nnz_v is
 *              (4*M*K bytes at V = 1: twice the dense fp16 matrix), memset on every full and
 *              count call.  Keep it between calls when the pattern will be refreshed.
 *   nnzT_host: if non-NULL, the call synchronises `stream` and stores rowT_ptr[ceil(K/V)].
 *   Count mode (colT_idx == NULL) writes rowT_ptr only; full mode needs colT_idx / valsT
 *   capacities >= nnzT (from a count-mode call, or the bound ceil(K/V) * M).
 *   Deterministic: no atomics on outputs (the workspace collects per-(column group,
 *   window) row masks with atomicOr, which is order-independent).
 */
int64_t vs_transpose_colvec_workspace(int64_t M, int64_t K, int V);
/*
 * vs_transpose_colvec_values — refreshes valsT for new values of A with an unchanged
 * pattern (a training step updates W's values, not its pattern): rowT_ptr / colT_idx and the
 * workspace must come from a previous full-mode vs_transpose_colvec call on the same row_ptr
 * / col_idx.  valsT[q*V + j] = A[colT_idx[q]][kw*V + j] from the new vals for every vector q
 * of that pattern (elements of A that are not stored give +0.0).  Two kernels, asynchronous.
 *   Build a pattern that will be refreshed with vals == NULL (pattern-only): every stored
 *   element of A (rows < M) then has its slot in valsT.  A pattern built FROM VALUES holds
 *   only the elements that were nonzero at build time; a stored element that was +0.0 then
 *   and is nonzero now is not placed by the refresh (its contribution to W^T is lost).
 */
vs_status_t vs_transpose_colvec_values(int64_t M, int64_t K, int V,
                                       const int32_t* row_ptr, const int32_t* col_idx,
                                       const void* vals, const int32_t* rowT_ptr, void* valsT,
                                       const void* workspace, vs_stream_t stream);
vs_status_t vs_transpose_colvec(int64_t M, int64_t K, int V,
                                const int32_t* row_ptr, const int32_t* col_idx, const void* vals,
                                int32_t* rowT_ptr, int32_t* colT_idx, void* valsT,
                                void* workspace, int64_t* nnzT_host, vs_stream_t stream);

/*
 * vs_spmm — C[M x N] = A[M x K] * B[K x N], A sparse in column-vector CSR.
 * Problem statement §4.1 P:571-588 (B, C row-major; A in CSR); kernel §5.3-5.4
 * P:846-921 (each output tile V x TileN).
 *
 *   row_ptr[W+1], col_idx[nnz_v], vals[nnz_v*V] : A as above, W = ceil(M/V).
 *   B : fp16 [K x N] row-major.   C : fp16 [M x N] row-major, fully overwritten
 *   (beta = 0; windows without vectors produce zeros).
 *   C[i][j] = fp16_rn( sum_{p in window i/V} vals[p*V + i%V] * B[col_idx[p]][j] ),
 *   summed in fp32.
 *   M == 0 or N == 0: no-op.  K == 0 or nnz_v == 0: C is zero-filled.
 */
vs_status_t vs_spmm(int64_t M, int64_t K, int64_t N, int V,
                    const int32_t* row_ptr, const int32_t* col_idx, const void* vals,
                    const void* B, void* C, vs_stream_t stream);

/*
 * vs_spmm_scatter — vs_spmm whose output tiles are stored into n_dst destinations: the fused
 * replicated-output epilogue of the multi-GPU N-panel sharding (the
 * paper is single-GPU, the sharding follows the north star).  For d < n_dst:
 *   C_dst[d][i*ldc + j] = fp16_rn( sum_p vals[p*V + i%V] * B[col_idx[p]][j] ),  i < M, j < N,
 * bit-identical to vs_spmm's C[i][j]; columns >= N of a destination row are not touched.
 *   B      : fp16 [K x N] row-major (this rank's panel).
 *   C_dst  : HOST array of n_dst (1 <= n_dst <= VS_SPMM_SCATTER_MAX) device-addressable
 *            pointers, read during the call: e.g. every rank's symmetric-memory C buffer
 *            (peer pointers over NVLink / NVSwitch), each offset to this rank's first column,
 *            so one kernel writes the rank's panel into every replica of the row-major C.
 *   ldc    : leading dimension (elements) of every destination, ldc >= N.
 * The caller orders the peers' reads after the stores (e.g. a symmetric-memory barrier on
 * the stream).  Errors as vs_spmm, plus VS_ERROR_INVALID_VALUE for a NULL C_dst, n_dst out of
 * range or ldc < N.  The 16-byte store path needs 16-byte aligned destinations and
 * ldc % 8 == 0; anything else takes the guarded path (same bits).
 */
#define VS_SPMM_SCATTER_MAX 8
vs_status_t vs_spmm_scatter(int64_t M, int64_t K, int64_t N, int V,
                            const int32_t* row_ptr, const int32_t* col_idx, const void* vals,
                            const void* B, void* const* C_dst, int n_dst, int64_t ldc,
                            vs_stream_t stream);

/*
 * vs_sddmm — out = (A * B) sampled at a column-vector mask D [M x N].
 * Problem statement §4.1 P:589-593 (C in CSR, A row-major, B column-major "to replace
 * the transpose"); kernel §6.3-6.4; D a binary mask stored in the
 * column-vector encoding.
 *
 *   row_ptr[W+1], col_idx[nnz_v] : the mask pattern over [M x N], W = ceil(M/V).
 *   A  : fp16 [M x K] row-major.
 *   Bt : fp16 [N x K] row-major (= the paper's column-major B [K x N]).
 *   out_vals : fp16 [nnz_v * V], aligned with col_idx:
 *     out_vals[p*V + r] = fp16_rn( sum_{k<K} A[wV+r][k] * Bt[col_idx[p]][k] ) for
 *     p in window w and wV+r < M; padded rows (wV+r >= M) get +0.0.
 *   The mask only selects positions: no scaling and no multiplication by mask values.
 *   M == 0, N == 0 or nnz_v == 0: no-op.  K == 0: out_vals zero-filled.
 *   Kernels (DESIGN.md 7.3 / 7.8): the 128-row blocks of the mask whose stored density is
 *   above V/32, in problems with K >= 256 (and K % 8 == 0, 16-byte aligned A and Bt), are
 *   computed as dense 128 x 128 tcgen05 tiles and sampled; the other blocks by the
 *   column-vector gather kernel.  The choice depends only on the block's vectors and on K and
 *   N, so it is the same for vs_sddmm_batched and for any 128-row-aligned row-window shard
 *   (same bits).  A window whose col_idx is not strictly ascending inside a dense block is
 *   recomputed by the gather kernel after the dense kernel (any order and duplicates are
 *   supported; each stored vector gets its own output).  The call enqueues two kernels in
 *   stream order (dense tiles, then the gather kernel, which may start early by programmatic
 *   dependent launch when the dense grid is small); the call completes when both have.
 */
vs_status_t vs_sddmm(int64_t M, int64_t N, int64_t K, int V,
                     const int32_t* row_ptr, const int32_t* col_idx,
                     const void* A, const void* Bt, void* out_vals, vs_stream_t stream);

/*
 * vs_softmax_colvec — row softmax over the stored entries of a column-vector CSR matrix
 * (NEXT item of the hot path: sparse attention, Eq. 1 P:1535-1545,
 * A = Softmax((Q K^T o C) / sqrt(k)); the paper's softmax kernel on the column-vector
 * encoding).  For every row i = wV + r < M:
 *   out[p*V + r] = exp(scale*x_p - m) / sum_q exp(scale*x_q - m),  x_p = vals[p*V + r],
 * over the stored vectors p of window w (m = the row's max of scale*x).  Rows >= M (padding
 * of the last window) get +0.  Entries outside the mask take no part (they are -inf in the
 * dense view).  fp16 in/out, fp32 arithmetic.
 *   vals, out : fp16 [nnz_v * V]; out may equal vals (in place).  For V = 4 and 8 both must be
 *               2V-byte aligned (VS_ERROR_MISALIGNED otherwise).
 *   M == 0 or nnz_v == 0: no-op.
 */
vs_status_t vs_softmax_colvec(int64_t M, int V, const int32_t* row_ptr, const void* vals,
                              void* out, float scale, vs_stream_t stream);

/*
 * Batched entry points: many independent problems per call (SURVEY §8(f) rank 3 — the
 * DLMC-sized problems of the paper's benchmarks, are launch-latency bound on
 * B200 one at a time).
 *
 *   problems : HOST array of `count` descriptors, read during the call only.  Each entry has
 *              exactly the semantics, preconditions and alignment rules of the single call;
 *              problems may differ in every field and must not write overlapping outputs.
 *   The library groups the problems by kernel configuration and launches one kernel per
 *   group of up to 128 problems (the descriptors travel as a kernel parameter).  Results
 *   are bitwise identical to calling the single entry point once per problem.
 *   Errors: every entry is checked before anything is enqueued; the first invalid entry
 *   makes the call return its status (VS_ERROR_INVALID_VALUE / VS_ERROR_MISALIGNED).
 *   count == 0 is a no-op.  Asynchronous; the encoder batch never returns nnz_v.
 */
typedef struct {
  int64_t M, K, N;
  int32_t V, reserved;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const void* vals;
  const void* B;
  void* C;
} vs_spmm_problem_t;

typedef struct {
  int64_t M, N, K;
  int32_t V, reserved;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const void* A;
  const void* Bt;
  void* out_vals;
} vs_sddmm_problem_t;

typedef struct {
  int64_t M, K;
  int32_t V, reserved;
  const void* dense;
  const uint8_t* mask;
  int32_t* row_ptr;
  int32_t* col_idx; /* NULL: count mode (row_ptr only) */
  void* vals;
} vs_encode_problem_t;

vs_status_t vs_spmm_batched(int64_t count, const vs_spmm_problem_t* problems, vs_stream_t stream);
vs_status_t vs_sddmm_batched(int64_t count, const vs_sddmm_problem_t* problems,
                             vs_stream_t stream);
vs_status_t vs_encode_colvec_batched(int64_t count, const vs_encode_problem_t* problems,
                                     vs_stream_t stream);

typedef struct {
  int64_t M;
  int32_t V;
  float scale;
  const int32_t* row_ptr;
  const void* vals;
  void* out;
} vs_softmax_problem_t;

vs_status_t vs_softmax_colvec_batched(int64_t count, const vs_softmax_problem_t* problems,
                                      vs_stream_t stream);

#ifdef __cplusplus
}
#endif

#endif /* VS_H_ */
