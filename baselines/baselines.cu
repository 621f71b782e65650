// baselines.cu — same-box comparison points for bench.py (NOT part of the product path):
//   cublasHgemm (fp16 compute, the paper's "cuBLASHgemm"),
//   cublasGemmEx (fp16 I/O, fp32 compute),
//   cusparseSpMM on Blocked-ELL (the paper's TCU baseline, built as in
//   §7.1.1) and on V-expanded scalar CSR,
//   cusparseSDDMM on V-expanded scalar CSR.
// Plans hold descriptors + workspace so that a timed run is exactly one library call.
#include <cublas_v2.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <cusparse.h>
#include <stdint.h>

#include <cstdlib>

namespace {
struct Handles {
  cublasHandle_t blas = nullptr;
  cusparseHandle_t sp = nullptr;
};

enum Kind { SPMM = 0, SDDMM = 1 };

struct Plan {
  Handles* h;
  int kind;
  cusparseSpMatDescr_t sp = nullptr;
  cusparseDnMatDescr_t d1 = nullptr, d2 = nullptr;
  void* buf = nullptr;
  float alpha = 1.f, beta = 0.f;
  cusparseSpMMAlg_t spmm_alg;
  cudaStream_t stream;
};
}  // namespace

extern "C" {

void* bl_create() {
  Handles* h = new Handles();
  if (cublasCreate(&h->blas) != CUBLAS_STATUS_SUCCESS) { delete h; return nullptr; }
  if (cusparseCreate(&h->sp) != CUSPARSE_STATUS_SUCCESS) { cublasDestroy(h->blas); delete h; return nullptr; }
  return h;
}

void bl_destroy(void* p) {
  Handles* h = static_cast<Handles*>(p);
  if (!h) return;
  cublasDestroy(h->blas);
  cusparseDestroy(h->sp);
  delete h;
}

// Row-major C[M x N] = A[M x K] * B[K x N] as column-major C^T = B^T A^T.
int bl_hgemm(void* p, int64_t M, int64_t N, int64_t K, const void* A, const void* B, void* C,
             void* stream) {
  Handles* h = static_cast<Handles*>(p);
  cublasSetStream(h->blas, (cudaStream_t)stream);
  __half one = __float2half(1.f), zero = __float2half(0.f);
  return (int)cublasHgemm(h->blas, CUBLAS_OP_N, CUBLAS_OP_N, (int)N, (int)M, (int)K, &one,
                          (const __half*)B, (int)N, (const __half*)A, (int)K, &zero, (__half*)C,
                          (int)N);
}

int bl_gemmex(void* p, int64_t M, int64_t N, int64_t K, const void* A, const void* B, void* C,
              void* stream) {
  Handles* h = static_cast<Handles*>(p);
  cublasSetStream(h->blas, (cudaStream_t)stream);
  float one = 1.f, zero = 0.f;
  return (int)cublasGemmEx(h->blas, CUBLAS_OP_N, CUBLAS_OP_N, (int)N, (int)M, (int)K, &one, B,
                           CUDA_R_16F, (int)N, A, CUDA_R_16F, (int)K, &zero, C, CUDA_R_16F,
                           (int)N, CUBLAS_COMPUTE_32F, CUBLAS_GEMM_DEFAULT);
}

static int finish_spmm_plan(Plan* pl, int* status) {
  size_t sz = 0;
  cusparseStatus_t st = cusparseSpMM_bufferSize(pl->h->sp, CUSPARSE_OPERATION_NON_TRANSPOSE,
                                                CUSPARSE_OPERATION_NON_TRANSPOSE, &pl->alpha, pl->sp,
                                                pl->d1, &pl->beta, pl->d2, CUDA_R_32F, pl->spmm_alg, &sz);
  if (st != CUSPARSE_STATUS_SUCCESS) { *status = (int)st; return 0; }
  if (sz && cudaMalloc(&pl->buf, sz) != cudaSuccess) { *status = -1; return 0; }
  st = cusparseSpMM_preprocess(pl->h->sp, CUSPARSE_OPERATION_NON_TRANSPOSE,
                               CUSPARSE_OPERATION_NON_TRANSPOSE, &pl->alpha, pl->sp, pl->d1,
                               &pl->beta, pl->d2, CUDA_R_32F, pl->spmm_alg, pl->buf);
  if (st != CUSPARSE_STATUS_SUCCESS) { *status = (int)st; return 0; }
  *status = 0;
  return 1;
}

void bl_plan_free(void* p) {
  Plan* pl = static_cast<Plan*>(p);
  if (!pl) return;
  if (pl->sp) cusparseDestroySpMat(pl->sp);
  if (pl->d1) cusparseDestroyDnMat(pl->d1);
  if (pl->d2) cusparseDestroyDnMat(pl->d2);
  if (pl->buf) cudaFree(pl->buf);
  delete pl;
}

// Scalar CSR (fp16 values) SpMM: C[M x N] = A * B, B and C row-major fp16.
void* bl_spmm_csr_plan(void* h, int64_t M, int64_t K, int64_t N, int64_t nnz, void* row_ptr,
                       void* col_idx, void* vals, void* B, void* C, void* stream, int* status) {
  Plan* pl = new Plan();
  pl->h = static_cast<Handles*>(h);
  pl->kind = SPMM;
  pl->stream = (cudaStream_t)stream;
  pl->spmm_alg = CUSPARSE_SPMM_CSR_ALG2;
  cusparseSetStream(pl->h->sp, pl->stream);
  cusparseStatus_t st = cusparseCreateCsr(&pl->sp, M, K, nnz, row_ptr, col_idx, vals, CUSPARSE_INDEX_32I,
                                          CUSPARSE_INDEX_32I, CUSPARSE_INDEX_BASE_ZERO, CUDA_R_16F);
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseCreateDnMat(&pl->d1, K, N, N, B, CUDA_R_16F, CUSPARSE_ORDER_ROW);
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseCreateDnMat(&pl->d2, M, N, N, C, CUDA_R_16F, CUSPARSE_ORDER_ROW);
  if (st != CUSPARSE_STATUS_SUCCESS) { *status = (int)st; bl_plan_free(pl); return nullptr; }
  if (!finish_spmm_plan(pl, status)) { bl_plan_free(pl); return nullptr; }
  return pl;
}

// Blocked-ELL SpMM: ell_cols = blocks per block-row * block size, col_ind [M/bs x ell_cols/bs].
void* bl_spmm_bell_plan(void* h, int64_t M, int64_t K, int64_t N, int64_t block, int64_t ell_cols,
                        void* ell_col_ind, void* ell_vals, void* B, void* C, void* stream,
                        int* status) {
  Plan* pl = new Plan();
  pl->h = static_cast<Handles*>(h);
  pl->kind = SPMM;
  pl->stream = (cudaStream_t)stream;
  pl->spmm_alg = CUSPARSE_SPMM_BLOCKED_ELL_ALG1;
  cusparseSetStream(pl->h->sp, pl->stream);
  cusparseStatus_t st = cusparseCreateBlockedEll(&pl->sp, M, K, block, ell_cols, ell_col_ind, ell_vals,
                                                 CUSPARSE_INDEX_32I, CUSPARSE_INDEX_BASE_ZERO, CUDA_R_16F);
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseCreateDnMat(&pl->d1, K, N, N, B, CUDA_R_16F, CUSPARSE_ORDER_ROW);
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseCreateDnMat(&pl->d2, M, N, N, C, CUDA_R_16F, CUSPARSE_ORDER_ROW);
  if (st != CUSPARSE_STATUS_SUCCESS) { *status = (int)st; bl_plan_free(pl); return nullptr; }
  if (!finish_spmm_plan(pl, status)) { bl_plan_free(pl); return nullptr; }
  return pl;
}

// SDDMM on scalar CSR: out(CSR vals) = (A[M x K] * B[K x N]) o pattern; A, B row-major.
// value_type: 0 = fp16 values, 1 = fp32 values (A, B, out all of that type).
void* bl_sddmm_csr_plan(void* h, int64_t M, int64_t N, int64_t K, int64_t nnz, void* row_ptr,
                        void* col_idx, void* out_vals, void* A, void* B, int value_type,
                        void* stream, int* status) {
  Plan* pl = new Plan();
  pl->h = static_cast<Handles*>(h);
  pl->kind = SDDMM;
  pl->stream = (cudaStream_t)stream;
  cudaDataType dt = value_type == 0 ? CUDA_R_16F : CUDA_R_32F;
  cusparseSetStream(pl->h->sp, pl->stream);
  cusparseStatus_t st = cusparseCreateCsr(&pl->sp, M, N, nnz, row_ptr, col_idx, out_vals,
                                          CUSPARSE_INDEX_32I, CUSPARSE_INDEX_32I,
                                          CUSPARSE_INDEX_BASE_ZERO, dt);
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseCreateDnMat(&pl->d1, M, K, K, A, dt, CUSPARSE_ORDER_ROW);
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseCreateDnMat(&pl->d2, K, N, N, B, dt, CUSPARSE_ORDER_ROW);
  size_t sz = 0;
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseSDDMM_bufferSize(pl->h->sp, CUSPARSE_OPERATION_NON_TRANSPOSE,
                                  CUSPARSE_OPERATION_NON_TRANSPOSE, &pl->alpha, pl->d1, pl->d2,
                                  &pl->beta, pl->sp, CUDA_R_32F, CUSPARSE_SDDMM_ALG_DEFAULT, &sz);
  if (st == CUSPARSE_STATUS_SUCCESS && sz && cudaMalloc(&pl->buf, sz) != cudaSuccess) {
    *status = -1; bl_plan_free(pl); return nullptr;
  }
  if (st == CUSPARSE_STATUS_SUCCESS)
    st = cusparseSDDMM_preprocess(pl->h->sp, CUSPARSE_OPERATION_NON_TRANSPOSE,
                                  CUSPARSE_OPERATION_NON_TRANSPOSE, &pl->alpha, pl->d1, pl->d2,
                                  &pl->beta, pl->sp, CUDA_R_32F, CUSPARSE_SDDMM_ALG_DEFAULT, pl->buf);
  if (st != CUSPARSE_STATUS_SUCCESS) { *status = (int)st; bl_plan_free(pl); return nullptr; }
  *status = 0;
  return pl;
}

int bl_plan_run(void* p) {
  Plan* pl = static_cast<Plan*>(p);
  cusparseSetStream(pl->h->sp, pl->stream);
  if (pl->kind == SPMM)
    return (int)cusparseSpMM(pl->h->sp, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE,
                             &pl->alpha, pl->sp, pl->d1, &pl->beta, pl->d2, CUDA_R_32F, pl->spmm_alg,
                             pl->buf);
  return (int)cusparseSDDMM(pl->h->sp, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE,
                            &pl->alpha, pl->d1, pl->d2, &pl->beta, pl->sp, CUDA_R_32F,
                            CUSPARSE_SDDMM_ALG_DEFAULT, pl->buf);
}

}  // extern "C"
