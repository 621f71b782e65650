// vs_api.cu — the C ABI of include/vs.h: argument checks, dispatch, launch status.
// No exception crosses this boundary; every entry point returns a vs_status_t.
#include <mutex>
#include <vector>

#include "../../include/vs.h"
#include "common.cuh"

namespace vs {
cudaError_t launch_encode(int64_t M, int64_t K, int V, const void* dense, const uint8_t* mask,
                          int32_t* row_ptr, int32_t* col_idx, void* vals, cudaStream_t s);
cudaError_t launch_spmm(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                        const int32_t* col_idx, const void* vals, const void* B, void* C,
                        int num_sms, cudaStream_t s);
cudaError_t launch_spmm_scatter(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                                const int32_t* col_idx, const void* vals, const void* B,
                                void* const* C_dst, int n_dst, int64_t ldc, int num_sms, cudaStream_t s);
cudaError_t launch_sddmm(int64_t M, int64_t N, int64_t K, int V, const int32_t* row_ptr,
                         const int32_t* col_idx, const void* A, const void* Bt, void* out,
                         int num_sms, cudaStream_t s);
cudaError_t launch_spmm_batched(int64_t count, const int64_t* M, const int64_t* K, const int64_t* N,
                                const int* V, const int32_t* const* row_ptr,
                                const int32_t* const* col_idx, const void* const* vals,
                                const void* const* B, void* const* C, int num_sms, cudaStream_t s);
cudaError_t launch_sddmm_batched(int64_t count, const int64_t* M, const int64_t* N, const int64_t* K,
                                 const int* V, const int32_t* const* row_ptr,
                                 const int32_t* const* col_idx, const void* const* A,
                                 const void* const* Bt, void* const* out, int num_sms,
                                 cudaStream_t s);
cudaError_t launch_encode_batched(int64_t count, const int64_t* M, const int64_t* K, const int* V,
                                  const void* const* dense, const uint8_t* const* mask,
                                  int32_t* const* row_ptr, int32_t* const* col_idx,
                                  void* const* vals, int num_sms, cudaStream_t s);
cudaError_t launch_softmax(int64_t M, int V, const int32_t* row_ptr, const void* vals, void* out,
                           float scale, cudaStream_t s);
cudaError_t launch_softmax_batched(int64_t count, const int64_t* M, const int* V,
                                   const int32_t* const* row_ptr, const void* const* vals,
                                   void* const* out, const float* scale, cudaStream_t s);
int64_t transpose_workspace_bytes(int64_t M, int64_t K, int V);
cudaError_t launch_transpose(int64_t M, int64_t K, int V, const int32_t* row_ptr,
                             const int32_t* col_idx, const void* vals, int32_t* rowT, int32_t* colT,
                             void* valsT, void* workspace, int num_sms, cudaStream_t s);
cudaError_t launch_transpose_values(int64_t M, int64_t K, int V, const int32_t* row_ptr,
                                    const int32_t* col_idx, const void* vals, const int32_t* rowT,
                                    void* valsT, const void* workspace, int num_sms, cudaStream_t s);
}  // namespace vs

namespace {

constexpr int kMaxDevices = 64;
struct DevInfo {
  int ok;  // 1 = sm_100, 0 = other
  int num_sms;
};
DevInfo g_dev[kMaxDevices];
std::once_flag g_dev_once[kMaxDevices];

// Device attributes of the current device, queried once per device.
bool device_info(DevInfo* out) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return false;
  std::call_once(g_dev_once[dev], [dev] {
    int major = 0, minor = 0, sms = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    g_dev[dev].ok = (major == 10 && minor == 0) ? 1 : 0;
    g_dev[dev].num_sms = sms > 0 ? sms : 148;
  });
  *out = g_dev[dev];
  return true;
}

bool valid_v(int V) { return V == 1 || V == 2 || V == 4 || V == 8; }
bool al(const void* p, uintptr_t a) { return (reinterpret_cast<uintptr_t>(p) & (a - 1)) == 0; }

vs_status_t from_cuda(cudaError_t e) { return e == cudaSuccess ? VS_SUCCESS : VS_ERROR_CUDA; }

vs_status_t check_device(DevInfo* info) {
  if (!device_info(info)) return VS_ERROR_CUDA;
  return info->ok ? VS_SUCCESS : VS_ERROR_NOT_SUPPORTED;
}

// Host-side argument checks shared by the single and batched entry points.
vs_status_t check_encode(int64_t M, int64_t K, int V, const void* dense, const uint8_t* mask,
                         int32_t* row_ptr, int32_t* col_idx, void* vals) {
  if (!valid_v(V) || M < 0 || K < 0) return VS_ERROR_INVALID_VALUE;
  // dense / mask may be NULL only for an empty matrix (M * K == 0)
  if (M * K > 0 && dense == nullptr && mask == nullptr) return VS_ERROR_INVALID_VALUE;
  if (row_ptr == nullptr) return VS_ERROR_INVALID_VALUE;
  if (M * K > 0 && vals != nullptr && dense == nullptr) return VS_ERROR_INVALID_VALUE;
  if (!al(row_ptr, 4) || (col_idx && !al(col_idx, 4))) return VS_ERROR_MISALIGNED;
  if ((dense && !al(dense, 2)) || (vals && !al(vals, 2))) return VS_ERROR_MISALIGNED;
  // row_ptr / nnz_v are int32: refuse matrices whose vector count could reach 2^31
  if (M > 0 && (M + V - 1) / V * K >= (int64_t(1) << 31)) return VS_ERROR_NOT_SUPPORTED;
  return VS_SUCCESS;
}

vs_status_t check_spmm(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                       const int32_t* col_idx, const void* vals, const void* B, const void* C) {
  if (!valid_v(V) || M < 0 || K < 0 || N < 0) return VS_ERROR_INVALID_VALUE;
  if (M == 0 || N == 0) return VS_SUCCESS;
  // col_idx / vals / B may be NULL only when they are never read (nnz_v == 0 or K == 0)
  if (row_ptr == nullptr || C == nullptr) return VS_ERROR_INVALID_VALUE;
  if (!al(row_ptr, 4) || (col_idx && !al(col_idx, 4))) return VS_ERROR_MISALIGNED;
  if ((vals && !al(vals, 2)) || (B && !al(B, 2)) || !al(C, 2)) return VS_ERROR_MISALIGNED;
  return VS_SUCCESS;
}

vs_status_t check_sddmm(int64_t M, int64_t N, int64_t K, int V, const int32_t* row_ptr,
                        const int32_t* col_idx, const void* A, const void* Bt, const void* out) {
  if (!valid_v(V) || M < 0 || K < 0 || N < 0) return VS_ERROR_INVALID_VALUE;
  if (M == 0 || N == 0) return VS_SUCCESS;
  // col_idx / A / Bt / out_vals may be NULL only when never touched (nnz_v == 0)
  if (row_ptr == nullptr) return VS_ERROR_INVALID_VALUE;
  if (!al(row_ptr, 4) || (col_idx && !al(col_idx, 4))) return VS_ERROR_MISALIGNED;
  if ((A && !al(A, 2)) || (Bt && !al(Bt, 2)) || (out && !al(out, 2))) return VS_ERROR_MISALIGNED;
  return VS_SUCCESS;
}

vs_status_t check_softmax(int64_t M, int V, const int32_t* row_ptr, const void* vals,
                          const void* out) {
  if (!valid_v(V) || M < 0) return VS_ERROR_INVALID_VALUE;
  if (M == 0) return VS_SUCCESS;
  // vals / out may be NULL only when never touched (nnz_v == 0)
  if (row_ptr == nullptr) return VS_ERROR_INVALID_VALUE;
  if (!al(row_ptr, 4)) return VS_ERROR_MISALIGNED;
  const uintptr_t need = V >= 4 ? 2 * V : 2;
  if ((vals && !al(vals, need)) || (out && !al(out, need))) return VS_ERROR_MISALIGNED;
  return VS_SUCCESS;
}

}  // namespace

extern "C" {

const char* vs_status_string(vs_status_t s) {
  switch (s) {
    case VS_SUCCESS: return "VS_SUCCESS";
    case VS_ERROR_INVALID_VALUE: return "VS_ERROR_INVALID_VALUE";
    case VS_ERROR_NOT_SUPPORTED: return "VS_ERROR_NOT_SUPPORTED";
    case VS_ERROR_CUDA: return "VS_ERROR_CUDA";
    case VS_ERROR_MISALIGNED: return "VS_ERROR_MISALIGNED";
  }
  return "VS_ERROR_UNKNOWN";
}

int vs_version(void) { return 100; /* 0.1.0 */ }

vs_status_t vs_encode_colvec(int64_t M, int64_t K, int V, const void* dense, const uint8_t* mask,
                             int32_t* row_ptr, int32_t* col_idx, void* vals,
                             int64_t* nnz_vec_host, vs_stream_t stream) {
  vs_status_t st0 = check_encode(M, K, V, dense, mask, row_ptr, col_idx, vals);
  if (st0 != VS_SUCCESS) return st0;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const int64_t W = vs::ceil_div64(M, V);
  if (W == 0) {
    // row_ptr = [0]
    if (cudaMemsetAsync(row_ptr, 0, sizeof(int32_t), s) != cudaSuccess) return VS_ERROR_CUDA;
  } else {
    cudaError_t e = vs::launch_encode(M, K, V, dense, mask, row_ptr, col_idx, vals, s);
    if (e != cudaSuccess) return VS_ERROR_CUDA;
  }
  if (nnz_vec_host != nullptr) {
    int32_t nnz = 0;
    if (cudaMemcpyAsync(&nnz, row_ptr + W, sizeof(int32_t), cudaMemcpyDeviceToHost, s) !=
        cudaSuccess)
      return VS_ERROR_CUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess) return VS_ERROR_CUDA;
    *nnz_vec_host = nnz;
  }
  return VS_SUCCESS;
}

vs_status_t vs_spmm(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                    const int32_t* col_idx, const void* vals, const void* B, void* C,
                    vs_stream_t stream) {
  vs_status_t st0 = check_spmm(M, K, N, V, row_ptr, col_idx, vals, B, C);
  if (st0 != VS_SUCCESS || M == 0 || N == 0) return st0;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  if (K == 0) return from_cuda(cudaMemsetAsync(C, 0, (size_t)(M * N) * 2, s));
  return from_cuda(vs::launch_spmm(M, K, N, V, row_ptr, col_idx, vals, B, C, info.num_sms, s));
}

vs_status_t vs_spmm_scatter(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                            const int32_t* col_idx, const void* vals, const void* B,
                            void* const* C_dst, int n_dst, int64_t ldc, vs_stream_t stream) {
  if (C_dst == nullptr || n_dst < 1 || n_dst > VS_SPMM_SCATTER_MAX || ldc < N)
    return VS_ERROR_INVALID_VALUE;
  for (int d = 0; d < n_dst; ++d) {
    // each destination is checked like vs_spmm's C
    const vs_status_t st = check_spmm(M, K, N, V, row_ptr, col_idx, vals, B, C_dst[d]);
    if (st != VS_SUCCESS) return st;
  }
  if (M == 0 || N == 0) return VS_SUCCESS;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  if (K == 0) {  // zero fill of the N columns of every destination
    for (int d = 0; d < n_dst; ++d)
      if (cudaMemset2DAsync(C_dst[d], (size_t)ldc * 2, 0, (size_t)N * 2, (size_t)M, s) != cudaSuccess)
        return VS_ERROR_CUDA;
    return VS_SUCCESS;
  }
  return from_cuda(vs::launch_spmm_scatter(M, K, N, V, row_ptr, col_idx, vals, B, C_dst, n_dst, ldc,
                                           info.num_sms, s));
}

vs_status_t vs_sddmm(int64_t M, int64_t N, int64_t K, int V, const int32_t* row_ptr,
                     const int32_t* col_idx, const void* A, const void* Bt, void* out_vals,
                     vs_stream_t stream) {
  vs_status_t st0 = check_sddmm(M, N, K, V, row_ptr, col_idx, A, Bt, out_vals);
  if (st0 != VS_SUCCESS || M == 0 || N == 0) return st0;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  return from_cuda(vs::launch_sddmm(M, N, K, V, row_ptr, col_idx, A, Bt, out_vals, info.num_sms, s));
}

int64_t vs_transpose_colvec_workspace(int64_t M, int64_t K, int V) {
  if (!valid_v(V) || M < 0 || K < 0) return 0;
  return vs::transpose_workspace_bytes(M, K, V);
}

vs_status_t vs_transpose_colvec(int64_t M, int64_t K, int V, const int32_t* row_ptr,
                                const int32_t* col_idx, const void* vals, int32_t* rowT_ptr,
                                int32_t* colT_idx, void* valsT, void* workspace,
                                int64_t* nnzT_host, vs_stream_t stream) {
  if (!valid_v(V) || M < 0 || K < 0 || rowT_ptr == nullptr) return VS_ERROR_INVALID_VALUE;
  if (valsT != nullptr && (vals == nullptr || colT_idx == nullptr)) return VS_ERROR_INVALID_VALUE;
  const int64_t W = (M + V - 1) / V;
  if (W > 0 && K > 0 && (row_ptr == nullptr || workspace == nullptr)) return VS_ERROR_INVALID_VALUE;
  if (M >= (int64_t(1) << 23)) return VS_ERROR_NOT_SUPPORTED;  // packed 23-bit prefixes
  if (!al(rowT_ptr, 4) || (row_ptr && !al(row_ptr, 4)) || (col_idx && !al(col_idx, 4)) ||
      (colT_idx && !al(colT_idx, 4)) || (workspace && !al(workspace, 4)))
    return VS_ERROR_MISALIGNED;
  if ((vals && !al(vals, 2)) || (valsT && !al(valsT, 2))) return VS_ERROR_MISALIGNED;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  st = from_cuda(vs::launch_transpose(M, K, V, row_ptr, col_idx, vals, rowT_ptr, colT_idx, valsT,
                                      workspace, info.num_sms, s));
  if (st != VS_SUCCESS || nnzT_host == nullptr) return st;
  int32_t n = 0;
  const int64_t KT = (K + V - 1) / V;
  if (cudaMemcpyAsync(&n, rowT_ptr + KT, 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return VS_ERROR_CUDA;
  *nnzT_host = n;
  return VS_SUCCESS;
}

vs_status_t vs_transpose_colvec_values(int64_t M, int64_t K, int V, const int32_t* row_ptr,
                                       const int32_t* col_idx, const void* vals,
                                       const int32_t* rowT_ptr, void* valsT, const void* workspace,
                                       vs_stream_t stream) {
  if (!valid_v(V) || M < 0 || K < 0 || rowT_ptr == nullptr) return VS_ERROR_INVALID_VALUE;
  if (M == 0 || K == 0) return VS_SUCCESS;
  if (row_ptr == nullptr || workspace == nullptr || vals == nullptr || valsT == nullptr)
    return VS_ERROR_INVALID_VALUE;
  if (M >= (int64_t(1) << 23)) return VS_ERROR_NOT_SUPPORTED;
  if (!al(rowT_ptr, 4) || !al(row_ptr, 4) || (col_idx && !al(col_idx, 4)) || !al(workspace, 4) ||
      !al(vals, 2) || !al(valsT, 2))
    return VS_ERROR_MISALIGNED;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  return from_cuda(vs::launch_transpose_values(M, K, V, row_ptr, col_idx, vals, rowT_ptr, valsT,
                                               workspace, info.num_sms,
                                               reinterpret_cast<cudaStream_t>(stream)));
}

vs_status_t vs_softmax_colvec(int64_t M, int V, const int32_t* row_ptr, const void* vals,
                              void* out, float scale, vs_stream_t stream) {
  vs_status_t st0 = check_softmax(M, V, row_ptr, vals, out);
  if (st0 != VS_SUCCESS || M == 0) return st0;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  return from_cuda(vs::launch_softmax(M, V, row_ptr, vals, out, scale,
                                      reinterpret_cast<cudaStream_t>(stream)));
}

vs_status_t vs_softmax_colvec_batched(int64_t count, const vs_softmax_problem_t* problems,
                                      vs_stream_t stream) {
  if (count < 0 || (count > 0 && problems == nullptr)) return VS_ERROR_INVALID_VALUE;
  for (int64_t i = 0; i < count; ++i) {
    const vs_softmax_problem_t& p = problems[i];
    const vs_status_t st = check_softmax(p.M, p.V, p.row_ptr, p.vals, p.out);
    if (st != VS_SUCCESS) return st;
  }
  if (count == 0) return VS_SUCCESS;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  std::vector<int64_t> M;
  std::vector<int> V;
  std::vector<const int32_t*> rp;
  std::vector<const void*> va;
  std::vector<void*> out;
  std::vector<float> sc;
  for (int64_t i = 0; i < count; ++i) {
    const vs_softmax_problem_t& p = problems[i];
    if (p.M == 0) continue;
    M.push_back(p.M); V.push_back(p.V); rp.push_back(p.row_ptr); va.push_back(p.vals);
    out.push_back(p.out); sc.push_back(p.scale);
  }
  if (M.empty()) return VS_SUCCESS;
  return from_cuda(vs::launch_softmax_batched((int64_t)M.size(), M.data(), V.data(), rp.data(),
                                              va.data(), out.data(), sc.data(),
                                              reinterpret_cast<cudaStream_t>(stream)));
}

vs_status_t vs_spmm_batched(int64_t count, const vs_spmm_problem_t* problems, vs_stream_t stream) {
  if (count < 0 || (count > 0 && problems == nullptr)) return VS_ERROR_INVALID_VALUE;
  for (int64_t i = 0; i < count; ++i) {
    const vs_spmm_problem_t& p = problems[i];
    const vs_status_t st = check_spmm(p.M, p.K, p.N, p.V, p.row_ptr, p.col_idx, p.vals, p.B, p.C);
    if (st != VS_SUCCESS) return st;
  }
  if (count == 0) return VS_SUCCESS;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  std::vector<int64_t> M, K, N;
  std::vector<int> V;
  std::vector<const int32_t*> rp, ci;
  std::vector<const void*> va, B;
  std::vector<void*> C;
  for (int64_t i = 0; i < count; ++i) {
    const vs_spmm_problem_t& p = problems[i];
    if (p.M == 0 || p.N == 0) continue;
    if (p.K == 0) {
      if (cudaMemsetAsync(p.C, 0, (size_t)(p.M * p.N) * 2, s) != cudaSuccess) return VS_ERROR_CUDA;
      continue;
    }
    M.push_back(p.M); K.push_back(p.K); N.push_back(p.N); V.push_back(p.V);
    rp.push_back(p.row_ptr); ci.push_back(p.col_idx); va.push_back(p.vals); B.push_back(p.B);
    C.push_back(p.C);
  }
  if (M.empty()) return VS_SUCCESS;
  return from_cuda(vs::launch_spmm_batched((int64_t)M.size(), M.data(), K.data(), N.data(), V.data(),
                                           rp.data(), ci.data(), va.data(), B.data(), C.data(),
                                           info.num_sms, s));
}

vs_status_t vs_sddmm_batched(int64_t count, const vs_sddmm_problem_t* problems,
                             vs_stream_t stream) {
  if (count < 0 || (count > 0 && problems == nullptr)) return VS_ERROR_INVALID_VALUE;
  for (int64_t i = 0; i < count; ++i) {
    const vs_sddmm_problem_t& p = problems[i];
    const vs_status_t st = check_sddmm(p.M, p.N, p.K, p.V, p.row_ptr, p.col_idx, p.A, p.Bt, p.out_vals);
    if (st != VS_SUCCESS) return st;
  }
  if (count == 0) return VS_SUCCESS;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  std::vector<int64_t> M, N, K;
  std::vector<int> V;
  std::vector<const int32_t*> rp, ci;
  std::vector<const void*> A, Bt;
  std::vector<void*> out;
  for (int64_t i = 0; i < count; ++i) {
    const vs_sddmm_problem_t& p = problems[i];
    if (p.M == 0 || p.N == 0) continue;
    M.push_back(p.M); N.push_back(p.N); K.push_back(p.K); V.push_back(p.V); rp.push_back(p.row_ptr);
    ci.push_back(p.col_idx); A.push_back(p.A); Bt.push_back(p.Bt); out.push_back(p.out_vals);
  }
  if (M.empty()) return VS_SUCCESS;
  return from_cuda(vs::launch_sddmm_batched((int64_t)M.size(), M.data(), N.data(), K.data(), V.data(), rp.data(),
                                            ci.data(), A.data(), Bt.data(), out.data(),
                                            info.num_sms, s));
}

vs_status_t vs_encode_colvec_batched(int64_t count, const vs_encode_problem_t* problems,
                                     vs_stream_t stream) {
  if (count < 0 || (count > 0 && problems == nullptr)) return VS_ERROR_INVALID_VALUE;
  for (int64_t i = 0; i < count; ++i) {
    const vs_encode_problem_t& p = problems[i];
    const vs_status_t st = check_encode(p.M, p.K, p.V, p.dense, p.mask, p.row_ptr, p.col_idx, p.vals);
    if (st != VS_SUCCESS) return st;
  }
  if (count == 0) return VS_SUCCESS;
  DevInfo info;
  vs_status_t st = check_device(&info);
  if (st != VS_SUCCESS) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  std::vector<int64_t> M, K;
  std::vector<int> V;
  std::vector<const void*> dense;
  std::vector<const uint8_t*> mask;
  std::vector<int32_t*> rp, ci;
  std::vector<void*> vals;
  for (int64_t i = 0; i < count; ++i) {
    const vs_encode_problem_t& p = problems[i];
    if (p.M == 0) {  // W == 0: row_ptr = [0]
      if (cudaMemsetAsync(p.row_ptr, 0, sizeof(int32_t), s) != cudaSuccess) return VS_ERROR_CUDA;
      continue;
    }
    M.push_back(p.M); K.push_back(p.K); V.push_back(p.V); dense.push_back(p.dense);
    mask.push_back(p.mask); rp.push_back(p.row_ptr); ci.push_back(p.col_idx); vals.push_back(p.vals);
  }
  if (M.empty()) return VS_SUCCESS;
  return from_cuda(vs::launch_encode_batched((int64_t)M.size(), M.data(), K.data(), V.data(),
                                             dense.data(), mask.data(), rp.data(), ci.data(),
                                             vals.data(), info.num_sms, s));
}

}  // extern "C"
