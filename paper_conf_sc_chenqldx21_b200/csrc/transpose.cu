// transpose.cu — column-vector encoding of A^T from the encoding of A (the
// training-side operand: dX = W^T * dY, "Case 1", and the transposed sparse
// operand of the Discussion).
//
// A [M x K] is stored as V x 1 column vectors (windows w of V rows).  A^T [K x M] is encoded
// with the same grain: window kw = rows kw*V .. kw*V+V-1 of A^T (= columns of A), vector
// (kw, m) = A[m][kw*V .. kw*V+V-1], kept iff one of its V fp16 bit patterns is nonzero (the
// encoder's keep rule, R5) -- so the result equals encode(decode(A)^T) bit for bit, whatever
// the pattern.  For the paper's square V x V blocks every block gives exactly V
// vectors of A^T and nothing is padded.
//
// Deterministic, no sort, no atomics on outputs:
//   T1 (one warp per window w of A): for every stored vector p (column k = col_idx[p]),
//      the bit mask of its rows with nonzero bits is OR-ed into P[kw][w] (kw = k / V) with
//      atomicOr -- order-independent.  P is a caller workspace of ceil(K/V) x ceil(M/V)
//      int32, zeroed first.
//   T2 (one warp per kw): exclusive prefix over w of popc(P[kw][w]), packed into P as
//      (prefix << 8) | mask; the column total goes to rowT[kw + 1].
//   T3 (one CTA): rowT = inclusive prefix of the totals (rowT[0] = 0).
//   T4 (one warp per window w, full mode only): vector p, row r with mask bit r set: A^T
//      vector (kw, m = wV + r) sits at rowT[kw] + prefix + popc(mask below r); its column
//      index is m and its element k % V is vals[p*V + r] (elements of absent columns stay
//      at the +0.0 of a memset).
#include <cstdint>

#include "common.cuh"

namespace vs {

constexpr int kTrWarps = 8;
constexpr int kTrScan = 1024;

template <bool HAS_VALS>
__device__ __forceinline__ uint32_t row_bits(const uint16_t* __restrict__ vals, int64_t p, int V,
                                             int64_t row0, int64_t M) {
  uint32_t bits = 0;
  for (int r = 0; r < V; ++r) {
    if (row0 + r >= M) break;
    const bool nz = HAS_VALS ? (ldg16(vals + p * V + r) != 0) : true;
    bits |= (nz ? 1u : 0u) << r;
  }
  return bits;
}

template <bool HAS_VALS>
__global__ void __launch_bounds__(kTrWarps * 32)
    tr_mark_kernel(int64_t M, int V, int64_t W, const int32_t* __restrict__ row_ptr,
                   const int32_t* __restrict__ col_idx, const uint16_t* __restrict__ vals,
                   int32_t* __restrict__ P) {
  const int64_t w = (int64_t)blockIdx.x * kTrWarps + (threadIdx.x >> 5);
  if (w >= W) return;
  const int lane = lane_id();
  const int64_t pb = row_ptr[w], pe = row_ptr[w + 1];
  for (int64_t p = pb + lane; p < pe; p += 32) {
    const int32_t k = ldg32i(col_idx + p);
    const uint32_t bits = row_bits<HAS_VALS>(vals, p, V, w * V, M);
    if (bits) atomicOr(reinterpret_cast<unsigned int*>(P + (int64_t)(k / V) * W + w), bits);
  }
}

// one warp per kw: exclusive prefix of popc over the W entries of P[kw][*], in place
__global__ void __launch_bounds__(kTrWarps * 32)
    tr_colscan_kernel(int64_t KT, int64_t W, int32_t* __restrict__ P, int32_t* __restrict__ rowT) {
  const int64_t kw = (int64_t)blockIdx.x * kTrWarps + (threadIdx.x >> 5);
  if (kw >= KT) return;
  const int lane = lane_id();
  int32_t* row = P + kw * W;
  int32_t carry = 0;
  for (int64_t base = 0; base < W; base += 32) {
    const int64_t w = base + lane;
    const int32_t m = w < W ? row[w] : 0;
    const int32_t c = __popc(m & 0xFF);
    int32_t incl = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t x = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += x;
    }
    if (w < W) row[w] = ((carry + incl - c) << 8) | (m & 0xFF);
    carry += __shfl_sync(0xffffffffu, incl, 31);
  }
  if (lane == 0) rowT[kw + 1] = carry;
}

// one CTA: rowT[1..n] holds counts -> inclusive prefix in place, rowT[0] = 0
__global__ void __launch_bounds__(kTrScan) tr_scan_kernel(int32_t* __restrict__ rowT, int64_t n) {
  __shared__ int32_t warp_tot[kTrScan / 32];
  __shared__ int32_t carry_sh;
  const int lane = lane_id(), wid = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    carry_sh = 0;
    rowT[0] = 0;
  }
  __syncthreads();
  for (int64_t base = 0; base < n; base += kTrScan) {
    const int64_t i = base + threadIdx.x;
    const int32_t v = i < n ? rowT[i + 1] : 0;
    int32_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t x = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += x;
    }
    if (lane == 31) warp_tot[wid] = incl;
    __syncthreads();
    if (wid == 0) {
      int32_t t = warp_tot[lane];
      int32_t ti = t;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t x = __shfl_up_sync(0xffffffffu, ti, o);
        if (lane >= o) ti += x;
      }
      warp_tot[lane] = ti - t;  // exclusive prefix of warp totals
    }
    __syncthreads();
    const int32_t carry = carry_sh;
    if (i < n) rowT[i + 1] = carry + warp_tot[wid] + incl;
    __syncthreads();
    if (threadIdx.x == kTrScan - 1) carry_sh = carry + warp_tot[wid] + incl;
    __syncthreads();
  }
}

template <bool HAS_VALS>
__global__ void __launch_bounds__(kTrWarps * 32)
    tr_place_kernel(int64_t M, int V, int64_t W, const int32_t* __restrict__ row_ptr,
                    const int32_t* __restrict__ col_idx, const uint16_t* __restrict__ vals,
                    const int32_t* __restrict__ P, const int32_t* __restrict__ rowT,
                    int32_t* __restrict__ colT, uint16_t* __restrict__ valsT) {
  const int64_t w = (int64_t)blockIdx.x * kTrWarps + (threadIdx.x >> 5);
  if (w >= W) return;
  const int lane = lane_id();
  const int64_t pb = row_ptr[w], pe = row_ptr[w + 1];
  for (int64_t p = pb + lane; p < pe; p += 32) {
    const int32_t k = ldg32i(col_idx + p);
    const int64_t kw = k / V;
    const int32_t e = P[kw * W + w];
    const uint32_t mask = (uint32_t)e & 0xFF;
    const int64_t base = (int64_t)rowT[kw] + (e >> 8);
    const uint32_t bits = row_bits<HAS_VALS>(vals, p, V, w * V, M);
    for (int r = 0; r < V; ++r) {
      if (!((bits >> r) & 1u)) continue;
      const int64_t pos = base + __popc(mask & ((1u << r) - 1u));
      colT[pos] = (int32_t)(w * V + r);  // the same value from every vector of the group
      if (HAS_VALS && valsT != nullptr) valsT[pos * V + (k - kw * V)] = ldg16(vals + p * V + r);
    }
  }
}

// values refresh of an existing transposed pattern: like tr_place_kernel, but the rows
// placed are those present in the packed mask of P (the pattern of the previous full call)
__global__ void __launch_bounds__(kTrWarps * 32)
    tr_place_values_kernel(int64_t M, int V, int64_t W, const int32_t* __restrict__ row_ptr,
                           const int32_t* __restrict__ col_idx, const uint16_t* __restrict__ vals,
                           const int32_t* __restrict__ P, const int32_t* __restrict__ rowT,
                           uint16_t* __restrict__ valsT) {
  const int64_t w = (int64_t)blockIdx.x * kTrWarps + (threadIdx.x >> 5);
  if (w >= W) return;
  const int lane = lane_id();
  const int64_t pb = row_ptr[w], pe = row_ptr[w + 1];
  for (int64_t p = pb + lane; p < pe; p += 32) {
    const int32_t k = ldg32i(col_idx + p);
    const int64_t kw = k / V;
    const int32_t e = P[kw * W + w];
    const uint32_t mask = (uint32_t)e & 0xFF;
    const int64_t base = (int64_t)rowT[kw] + (e >> 8);
    for (int r = 0; r < V; ++r) {
      if (!((mask >> r) & 1u)) continue;
      const int64_t pos = base + __popc(mask & ((1u << r) - 1u));
      valsT[pos * V + (k - kw * V)] = ldg16(vals + p * V + r);
    }
  }
}

// zero valsT[0 .. rowT[KT] * V) (the size is only known on the device)
__global__ void tr_zero_kernel(const int32_t* __restrict__ rowT, int64_t KT, int V,
                               uint16_t* __restrict__ valsT) {
  const int64_t n = (int64_t)rowT[KT] * V;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    valsT[i] = 0;
}

// values refresh: the pattern (rowT, colT) and the packed prefixes in P come from a previous
// full call with the same workspace; only valsT is rewritten from the new vals
cudaError_t launch_transpose_values(int64_t M, int64_t K, int V, const int32_t* row_ptr,
                                    const int32_t* col_idx, const void* vals, const int32_t* rowT,
                                    void* valsT, const void* workspace, int num_sms, cudaStream_t s) {
  const int64_t W = ceil_div64(M, V), KT = ceil_div64(K, V);
  if (W == 0 || KT == 0) return cudaSuccess;
  tr_zero_kernel<<<num_sms * 4, 256, 0, s>>>(rowT, KT, V, static_cast<uint16_t*>(valsT));
  // pattern bits from the stored vectors (HAS_VALS = false): every stored row < M is placed
  tr_place_values_kernel<<<(unsigned)ceil_div64(W, kTrWarps), kTrWarps * 32, 0, s>>>(
      M, V, W, row_ptr, col_idx, static_cast<const uint16_t*>(vals),
      static_cast<const int32_t*>(workspace), rowT, static_cast<uint16_t*>(valsT));
  return cudaGetLastError();
}

int64_t transpose_workspace_bytes(int64_t M, int64_t K, int V) {
  return 4 * ceil_div64(K, V) * ceil_div64(M, V);
}

// count mode: colT == nullptr (rowT only)
cudaError_t launch_transpose(int64_t M, int64_t K, int V, const int32_t* row_ptr,
                             const int32_t* col_idx, const void* vals, int32_t* rowT, int32_t* colT,
                             void* valsT, void* workspace, int num_sms, cudaStream_t s) {
  const int64_t W = ceil_div64(M, V), KT = ceil_div64(K, V);
  int32_t* P = static_cast<int32_t*>(workspace);
  const uint16_t* v16 = static_cast<const uint16_t*>(vals);
  cudaError_t e = cudaMemsetAsync(rowT, 0, (size_t)(KT + 1) * 4, s);
  if (e != cudaSuccess || KT == 0) return e;
  if (W > 0) {
    if ((e = cudaMemsetAsync(P, 0, (size_t)(KT * W) * 4, s)) != cudaSuccess) return e;
    const unsigned gw = (unsigned)ceil_div64(W, kTrWarps);
    if (vals) tr_mark_kernel<true><<<gw, kTrWarps * 32, 0, s>>>(M, V, W, row_ptr, col_idx, v16, P);
    else tr_mark_kernel<false><<<gw, kTrWarps * 32, 0, s>>>(M, V, W, row_ptr, col_idx, v16, P);
    tr_colscan_kernel<<<(unsigned)ceil_div64(KT, kTrWarps), kTrWarps * 32, 0, s>>>(KT, W, P, rowT);
  }
  tr_scan_kernel<<<1, kTrScan, 0, s>>>(rowT, KT);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  if (colT == nullptr || W == 0) return cudaSuccess;
  if (valsT != nullptr)
    tr_zero_kernel<<<num_sms * 4, 256, 0, s>>>(rowT, KT, V, static_cast<uint16_t*>(valsT));
  const unsigned gw = (unsigned)ceil_div64(W, kTrWarps);
  if (vals)
    tr_place_kernel<true><<<gw, kTrWarps * 32, 0, s>>>(M, V, W, row_ptr, col_idx, v16, P, rowT, colT,
                                                       static_cast<uint16_t*>(valsT));
  else
    tr_place_kernel<false><<<gw, kTrWarps * 32, 0, s>>>(M, V, W, row_ptr, col_idx, v16, P, rowT, colT,
                                                        nullptr);
  return cudaGetLastError();
}

}  // namespace vs
