// softmax.cu — row softmax over a column-vector-sparse matrix (the
// sparse attention of Eq. 1: A = Softmax((Q K^T o C) / sqrt(k)); the paper's
// "custom softmax kernel that works on column vector sparse encoding").
//
//   out[p*V + r] = exp(s*x_p - m) / sum_q exp(s*x_q - m),  x_p = vals[p*V + r],
// over the stored vectors p of window w, for every row i = wV + r < M (m = max_p s*x_p);
// rows >= M (padding of the last window) get 0.  fp16 in/out, fp32 arithmetic.  A -inf score
// contributes exp(-inf) = 0; a row whose stored scores are all -inf outputs 0 (DESIGN R23).
//
// One warp per window; lane l owns vectors rb + l, rb + l + 32, ...  Pass 1 keeps an online
// (max, sum) per row in each lane (sum rescaled when the max grows) and combines the lanes
// with shuffles; pass 2 re-reads the window (L1-resident) and writes the normalised values.
// out may alias vals (every element is read before it is written by the same lane).
#include <algorithm>
#include <utility>
#include <vector>

#include "common.cuh"

namespace vs {

constexpr int kSoftmaxWarps = 4;

template <int V>
__device__ __forceinline__ void load_vec(const uint16_t* __restrict__ vals, int64_t p, float (&x)[V]) {
  const uint16_t* src = vals + p * V;
  if constexpr (V == 8) {
    const uint4 u = *reinterpret_cast<const uint4*>(src);
    const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const __half2 h = *reinterpret_cast<const __half2*>(&w[q]);
      x[2 * q] = __low2float(h);
      x[2 * q + 1] = __high2float(h);
    }
  } else if constexpr (V == 4) {
    const uint2 u = *reinterpret_cast<const uint2*>(src);
    const uint32_t w[2] = {u.x, u.y};
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const __half2 h = *reinterpret_cast<const __half2*>(&w[q]);
      x[2 * q] = __low2float(h);
      x[2 * q + 1] = __high2float(h);
    }
  } else {
#pragma unroll
    for (int r = 0; r < V; ++r) x[r] = __half2float(*reinterpret_cast<const __half*>(src + r));
  }
}

template <int V>
__device__ __forceinline__ void store_vec(uint16_t* __restrict__ out, int64_t p, const float (&y)[V]) {
  uint16_t* dst = out + p * V;
  if constexpr (V == 8) {
    stg128(dst, make_uint4(f2_to_h2(y[0], y[1]), f2_to_h2(y[2], y[3]), f2_to_h2(y[4], y[5]),
                           f2_to_h2(y[6], y[7])));
  } else if constexpr (V == 4) {
    *reinterpret_cast<uint2*>(dst) = make_uint2(f2_to_h2(y[0], y[1]), f2_to_h2(y[2], y[3]));
  } else {
#pragma unroll
    for (int r = 0; r < V; ++r) dst[r] = f_to_h(y[r]);
  }
}

// VEC_IO: vals / out aligned to 2V bytes (vector loads for V = 4, 8).
template <int V>
__device__ __forceinline__ void softmax_window(int64_t M, int64_t w, const int32_t* __restrict__ row_ptr,
                                               const uint16_t* vals, uint16_t* out, float scale) {
  const int lane = lane_id();
  const int64_t rb = row_ptr[w], re = row_ptr[w + 1];
  // scale * log2(e): exp(s*x - m) = exp2(s*log2e*x - m')
  const float sl = scale * 1.4426950408889634f;
  float m[V], sum[V];
#pragma unroll
  for (int r = 0; r < V; ++r) {
    m[r] = -INFINITY;
    sum[r] = 0.f;
  }
  for (int64_t p = rb + lane; p < re; p += 32) {
    float x[V];
    load_vec<V>(vals, p, x);
#pragma unroll
    for (int r = 0; r < V; ++r) {
      const float y = x[r] * sl;
      const float nm = fmaxf(m[r], y);
      // a -inf score (masked out by the caller) adds nothing; while the row has seen only
      // -inf, m stays -inf and sum 0 (no inf - inf)
      if (nm == -INFINITY) continue;
      sum[r] = sum[r] * exp2f(m[r] - nm) + exp2f(y - nm);
      m[r] = nm;
    }
  }
  // combine the lanes' (max, sum) pairs
#pragma unroll
  for (int r = 0; r < V; ++r) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const float om = __shfl_xor_sync(0xffffffffu, m[r], o);
      const float os = __shfl_xor_sync(0xffffffffu, sum[r], o);
      const float nm = fmaxf(m[r], om);
      const float a = (m[r] == -INFINITY) ? 0.f : sum[r] * exp2f(m[r] - nm);
      const float b = (om == -INFINITY) ? 0.f : os * exp2f(om - nm);
      m[r] = nm;
      sum[r] = a + b;
    }
  }
  float inv[V];
#pragma unroll
  for (int r = 0; r < V; ++r) inv[r] = (w * V + r < M && sum[r] > 0.f) ? 1.f / sum[r] : 0.f;
  for (int64_t p = rb + lane; p < re; p += 32) {
    float x[V];
    load_vec<V>(vals, p, x);
    float y[V];
#pragma unroll
    for (int r = 0; r < V; ++r) y[r] = inv[r] == 0.f ? 0.f : exp2f(x[r] * sl - m[r]) * inv[r];
    store_vec<V>(out, p, y);
  }
}

template <int V>
__global__ void __launch_bounds__(kSoftmaxWarps * 32)
    softmax_kernel(int64_t M, int64_t W, const int32_t* __restrict__ row_ptr,
                   const uint16_t* vals, uint16_t* out, float scale) {
  const int64_t w = (int64_t)blockIdx.x * kSoftmaxWarps + (threadIdx.x >> 5);
  if (w < W) softmax_window<V>(M, w, row_ptr, vals, out, scale);
}

struct SoftmaxDesc {
  int64_t M, W;
  const int32_t* row_ptr;
  const uint16_t* vals;
  uint16_t* out;
  float scale;
};
constexpr int kSoftmaxMaxBatch = 128;
struct SoftmaxBatch {
  int count;
  int64_t first_block[kSoftmaxMaxBatch + 1];
  SoftmaxDesc d[kSoftmaxMaxBatch];
};

template <int V>
__global__ void __launch_bounds__(kSoftmaxWarps * 32) softmax_batched_kernel(const __grid_constant__ SoftmaxBatch b) {
  const int p = first_problem(b.first_block, b.count, (int64_t)blockIdx.x);
  const SoftmaxDesc& d = b.d[p];
  const int64_t w = (blockIdx.x - b.first_block[p]) * kSoftmaxWarps + (threadIdx.x >> 5);
  if (w < d.W) softmax_window<V>(d.M, w, d.row_ptr, d.vals, d.out, d.scale);
}

template <int V>
static void launch_v(int64_t M, int64_t W, const int32_t* row_ptr, const uint16_t* vals,
                     uint16_t* out, float scale, cudaStream_t s) {
  softmax_kernel<V><<<(unsigned)ceil_div64(W, kSoftmaxWarps), kSoftmaxWarps * 32, 0, s>>>(
      M, W, row_ptr, vals, out, scale);
}

// V = 4 / 8 use vector loads: vals and out must be 2V-byte aligned (checked by the caller;
// otherwise the V-scalar path of V = 1 semantics is not available, so the caller rejects).
cudaError_t launch_softmax(int64_t M, int V, const int32_t* row_ptr, const void* vals, void* out,
                           float scale, cudaStream_t s) {
  const int64_t W = ceil_div64(M, V);
  if (W == 0) return cudaSuccess;
  if (ceil_div64(W, kSoftmaxWarps) > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
  const uint16_t* v = static_cast<const uint16_t*>(vals);
  uint16_t* o = static_cast<uint16_t*>(out);
  switch (V) {
    case 1: launch_v<1>(M, W, row_ptr, v, o, scale, s); break;
    case 2: launch_v<2>(M, W, row_ptr, v, o, scale, s); break;
    case 4: launch_v<4>(M, W, row_ptr, v, o, scale, s); break;
    default: launch_v<8>(M, W, row_ptr, v, o, scale, s); break;
  }
  return cudaGetLastError();
}

cudaError_t launch_softmax_batched(int64_t count, const int64_t* M, const int* V,
                                   const int32_t* const* row_ptr, const void* const* vals,
                                   void* const* out, const float* scale, cudaStream_t s) {
  std::vector<std::pair<int, int64_t>> order;
  for (int64_t i = 0; i < count; ++i) order.push_back({V[i], i});
  std::stable_sort(order.begin(), order.end(),
                   [](const auto& a, const auto& b) { return a.first < b.first; });
  SoftmaxBatch batch;
  size_t i = 0;
  while (i < order.size()) {
    const int v = order[i].first;
    batch.count = 0;
    int64_t blocks = 0;
    while (i < order.size() && order[i].first == v && batch.count < kSoftmaxMaxBatch) {
      const int64_t p = order[i].second;
      const int64_t W = ceil_div64(M[p], v);
      const int64_t nb = ceil_div64(W, kSoftmaxWarps);
      if (blocks + nb > 0x7fffffffLL) break;
      batch.d[batch.count] = {M[p], W, row_ptr[p], static_cast<const uint16_t*>(vals[p]),
                              static_cast<uint16_t*>(out[p]), scale[p]};
      batch.first_block[batch.count++] = blocks;
      blocks += nb;
      ++i;
    }
    if (batch.count == 0) return cudaErrorInvalidConfiguration;
    batch.first_block[batch.count] = blocks;
    if (blocks > 0) {
      switch (v) {
        case 1: softmax_batched_kernel<1><<<(unsigned)blocks, kSoftmaxWarps * 32, 0, s>>>(batch); break;
        case 2: softmax_batched_kernel<2><<<(unsigned)blocks, kSoftmaxWarps * 32, 0, s>>>(batch); break;
        case 4: softmax_batched_kernel<4><<<(unsigned)blocks, kSoftmaxWarps * 32, 0, s>>>(batch); break;
        default: softmax_batched_kernel<8><<<(unsigned)blocks, kSoftmaxWarps * 32, 0, s>>>(batch); break;
      }
    }
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace vs
