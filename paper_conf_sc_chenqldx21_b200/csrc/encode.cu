// encode.cu — dense fp16 matrix / uint8 mask -> column-vector CSR (§4.2, Fig. 8).
//
// Three stream-ordered kernels:
//   1. encode_count   : one warp per row window; each lane tests 8 consecutive columns per
//                       step (one 16-byte load per row of the window), keep bit = any nonzero
//                       fp16 bit pattern (or mask byte) over the window's V rows; the warp's
//                       popcount total goes to row_ptr[w+1].
//   2. scan_inplace   : one CTA turns the per-window counts into the inclusive prefix, so
//                       row_ptr[w] is the first vector of window w (row_ptr[0] = 0).
//   3. encode_compact : one warp per window again; a warp-wide exclusive scan of the lanes'
//                       keep counts gives every kept column its slot; the lane writes col_idx
//                       and the V values of the vector (transposed from the V row loads into
//                       vector-major order).
// Columns are visited in ascending order, so col_idx ascends inside each window (Fig. 8).
#include "common.cuh"

namespace vs {

constexpr int kEncWarps = 4;                     // warps (windows) per CTA
constexpr int kColsPerLane = 8;                  // columns per lane per step
constexpr int kColsPerStep = kColsPerLane * 32;  // 256 columns per warp step

// Loads the 8 columns [c, c+8) of row i as halves; returns them in h[8]; missing -> 0.
template <bool VEC>
__device__ __forceinline__ void load_row8(const uint16_t* __restrict__ dense, int64_t i, int64_t K,
                                          int64_t c, uint16_t (&h)[8]) {
  const uint16_t* row = dense + i * K;
  if (VEC) {
    if (c < K) {  // K % 8 == 0: the 8 columns are all in range
      uint4 v = ldg128_na(row + c);
      uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        h[2 * q] = (uint16_t)(w[q] & 0xFFFF);
        h[2 * q + 1] = (uint16_t)(w[q] >> 16);
      }
    } else {
#pragma unroll
      for (int j = 0; j < 8; ++j) h[j] = 0;
    }
  } else {
#pragma unroll
    for (int j = 0; j < 8; ++j) h[j] = (c + j < K) ? ldg16(row + c + j) : (uint16_t)0;
  }
}

template <bool VEC>
__device__ __forceinline__ uint32_t mask_keep8(const uint8_t* __restrict__ mask, int64_t i, int64_t K,
                                               int64_t c) {
  const uint8_t* row = mask + i * K;
  uint32_t bits = 0;
  if (VEC) {
    if (c < K) {
      uint2 v = *reinterpret_cast<const uint2*>(row + c);
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        bits |= (((v.x >> (8 * j)) & 0xFF) != 0) << j;
        bits |= (((v.y >> (8 * j)) & 0xFF) != 0) << (j + 4);
      }
    }
  } else {
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (c + j < K && row[c + j] != 0) bits |= 1u << j;
  }
  return bits;
}

// keep bits of the 8 columns [c, c+8) of window w (+ the values when WANT_VALS).
template <int V, bool VEC, bool HAS_MASK, bool WANT_VALS>
__device__ __forceinline__ uint32_t window_keep8(const uint16_t* __restrict__ dense,
                                                 const uint8_t* __restrict__ mask, int64_t M,
                                                 int64_t K, int64_t w, int64_t c,
                                                 uint16_t (&h)[V][8]) {
  uint32_t keep = 0;
#pragma unroll
  for (int r = 0; r < V; ++r) {
    int64_t i = w * V + r;
    bool in = i < M;
    if (HAS_MASK) {
      if (in) keep |= mask_keep8<VEC>(mask, i, K, c);
    }
    if (WANT_VALS || !HAS_MASK) {
      if (in) {
        load_row8<VEC>(dense, i, K, c, h[r]);
      } else {
#pragma unroll
        for (int j = 0; j < 8; ++j) h[r][j] = 0;
      }
      if (!HAS_MASK) {
#pragma unroll
        for (int j = 0; j < 8; ++j) keep |= (h[r][j] != 0) << j;
      }
    }
  }
  return keep;
}

template <int V, bool VEC, bool HAS_MASK>
__global__ void __launch_bounds__(kEncWarps * 32)
    encode_count_kernel(int64_t M, int64_t K, int64_t W, const uint16_t* __restrict__ dense,
                        const uint8_t* __restrict__ mask, int32_t* __restrict__ row_ptr) {
  const int lane = lane_id();
  const int64_t w = (int64_t)blockIdx.x * kEncWarps + (threadIdx.x >> 5);
  if (w >= W) return;
  uint32_t count = 0;
  uint16_t h[V][8];
  for (int64_t c0 = 0; c0 < K; c0 += kColsPerStep) {
    int64_t c = c0 + lane * kColsPerLane;
    uint32_t keep = window_keep8<V, VEC, HAS_MASK, false>(dense, mask, M, K, w, c, h);
    count += __popc(keep);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) count += __shfl_xor_sync(0xffffffffu, count, o);
  if (lane == 0) row_ptr[w + 1] = (int32_t)count;
  if (w == 0 && lane == 0) row_ptr[0] = 0;
}

// In-place inclusive scan of row_ptr[1..W] (per-window counts) by one CTA of 1024 threads.
constexpr int kScanThreads = 1024;
constexpr int kScanPerThread = 4;
__global__ void __launch_bounds__(kScanThreads) scan_inplace_kernel(int32_t* __restrict__ row_ptr,
                                                                    int64_t W) {
  __shared__ int32_t warp_sums[32];
  __shared__ int32_t carry_s;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  if (tid == 0) carry_s = 0;
  __syncthreads();
  int32_t* a = row_ptr + 1;
  for (int64_t base = 0; base < W; base += (int64_t)kScanThreads * kScanPerThread) {
    int32_t v[kScanPerThread];
    int32_t local = 0;
#pragma unroll
    for (int j = 0; j < kScanPerThread; ++j) {
      int64_t idx = base + (int64_t)tid * kScanPerThread + j;
      v[j] = idx < W ? a[idx] : 0;
      local += v[j];
    }
    int32_t incl = local;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    if (lane == 31) warp_sums[wid] = incl;
    __syncthreads();
    if (wid == 0) {
      int32_t s = warp_sums[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int32_t t = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += t;
      }
      warp_sums[lane] = s;  // inclusive over warps
    }
    __syncthreads();
    int32_t carry = carry_s;
    int32_t run = carry + (wid > 0 ? warp_sums[wid - 1] : 0) + incl - local;
#pragma unroll
    for (int j = 0; j < kScanPerThread; ++j) {
      int64_t idx = base + (int64_t)tid * kScanPerThread + j;
      run += v[j];
      if (idx < W) a[idx] = run;
    }
    __syncthreads();
    if (tid == 0) carry_s = carry + warp_sums[31];
    __syncthreads();
  }
  if (tid == 0) row_ptr[0] = 0;
}

// Writes col_idx and (optionally) vals of window w; needs the scanned row_ptr.
template <int V, bool VEC, bool HAS_MASK, bool WRITE_VALS, bool VEC_VALS>
__global__ void __launch_bounds__(kEncWarps * 32)
    encode_compact_kernel(int64_t M, int64_t K, int64_t W, const uint16_t* __restrict__ dense,
                          const uint8_t* __restrict__ mask, const int32_t* __restrict__ row_ptr,
                          int32_t* __restrict__ col_idx, uint16_t* __restrict__ vals) {
  const int lane = lane_id();
  const int64_t w = (int64_t)blockIdx.x * kEncWarps + (threadIdx.x >> 5);
  if (w >= W) return;
  int64_t base = row_ptr[w];
  uint16_t h[V][8];
  for (int64_t c0 = 0; c0 < K; c0 += kColsPerStep) {
    int64_t c = c0 + lane * kColsPerLane;
    uint32_t keep = window_keep8<V, VEC, HAS_MASK, WRITE_VALS>(dense, mask, M, K, w, c, h);
    uint32_t n = __popc(keep);
    uint32_t incl = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    int64_t slot = base + (incl - n);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      if (keep & (1u << j)) {
        col_idx[slot] = (int32_t)(c + j);
        if (WRITE_VALS) {
          uint16_t* dst = vals + slot * V;
          if constexpr (VEC_VALS && V == 8) {
            stg128(dst, make_uint4(pack_h2(h[0][j], h[1][j]), pack_h2(h[2][j], h[3][j]),
                                   pack_h2(h[4][j], h[5][j]), pack_h2(h[6][j], h[7][j])));
          } else if constexpr (VEC_VALS && V == 4) {
            *reinterpret_cast<uint2*>(dst) =
                make_uint2(pack_h2(h[0][j], h[1][j]), pack_h2(h[2][j], h[3][j]));
          } else if constexpr (VEC_VALS && V == 2) {
            *reinterpret_cast<uint32_t*>(dst) = pack_h2(h[0][j], h[1][j]);
          } else {
#pragma unroll
            for (int r = 0; r < V; ++r) dst[r] = h[r][j];
          }
        }
        ++slot;
      }
    }
    base += __shfl_sync(0xffffffffu, incl, 31);
  }
}

// ---------------------------------------------------------------- host-side launchers

template <int V>
static cudaError_t launch_encode_v(int64_t M, int64_t K, const uint16_t* dense, const uint8_t* mask,
                                   int32_t* row_ptr, int32_t* col_idx, uint16_t* vals, bool vec,
                                   bool vec_vals, cudaStream_t s) {
  const int64_t W = ceil_div64(M, V);
  if (W == 0) return cudaSuccess;
  dim3 grid((unsigned)ceil_div64(W, kEncWarps)), block(kEncWarps * 32);
  const bool has_mask = mask != nullptr;
#define VS_COUNT(VECB, MASKB) \
  encode_count_kernel<V, VECB, MASKB><<<grid, block, 0, s>>>(M, K, W, dense, mask, row_ptr)
  if (vec) {
    if (has_mask) VS_COUNT(true, true); else VS_COUNT(true, false);
  } else {
    if (has_mask) VS_COUNT(false, true); else VS_COUNT(false, false);
  }
#undef VS_COUNT
  scan_inplace_kernel<<<1, kScanThreads, 0, s>>>(row_ptr, W);
  if (col_idx == nullptr) return cudaGetLastError();
  const bool wv = vals != nullptr;
#define VS_COMPACT(VECB, MASKB, WVB, VVB)                                              \
  encode_compact_kernel<V, VECB, MASKB, WVB, VVB><<<grid, block, 0, s>>>(M, K, W, dense, mask, \
                                                                          row_ptr, col_idx, vals)
#define VS_COMPACT2(VECB, MASKB)                                \
  do {                                                          \
    if (!wv) VS_COMPACT(VECB, MASKB, false, false);             \
    else if (vec_vals) VS_COMPACT(VECB, MASKB, true, true);     \
    else VS_COMPACT(VECB, MASKB, true, false);                  \
  } while (0)
  if (vec) {
    if (has_mask) VS_COMPACT2(true, true); else VS_COMPACT2(true, false);
  } else {
    if (has_mask) VS_COMPACT2(false, true); else VS_COMPACT2(false, false);
  }
#undef VS_COMPACT2
#undef VS_COMPACT
  return cudaGetLastError();
}

cudaError_t launch_encode(int64_t M, int64_t K, int V, const void* dense, const uint8_t* mask,
                          int32_t* row_ptr, int32_t* col_idx, void* vals, cudaStream_t s) {
  const uint16_t* d = static_cast<const uint16_t*>(dense);
  // vector path: 16-byte rows (fp16) / 8-byte rows (mask)
  bool vec = (K % 8 == 0);
  if (d && (reinterpret_cast<uintptr_t>(d) & 15)) vec = false;
  if (mask && (reinterpret_cast<uintptr_t>(mask) & 7)) vec = false;
  bool vec_vals = vals && ((reinterpret_cast<uintptr_t>(vals) & (2 * V - 1)) == 0);
  uint16_t* v = static_cast<uint16_t*>(vals);
  switch (V) {
    case 1: return launch_encode_v<1>(M, K, d, mask, row_ptr, col_idx, v, vec, vec_vals, s);
    case 2: return launch_encode_v<2>(M, K, d, mask, row_ptr, col_idx, v, vec, vec_vals, s);
    case 4: return launch_encode_v<4>(M, K, d, mask, row_ptr, col_idx, v, vec, vec_vals, s);
    case 8: return launch_encode_v<8>(M, K, d, mask, row_ptr, col_idx, v, vec, vec_vals, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace vs
