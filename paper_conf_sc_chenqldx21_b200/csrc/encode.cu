// encode.cu — dense fp16 matrix / uint8 mask -> column-vector CSR (§4.2, Fig. 8).
//
// Two kernels (+ one memset node), both with one CTA per row window and one warp per
// 256-column chunk (up to 8 warps); each lane tests 8 consecutive columns with one 16-byte
// load per row of the window.  Keep bit = any nonzero fp16 bit pattern (or mask byte) over
// the window's V rows.
//   1. encode_count_scan : counts the window's kept vectors into row_ptr[w+1]; the LAST CTA
//      to finish (a ticket taken with one atomic on row_ptr[0], preset to -1) turns the counts
//      into the inclusive prefix in place and sets row_ptr[0] = 0.  No CTA ever waits for
//      another, so any grid size and any concurrent work on the device are safe.
//   2. encode_compact    : re-reads the window (L2-resident), block-scans the lanes' keep
//      counts and writes col_idx and the V values of each kept vector (transposed from the V
//      row loads into vector-major order) starting at row_ptr[w].
// Columns are visited in ascending order, so col_idx ascends inside each window (Fig. 8).
#include "common.cuh"

namespace vs {

constexpr int kEncMaxThreads = 256;              // threads per CTA (one CTA per window)
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

// ------------------------------------------------------------------------ kernels

// Inclusive scan of a[0..n) in place by one CTA (all threads call it).
__device__ void block_scan_inplace(int32_t* a, int64_t n, int32_t* s_warp, int32_t* s_carry) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, nw = blockDim.x >> 5;
  if (tid == 0) *s_carry = 0;
  __syncthreads();
  constexpr int PER = 4;
  for (int64_t base = 0; base < n; base += (int64_t)blockDim.x * PER) {
    int32_t v[PER];
    int32_t local = 0;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      const int64_t idx = base + (int64_t)tid * PER + j;
      v[j] = idx < n ? __ldcg(a + idx) : 0;
      local += v[j];
    }
    int32_t incl = local;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    if (lane == 31) s_warp[wid] = incl;
    __syncthreads();
    int32_t before = *s_carry, total = 0;
    for (int i = 0; i < nw; ++i) {
      before += (i < wid) ? s_warp[i] : 0;
      total += s_warp[i];
    }
    int32_t run = before + incl - local;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      const int64_t idx = base + (int64_t)tid * PER + j;
      run += v[j];
      if (idx < n) a[idx] = run;
    }
    __syncthreads();
    if (tid == 0) *s_carry += total;
    __syncthreads();
  }
}

template <int V, bool VEC, bool HAS_MASK>
__global__ void __launch_bounds__(kEncMaxThreads)
    encode_count_scan_kernel(int64_t M, int64_t K, int64_t W, const uint16_t* __restrict__ dense,
                             const uint8_t* __restrict__ mask, int32_t* __restrict__ row_ptr) {
  __shared__ int32_t s_warp[kEncMaxThreads / 32];
  __shared__ int32_t s_carry;
  __shared__ int s_last;
  const int lane = lane_id(), wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int64_t w = blockIdx.x;
  uint16_t h[V][8];
  uint32_t count = 0;
  for (int64_t c0 = (int64_t)wid * kColsPerStep; c0 < K; c0 += (int64_t)nw * kColsPerStep) {
    const int64_t c = c0 + lane * kColsPerLane;
    count += __popc(window_keep8<V, VEC, HAS_MASK, false>(dense, mask, M, K, w, c, h));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) count += __shfl_xor_sync(0xffffffffu, count, o);
  if (lane == 0) s_warp[wid] = (int32_t)count;
  __syncthreads();
  if (threadIdx.x == 0) {
    int32_t tot = 0;
    for (int i = 0; i < nw; ++i) tot += s_warp[i];
    row_ptr[w + 1] = tot;
    __threadfence();  // publish the count before taking the ticket
    const int ticket = atomicAdd(row_ptr, 1);  // row_ptr[0] was preset to -1
    s_last = (ticket == (int)(W - 2));
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();  // all counts are visible to the last CTA
  block_scan_inplace(row_ptr + 1, W, s_warp, &s_carry);
  if (threadIdx.x == 0) row_ptr[0] = 0;
}

// Writes col_idx and (optionally) vals of window w from row_ptr[w] on.  Per round, warp i
// takes chunk (round * nwarps + i); a block-wide exclusive scan of the warps' keep counts
// gives each warp its slot range, so col_idx stays ascending.
template <int V, bool VEC, bool HAS_MASK, bool WRITE_VALS, bool VEC_VALS>
__global__ void __launch_bounds__(kEncMaxThreads)
    encode_compact_kernel(int64_t M, int64_t K, const uint16_t* __restrict__ dense,
                          const uint8_t* __restrict__ mask, const int32_t* __restrict__ row_ptr,
                          int32_t* __restrict__ col_idx, uint16_t* __restrict__ vals) {
  __shared__ uint32_t warp_cnt[kEncMaxThreads / 32];
  const int lane = lane_id(), wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int64_t w = blockIdx.x;
  int64_t base = row_ptr[w];
  uint16_t h[V][8];
  for (int64_t r0 = 0; r0 < K; r0 += (int64_t)nw * kColsPerStep) {
    const int64_t c = r0 + (int64_t)wid * kColsPerStep + lane * kColsPerLane;
    const uint32_t keep = window_keep8<V, VEC, HAS_MASK, WRITE_VALS>(dense, mask, M, K, w, c, h);
    const uint32_t n = __popc(keep);
    uint32_t incl = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    if (lane == 31) warp_cnt[wid] = incl;
    __syncthreads();
    uint32_t before = 0, total = 0;
    for (int i = 0; i < nw; ++i) {
      const uint32_t v = warp_cnt[i];
      before += (i < wid) ? v : 0;
      total += v;
    }
    int64_t slot = base + before + (incl - n);
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
    base += total;
    __syncthreads();  // warp_cnt is rewritten next round
  }
}

// ---------------------------------------------------------------- host-side launchers

template <int V, bool VEC, bool MASKB>
static void launch_v(int64_t M, int64_t K, int64_t W, const uint16_t* dense, const uint8_t* mask,
                     int32_t* row_ptr, int32_t* col_idx, uint16_t* vals, bool vec_vals, dim3 grid,
                     dim3 block, cudaStream_t s) {
  encode_count_scan_kernel<V, VEC, MASKB><<<grid, block, 0, s>>>(M, K, W, dense, mask, row_ptr);
  if (col_idx == nullptr) return;
  if (vals == nullptr)
    encode_compact_kernel<V, VEC, MASKB, false, false><<<grid, block, 0, s>>>(M, K, dense, mask, row_ptr, col_idx, vals);
  else if (vec_vals)
    encode_compact_kernel<V, VEC, MASKB, true, true><<<grid, block, 0, s>>>(M, K, dense, mask, row_ptr, col_idx, vals);
  else
    encode_compact_kernel<V, VEC, MASKB, true, false><<<grid, block, 0, s>>>(M, K, dense, mask, row_ptr, col_idx, vals);
}

template <int V>
static cudaError_t launch_encode_v(int64_t M, int64_t K, const uint16_t* dense, const uint8_t* mask,
                                   int32_t* row_ptr, int32_t* col_idx, uint16_t* vals, bool vec,
                                   bool vec_vals, cudaStream_t s) {
  const int64_t W = ceil_div64(M, V);
  if (W == 0) return cudaSuccess;
  if (W > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
  // one CTA per window, one warp per 256-column chunk (up to 8 warps)
  const int64_t chunks = ceil_div64(K, kColsPerStep);
  const int threads =
      (int)(32 * (chunks < 1 ? 1 : (chunks > kEncMaxThreads / 32 ? kEncMaxThreads / 32 : chunks)));
  dim3 grid((unsigned)W), block(threads);
  // row_ptr[0] = -1: the ticket counter of encode_count_scan (reset to 0 by the last CTA)
  cudaError_t e = cudaMemsetAsync(row_ptr, 0xFF, sizeof(int32_t), s);
  if (e != cudaSuccess) return e;
  const bool has_mask = mask != nullptr;
  if (vec) {
    if (has_mask) launch_v<V, true, true>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
    else launch_v<V, true, false>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
  } else {
    if (has_mask) launch_v<V, false, true>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
    else launch_v<V, false, false>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
  }
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
