// encode.cu — dense fp16 matrix / uint8 mask -> column-vector CSR (§4.2, Fig. 8).
//
// One kernel (encode_fused, below) with one CTA per row window and one warp per 256-column
// chunk (up to 8 warps); each lane tests 8 consecutive columns with one 16-byte load per
// row of the window.  Keep bit = any nonzero fp16 bit pattern (or mask byte) over the
// window's V rows.  Phase 1 counts the window; a decoupled look-back over row_ptr gives the
// window's first slot (row_ptr becomes the CSR row pointer in place); phase 2 writes col_idx
// and the V values of each kept vector (transposed from the V row loads into vector-major
// order).
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

// ---------------------------------------------------------------- single-pass encoder
//
// encode_fused: one kernel per call.  CTA w counts its window (phase 1), publishes the count,
// obtains the exclusive prefix of all earlier windows by a decoupled look-back over
// row_ptr itself, publishes its inclusive prefix, then (phase 2) writes col_idx / vals.
// row_ptr[w+1] doubles as the look-back status of window w (it is preset to -1 by one
// memset node):  -1 = nothing yet,  <= -2 = aggregate (count = -s-2) only,  >= 0 = inclusive
// prefix (final value).  CTAs are dispatched in blockIdx order, so a CTA only waits on CTAs
// that are already resident or finished.

// The status word is the only data exchanged between CTAs, so relaxed gpu-scope accesses
// suffice (no other memory is published through it); relaxed loads are not serialised the
// way acquire loads are, so a thread's look-back loads are all in flight at once.
__device__ __forceinline__ void st_status(int32_t* p, int32_t v) {
  asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int32_t ld_status(const int32_t* p) {
  int32_t v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Exclusive prefix of windows [0, w), computed by the whole CTA (all threads call it; all
// get the result).  One round reads the statuses of the kLookback nearest predecessors at
// once (all CTAs of a small problem run concurrently, so the nearest prefix is usually the
// sentinel P(0) before window 0 and one round suffices); the nearest published prefix ends
// the walk, aggregates before it are summed.
constexpr int kLookback = 1024;

__device__ __forceinline__ int64_t lookback(const int32_t* row_ptr, int64_t w, int32_t* s_min,
                                            int64_t* s_sum) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, nw = blockDim.x >> 5;
  const int per = kLookback / blockDim.x;  // statuses per thread per round (<= 32)
  int64_t excl = 0;
  int64_t j = w - 1;  // nearest window not yet accounted for (its status is row_ptr[j + 1])
  while (true) {
    int32_t st[32];
    int my_first = 0x7fffffff;  // smallest offset o (= j - idx) holding a prefix
    // issue all loads, then re-poll only the statuses not yet published
    bool pending = false;
#pragma unroll
    for (int q = 0; q < 32; ++q) {
      if (q >= per) break;
      const int64_t idx = j - (tid * per + q);
      // idx == -1: the P(0) sentinel; idx < -1: beyond it, never summed
      st[q] = idx >= 0 ? ld_status(row_ptr + idx + 1) : 0;
    }
#pragma unroll
    for (int q = 0; q < 32; ++q) pending |= (q < per) && st[q] == -1;
    while (pending) {
      pending = false;
#pragma unroll
      for (int q = 0; q < 32; ++q) {
        if (q >= per) break;
        if (st[q] == -1) st[q] = ld_status(row_ptr + (j - (tid * per + q)) + 1);
      }
#pragma unroll
      for (int q = 0; q < 32; ++q) pending |= (q < per) && st[q] == -1;
    }
#pragma unroll
    for (int q = 0; q < 32; ++q) {
      if (q >= per) break;
      const int o = tid * per + q;
      if (st[q] >= 0 && o < my_first) my_first = o;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) my_first = min(my_first, __shfl_xor_sync(0xffffffffu, my_first, o));
    if (lane == 0) s_min[wid] = my_first;
    __syncthreads();
    int first = 0x7fffffff;
    for (int i = 0; i < nw; ++i) first = min(first, s_min[i]);
    int64_t part = 0;
#pragma unroll
    for (int q = 0; q < 32; ++q) {
      if (q >= per) break;
      const int o = tid * per + q;
      const int32_t v = st[q];
      if (o < first) part += (int64_t)(-v - 2);  // aggregate (only -x-2 values precede first)
      else if (o == first) part += (int64_t)v;    // the nearest inclusive prefix
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
    if (lane == 0) s_sum[wid] = part;
    __syncthreads();
    for (int i = 0; i < nw; ++i) excl += s_sum[i];
    __syncthreads();  // s_min / s_sum reused next round
    if (first != 0x7fffffff) return excl;
    j -= kLookback;
  }
}

template <int V, bool VEC, bool HAS_MASK, bool WRITE_IDX, bool WRITE_VALS, bool VEC_VALS>
__global__ void __launch_bounds__(kEncMaxThreads)
    encode_fused_kernel(int64_t M, int64_t K, const uint16_t* __restrict__ dense,
                        const uint8_t* __restrict__ mask, int32_t* __restrict__ row_ptr,
                        int32_t* __restrict__ col_idx, uint16_t* __restrict__ vals) {
  __shared__ uint32_t warp_cnt[kEncMaxThreads / 32];
  __shared__ int32_t s_min[kEncMaxThreads / 32];
  __shared__ int64_t s_sum[kEncMaxThreads / 32];
  const int lane = lane_id(), wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int64_t w = blockIdx.x;
  uint16_t h[V][8];

  // phase 1: count the window's kept vectors
  uint32_t count = 0;
  for (int64_t c0 = (int64_t)wid * kColsPerStep; c0 < K; c0 += (int64_t)nw * kColsPerStep) {
    const int64_t c = c0 + lane * kColsPerLane;
    count += __popc(window_keep8<V, VEC, HAS_MASK, false>(dense, mask, M, K, w, c, h));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) count += __shfl_xor_sync(0xffffffffu, count, o);
  if (lane == 0) warp_cnt[wid] = count;
  __syncthreads();
  uint32_t tot = 0;
  for (int i = 0; i < nw; ++i) tot += warp_cnt[i];
  int64_t base;
  if (w == 0) {
    if (threadIdx.x == 0) {
      st_status(row_ptr + 1, (int32_t)tot);
      row_ptr[0] = 0;
    }
    base = 0;
  } else {
    if (threadIdx.x == 0) st_status(row_ptr + w + 1, -(int32_t)tot - 2);  // aggregate
    base = lookback(row_ptr, w, s_min, s_sum);
    if (threadIdx.x == 0) st_status(row_ptr + w + 1, (int32_t)(base + tot));  // inclusive prefix
  }
  if (!WRITE_IDX) return;

  // phase 2: write col_idx / vals (re-reads the window, now L1/L2 resident)
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
    __syncthreads();  // previous round's readers of warp_cnt are done
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
  }
}

// ---------------------------------------------------------------- host-side launchers

template <int V, bool VEC, bool MASKB>
static void launch_fused(int64_t M, int64_t K, int64_t W, const uint16_t* dense, const uint8_t* mask,
                         int32_t* row_ptr, int32_t* col_idx, uint16_t* vals, bool vec_vals,
                         dim3 grid, dim3 block, cudaStream_t s) {
  if (col_idx == nullptr)
    encode_fused_kernel<V, VEC, MASKB, false, false, false><<<grid, block, 0, s>>>(
        M, K, dense, mask, row_ptr, col_idx, vals);
  else if (vals == nullptr)
    encode_fused_kernel<V, VEC, MASKB, true, false, false><<<grid, block, 0, s>>>(
        M, K, dense, mask, row_ptr, col_idx, vals);
  else if (vec_vals)
    encode_fused_kernel<V, VEC, MASKB, true, true, true><<<grid, block, 0, s>>>(
        M, K, dense, mask, row_ptr, col_idx, vals);
  else
    encode_fused_kernel<V, VEC, MASKB, true, true, false><<<grid, block, 0, s>>>(
        M, K, dense, mask, row_ptr, col_idx, vals);
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
  // look-back status: row_ptr[1..W] = -1 ("nothing published yet")
  cudaError_t e = cudaMemsetAsync(row_ptr + 1, 0xFF, (size_t)W * sizeof(int32_t), s);
  if (e != cudaSuccess) return e;
  const bool has_mask = mask != nullptr;
  if (vec) {
    if (has_mask) launch_fused<V, true, true>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
    else launch_fused<V, true, false>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
  } else {
    if (has_mask) launch_fused<V, false, true>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
    else launch_fused<V, false, false>(M, K, W, dense, mask, row_ptr, col_idx, vals, vec_vals, grid, block, s);
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
