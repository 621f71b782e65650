// encode.cu — dense fp16 matrix / uint8 mask -> column-vector CSR (§4.2, Fig. 8).
//
// Three kernels, count and compact with one warp per row window (4 windows per CTA); each
// lane tests 8 consecutive columns per 256-column step with one 16-byte load per row of the
// window.  Keep bit = any nonzero fp16 bit pattern (or mask byte) over the window's V rows.
//   1. encode_count   : the warp's popcount total goes to row_ptr[w+1].
//   2. encode_scan    : one CTA turns the counts into the inclusive prefix in place and sets
//                       row_ptr[0] = 0.
//   3. encode_compact : re-reads the window (L2-resident), warp-scans the lanes' keep counts,
//      packs each 256-column chunk's kept columns and vectors (transposed from the V row loads
//      into vector-major order) in shared memory and writes them from row_ptr[w]
//      on with coalesced stores (batched DLMC encode 247 -> 213 us against per-lane
//      scattered stores).
// Columns are visited in ascending order, so col_idx ascends inside each window (Fig. 8).
#include <algorithm>
#include <utility>
#include <vector>

#include <cstdlib>

#include "common.cuh"

namespace vs {

constexpr int kEncWarps = 4;                     // windows (warps) per CTA
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

// Phase 1: one warp per window walks the window's 256-column chunks (the next chunk's rows
// are loaded while the current one is counted) and writes the count into row_ptr[w+1].
template <int V, bool VEC, bool HAS_MASK>
__device__ __forceinline__ void count_body(int64_t M, int64_t K, int64_t w,
                                           const uint16_t* __restrict__ dense,
                                           const uint8_t* __restrict__ mask,
                                           int32_t* __restrict__ row_ptr) {
  const int lane = lane_id();
  uint16_t h[V][8];
  uint32_t count = 0;
#pragma unroll 2
  for (int64_t c0 = 0; c0 < K; c0 += kColsPerStep) {
    const int64_t c = c0 + lane * kColsPerLane;
    count += __popc(window_keep8<V, VEC, HAS_MASK, false>(dense, mask, M, K, w, c, h));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) count += __shfl_xor_sync(0xffffffffu, count, o);
  if (lane == 0) row_ptr[w + 1] = (int32_t)count;
}

// Writes col_idx and (optionally) vals of window w from row_ptr[w] on.  One warp per window
// walks its 256-column chunks in order; a warp-wide exclusive scan of the lanes' keep counts
// gives every kept column its slot, so col_idx stays ascending.
template <int V, bool VEC, bool HAS_MASK, bool WRITE_VALS, bool VEC_VALS>
__device__ __forceinline__ void compact_body_direct(int64_t M, int64_t K, int64_t w,
                                             const uint16_t* __restrict__ dense,
                                             const uint8_t* __restrict__ mask,
                                             const int32_t* __restrict__ row_ptr,
                                             int32_t* __restrict__ col_idx,
                                             uint16_t* __restrict__ vals) {
  const int lane = lane_id();
  int64_t base = row_ptr[w];
  uint16_t h[V][8];
#pragma unroll 2
  for (int64_t c0 = 0; c0 < K; c0 += kColsPerStep) {
    const int64_t c = c0 + lane * kColsPerLane;
    const uint32_t keep = window_keep8<V, VEC, HAS_MASK, WRITE_VALS>(dense, mask, M, K, w, c, h);
    const uint32_t n = __popc(keep);
    uint32_t incl = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
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

// Same output as compact_body_direct, but each 256-column chunk's kept columns and vectors
// are first packed in shared memory (per warp) and then written with coalesced stores: lane i
// stores kept entry i, i + 32, ... (contiguous slots) instead of 8 scattered store rounds.
// VS_ENC_STAGED = 0 selects the direct variant.
#ifndef VS_ENC_STAGED
#define VS_ENC_STAGED 1
#endif
// resident CTAs per SM the compact kernels' registers are sized for (tools/tune.py, batched
// DLMC encode: 1 -> 233 us, 6 -> 211 us (80 registers), 8 -> 233 us, 12 -> 321 us: spills)
#ifndef VS_ENC_MINB
#define VS_ENC_MINB 6
#endif
// VS_ENC_PREFETCH: next-chunk row prefetch in the staged compact pass (dense input, V <= 4)
#ifndef VS_ENC_PREFETCH
#define VS_ENC_PREFETCH 1
#endif
// The 8 columns [c, c+8) of row i as one 16-byte word; zeros past M or K (K % 8 == 0).
__device__ __forceinline__ uint4 enc_raw_row(const uint16_t* __restrict__ dense, int64_t i, int64_t M,
                                             int64_t K, int64_t c) {
  return (i < M && c < K) ? ldg128_na(dense + i * K + c) : make_uint4(0, 0, 0, 0);
}
// Halves of the V raw row words into h and the keep bits (any nonzero bit pattern).
template <int V>
__device__ __forceinline__ uint32_t enc_unpack_keep(const uint4 (&raw)[V], uint16_t (&h)[V][8]) {
  uint32_t keep = 0;
#pragma unroll
  for (int r = 0; r < V; ++r) {
    const uint32_t wd[4] = {raw[r].x, raw[r].y, raw[r].z, raw[r].w};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      h[r][2 * q] = (uint16_t)(wd[q] & 0xFFFF);
      h[r][2 * q + 1] = (uint16_t)(wd[q] >> 16);
    }
#pragma unroll
    for (int j = 0; j < 8; ++j) keep |= (uint32_t)(h[r][j] != 0) << j;
  }
  return keep;
}

template <int V, bool VEC, bool HAS_MASK, bool WRITE_VALS, bool VEC_VALS>
__device__ __forceinline__ void compact_body(int64_t M, int64_t K, int64_t w,
                                             const uint16_t* __restrict__ dense,
                                             const uint8_t* __restrict__ mask,
                                             const int32_t* __restrict__ row_ptr,
                                             int32_t* __restrict__ col_idx,
                                             uint16_t* __restrict__ vals, int64_t base_in = -1) {
#if VS_ENC_STAGED
  __shared__ int32_t s_col_all[kEncWarps][kColsPerStep];
  __shared__ __align__(16) uint16_t s_val_all[kEncWarps][WRITE_VALS ? kColsPerStep * V : 8];
  const int wid = threadIdx.x >> 5;
  int32_t* s_col = s_col_all[wid];
  uint16_t* s_val = s_val_all[wid];
  const int lane = lane_id();
  int64_t base = base_in >= 0 ? base_in : row_ptr[w];
  uint16_t h[V][8];
  // Dense 16-byte path, V <= 4: the rows of the next 256-column chunk are loaded before the
  // current chunk is packed and stored (the shared-memory staging and __syncwarp of a chunk
  // otherwise keep the next chunk's loads from issuing early).  Same output.
  constexpr bool PF = VS_ENC_PREFETCH && VEC && !HAS_MASK && V <= 4;
  uint4 nxt[PF ? V : 1];
  if constexpr (PF) {
#pragma unroll
    for (int r = 0; r < V; ++r) nxt[r] = enc_raw_row(dense, w * V + r, M, K, (int64_t)lane * kColsPerLane);
  }
#pragma unroll 2
  for (int64_t c0 = 0; c0 < K; c0 += kColsPerStep) {
    const int64_t c = c0 + lane * kColsPerLane;
    uint32_t keep;
    if constexpr (PF) {
      uint4 cur[V];
#pragma unroll
      for (int r = 0; r < V; ++r) {
        cur[r] = nxt[r];
        nxt[r] = enc_raw_row(dense, w * V + r, M, K, c + kColsPerStep);
      }
      keep = enc_unpack_keep<V>(cur, h);
    } else {
      keep = window_keep8<V, VEC, HAS_MASK, WRITE_VALS>(dense, mask, M, K, w, c, h);
    }
    const uint32_t n = __popc(keep);
    uint32_t incl = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    const int total = (int)__shfl_sync(0xffffffffu, incl, 31);
    int slot = (int)(incl - n);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      if (keep & (1u << j)) {
        s_col[slot] = (int32_t)(c + j);
        if (WRITE_VALS) {
          uint16_t* sv = s_val + slot * V;
          if constexpr (V == 8) {
            *reinterpret_cast<uint4*>(sv) = make_uint4(pack_h2(h[0][j], h[1][j]), pack_h2(h[2][j], h[3][j]),
                                                       pack_h2(h[4][j], h[5][j]), pack_h2(h[6][j], h[7][j]));
          } else if constexpr (V == 4) {
            *reinterpret_cast<uint2*>(sv) = make_uint2(pack_h2(h[0][j], h[1][j]), pack_h2(h[2][j], h[3][j]));
          } else if constexpr (V == 2) {
            *reinterpret_cast<uint32_t*>(sv) = pack_h2(h[0][j], h[1][j]);
          } else {
            sv[0] = h[0][j];
          }
        }
        ++slot;
      }
    }
    __syncwarp();
    for (int i = lane; i < total; i += 32) {
      col_idx[base + i] = s_col[i];
      if (WRITE_VALS) {
        uint16_t* dst = vals + (base + i) * V;
        const uint16_t* sv = s_val + i * V;
        if constexpr (VEC_VALS && V == 8) {
          stg128(dst, *reinterpret_cast<const uint4*>(sv));
        } else if constexpr (VEC_VALS && V == 4) {
          *reinterpret_cast<uint2*>(dst) = *reinterpret_cast<const uint2*>(sv);
        } else if constexpr (VEC_VALS && V == 2) {
          *reinterpret_cast<uint32_t*>(dst) = *reinterpret_cast<const uint32_t*>(sv);
        } else {
#pragma unroll
          for (int r = 0; r < V; ++r) dst[r] = sv[r];
        }
      }
    }
    __syncwarp();
    base += total;
  }
#else
  (void)base_in;
  compact_body_direct<V, VEC, HAS_MASK, WRITE_VALS, VEC_VALS>(M, K, w, dense, mask, row_ptr, col_idx, vals);
#endif
}

// --------------------------------------------------------------- kernels and launchers
//
// Template flags: V, VEC (16-byte row loads: K % 8 == 0 and aligned rows), HAS_MASK, and for
// the compact kernel WRITE_VALS and VEC_VALS (vector stores of a whole vector).

template <int V, bool VEC, bool HAS_MASK>
__global__ void __launch_bounds__(kEncWarps * 32)
    encode_count_kernel(int64_t M, int64_t K, int64_t W, const uint16_t* __restrict__ dense,
                        const uint8_t* __restrict__ mask, int32_t* __restrict__ row_ptr) {
  const int64_t w = (int64_t)blockIdx.x * kEncWarps + (threadIdx.x >> 5);
  if (w < W) count_body<V, VEC, HAS_MASK>(M, K, w, dense, mask, row_ptr);
}

// Phase 2: counts -> inclusive prefix, in place (one CTA).
constexpr int kScanThreads = 1024;
__global__ void __launch_bounds__(kScanThreads) encode_scan_kernel(int32_t* __restrict__ row_ptr,
                                                                   int64_t W) {
  __shared__ int32_t s_warp[32];
  __shared__ int32_t s_carry;
  block_scan_inplace(row_ptr + 1, W, s_warp, &s_carry);
  if (threadIdx.x == 0) row_ptr[0] = 0;
}

template <int V, bool VEC, bool HAS_MASK, bool WRITE_VALS, bool VEC_VALS>
__global__ void __launch_bounds__(kEncWarps * 32, VS_ENC_MINB)
    encode_compact_kernel(int64_t M, int64_t K, int64_t W, const uint16_t* __restrict__ dense,
                          const uint8_t* __restrict__ mask, const int32_t* __restrict__ row_ptr,
                          int32_t* __restrict__ col_idx, uint16_t* __restrict__ vals) {
  const int64_t w = (int64_t)blockIdx.x * kEncWarps + (threadIdx.x >> 5);
  if (w < W)
    compact_body<V, VEC, HAS_MASK, WRITE_VALS, VEC_VALS>(M, K, w, dense, mask, row_ptr, col_idx, vals);
}

// Batched: one grid over the windows of up to kEncMaxBatch problems of one configuration
// (descriptors as a __grid_constant__ parameter; a CTA finds its problem by binary search).
struct EncDesc {
  int64_t M, K, W;
  const uint16_t* dense;
  const uint8_t* mask;
  int32_t* row_ptr;
  int32_t* col_idx;
  uint16_t* vals;
};
constexpr int kEncMaxBatch = 128;
struct EncBatch {
  int count;
  int64_t first_block[kEncMaxBatch + 1];
  EncDesc d[kEncMaxBatch];
};

// Batched kernels: one CTA per kEncWarps windows of one problem; the problem of a CTA is found
// by binary search over first_block.
template <int V, bool VEC, bool HAS_MASK>
__global__ void __launch_bounds__(kEncWarps * 32)
    encode_count_batched_kernel(const __grid_constant__ EncBatch b) {
  const int p = first_problem(b.first_block, b.count, (int64_t)blockIdx.x);
  const EncDesc& d = b.d[p];
  const int64_t w = (blockIdx.x - b.first_block[p]) * kEncWarps + (threadIdx.x >> 5);
  if (w < d.W) count_body<V, VEC, HAS_MASK>(d.M, d.K, w, d.dense, d.mask, d.row_ptr);
}

// one CTA per problem
__global__ void __launch_bounds__(kScanThreads) encode_scan_batched_kernel(const __grid_constant__ EncBatch b) {
  __shared__ int32_t s_warp[32];
  __shared__ int32_t s_carry;
  const EncDesc& d = b.d[blockIdx.x];
  block_scan_inplace(d.row_ptr + 1, d.W, s_warp, &s_carry);
  if (threadIdx.x == 0) d.row_ptr[0] = 0;
}

template <int V, bool VEC, bool HAS_MASK, bool WRITE_VALS, bool VEC_VALS>
__global__ void __launch_bounds__(kEncWarps * 32, VS_ENC_MINB)
    encode_compact_batched_kernel(const __grid_constant__ EncBatch b) {
  const int p = first_problem(b.first_block, b.count, (int64_t)blockIdx.x);
  const EncDesc& d = b.d[p];
  const int64_t w = (blockIdx.x - b.first_block[p]) * kEncWarps + (threadIdx.x >> 5);
  if (w < d.W)
    compact_body<V, VEC, HAS_MASK, WRITE_VALS, VEC_VALS>(d.M, d.K, w, d.dense, d.mask, d.row_ptr,
                                                         d.col_idx, d.vals);
}

// ---------------------------------------------------------- single pass (count + compact)
//
// VS_ENC_FUSED (build time; 0 in the shipped library -- measured slower, see below): full-mode
// batched / single encodes run as ONE pass
// over W.  A CTA takes a tile of T windows (T sized so the tiles of all resident CTAs fit in
// L2: the compact phase re-reads the tile from L2, not HBM), counts them, publishes the tile's
// aggregate in row_ptr at the tile's end slot (flag bit 30; row_ptr was set to a -1 sentinel
// by encode_fill_kernel), looks back over up to 32 predecessor tiles per step with one warp
// (decoupled look-back: aggregates are summed back to the nearest published inclusive prefix),
// publishes its inclusive prefix (the final row_ptr value of that slot), writes the row_ptr of
// its windows and compacts them.  Tiles are ordered by blockIdx, so every predecessor has
// started.  Same output as count -> scan -> compact, bit for bit (458 GPU tests).
// Measured on the DLMC batch (profiles/r02_encode_fused.md): encode class 0.323 ms with
// L2-sized tiles, 0.343 / 0.330 / 0.466 ms with 4 / 8 / 16 windows per tile, against 0.210 ms
// for the shipped count -> scan -> compact: the look-back over published tile statuses
// serialises the tiles of a problem and costs more than the second read of W saves.
#ifndef VS_ENC_FUSED
#define VS_ENC_FUSED 0
#endif
constexpr int32_t kEncAggFlag = 0x40000000;  // status = aggregate | flag; plain = inclusive
constexpr int kEncTileMax = 64;

struct EncFDesc {
  int64_t M, K, W, T;  // T: windows per tile (multiple of kEncWarps)
  const uint16_t* dense;
  const uint8_t* mask;
  int32_t* row_ptr;
  int32_t* col_idx;
  uint16_t* vals;
};
struct EncFBatch {
  int count;
  int64_t first_block[kEncMaxBatch + 1];  // prefix of tiles
  EncFDesc d[kEncMaxBatch];
};

// row_ptr[0 .. W] = -1 for every problem of the batch (the look-back's "not published")
__global__ void encode_fill_kernel(const __grid_constant__ EncFBatch b) {
  const EncFDesc& d = b.d[blockIdx.y];
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= d.W; i += (int64_t)gridDim.x * blockDim.x)
    d.row_ptr[i] = -1;
}

__device__ __forceinline__ int32_t ld_status(const int32_t* p) {
  int32_t v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_status(int32_t* p, int32_t v) {
  asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <int V, bool VEC, bool HAS_MASK, bool WRITE_VALS, bool VEC_VALS>
__global__ void __launch_bounds__(kEncWarps * 32, VS_ENC_MINB)
    encode_fused_batched_kernel(const __grid_constant__ EncFBatch b) {
  __shared__ int32_t cnt[kEncTileMax];
  __shared__ int64_t s_excl;
  const int p = first_problem(b.first_block, b.count, (int64_t)blockIdx.x);
  const EncFDesc& d = b.d[p];
  const int64_t tile = blockIdx.x - b.first_block[p];
  const int64_t w0 = tile * d.T;
  const int64_t w1 = w0 + d.T < d.W ? w0 + d.T : d.W;
  const int nwin = (int)(w1 - w0);
  const int warp = threadIdx.x >> 5, lane = lane_id();
  // ---- count (the tile's rows come from HBM here and from L2 in the compact phase)
  for (int wl = warp; wl < nwin; wl += kEncWarps) {
    uint16_t h[V][8];
    uint32_t c = 0;
#pragma unroll 2
    for (int64_t c0 = 0; c0 < d.K; c0 += kColsPerStep)
      c += __popc(window_keep8<V, VEC, HAS_MASK, false>(d.dense, d.mask, d.M, d.K, w0 + wl,
                                                         c0 + lane * kColsPerLane, h));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if (lane == 0) cnt[wl] = (int32_t)c;
  }
  __syncthreads();
  if (warp == 0) {
    // tile aggregate (lanes sum the counts)
    int32_t agg = 0;
    for (int i = lane; i < nwin; i += 32) agg += cnt[i];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) agg += __shfl_xor_sync(0xffffffffu, agg, o);
    int32_t* status = d.row_ptr + w1;  // this tile's end slot
    int64_t excl = 0;
    if (tile > 0) {
      if (lane == 0) st_status(status, agg | kEncAggFlag);
      // look back: lane j inspects tile (tile - 1 - j) of the current window of predecessors
      int64_t look = tile - 1;  // first predecessor not yet accounted
      while (true) {
        const int64_t t = look - lane;
        int32_t v = 0;
        bool ready = true, incl = false;
        if (t >= 0) {
          const int64_t e = (t + 1) * d.T < d.W ? (t + 1) * d.T : d.W;
          v = ld_status(d.row_ptr + e);
          ready = v != -1;
          incl = ready && !(v & kEncAggFlag);
        }
        // the nearest inclusive predecessor among the 32, and everything before it ready?
        const unsigned inc_mask = __ballot_sync(0xffffffffu, t >= 0 && incl);
        const int first_inc = inc_mask ? __ffs(inc_mask) - 1 : 32;
        const unsigned not_ready = __ballot_sync(0xffffffffu, t >= 0 && !ready && lane < first_inc);
        if (not_ready) {
          __nanosleep(64);
          continue;  // retry the same window of predecessors
        }
        // sum aggregates of lanes < first_inc (and the inclusive value at first_inc)
        int64_t part = 0;
        if (t >= 0 && lane < first_inc) part = v & ~kEncAggFlag;
        if (lane == first_inc && t >= 0) part = v;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
        excl += part;
        if (first_inc < 32 || look - 31 <= 0) break;  // reached an inclusive prefix or tile 0
        look -= 32;
      }
    }
    if (lane == 0) {
      st_status(status, (int32_t)(excl + agg));  // inclusive prefix = final row_ptr[w1]
      if (tile == 0) d.row_ptr[0] = 0;
      s_excl = excl;
    }
  }
  __syncthreads();
  // ---- exclusive starts of the tile's windows; row_ptr of all but the last (its end slot is
  // the status slot, already final)
  __shared__ int64_t starts[kEncTileMax];
  if (warp == 0) {
    int64_t run = s_excl;
    for (int base = 0; base < nwin; base += 32) {
      const int i = base + lane;
      const int32_t c = i < nwin ? cnt[i] : 0;
      int32_t incl = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t x = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += x;
      }
      const int64_t start = run + incl - c;
      if (i < nwin) {
        starts[i] = start;
        if (i + 1 < nwin) d.row_ptr[w0 + i + 1] = (int32_t)(start + c);
      }
      run += __shfl_sync(0xffffffffu, incl, 31);
    }
  }
  __syncthreads();
  // ---- compact (the tile's rows are L2-resident now)
  for (int wl = warp; wl < nwin; wl += kEncWarps)
    compact_body<V, VEC, HAS_MASK, WRITE_VALS, VEC_VALS>(d.M, d.K, w0 + wl, d.dense, d.mask, d.row_ptr,
                                                         d.col_idx, d.vals, starts[wl]);
}

// windows per tile: the tiles of ~2 resident CTAs per SM x 148 SMs within ~64 MB of L2
#ifndef VS_ENC_TILE
#define VS_ENC_TILE 0  // windows per tile; 0 = sized for L2
#endif
static int64_t enc_tile_windows(int64_t K, int V, bool dense, bool mask) {
  if (VS_ENC_TILE > 0) return VS_ENC_TILE;
  const int64_t bytes_per_window = (int64_t)V * K * ((dense ? 2 : 0) + (mask ? 1 : 0));
  int64_t t = bytes_per_window > 0 ? (int64_t)(192 * 1024) / bytes_per_window : kEncTileMax;
  t = t < kEncWarps ? kEncWarps : (t > kEncTileMax ? kEncTileMax : t);
  return t / kEncWarps * kEncWarps;
}

struct EncCfg {
  int V;
  bool VEC, MASK, IDX, VALS, VEC_VALS;
  int key() const { return (((((V * 2 + VEC) * 2 + MASK) * 2 + IDX) * 2 + VALS) * 2 + VEC_VALS); }
};

static EncCfg enc_config(int64_t K, int V, const void* dense, const uint8_t* mask,
                         const int32_t* col_idx, const void* vals) {
  EncCfg c;
  c.V = V;
  // vector path: 16-byte rows (fp16) / 8-byte rows (mask)
  c.VEC = (K % 8 == 0) && !(dense && (reinterpret_cast<uintptr_t>(dense) & 15)) &&
          !(mask && (reinterpret_cast<uintptr_t>(mask) & 7));
  c.MASK = mask != nullptr;
  c.IDX = col_idx != nullptr;
  c.VALS = c.IDX && vals != nullptr;
  c.VEC_VALS = c.VALS && ((reinterpret_cast<uintptr_t>(vals) & (2 * V - 1)) == 0);
  return c;
}

struct EncKernels {
  void (*count_single)(int64_t, int64_t, int64_t, const uint16_t*, const uint8_t*, int32_t*);
  void (*compact_single)(int64_t, int64_t, int64_t, const uint16_t*, const uint8_t*, const int32_t*,
                         int32_t*, uint16_t*);
  void (*count_batched)(EncBatch);
  void (*compact_batched)(EncBatch);
  void (*fused_batched)(EncFBatch);
};

template <int V, bool VEC, bool MASKB>
static EncKernels enc_kernels_vm(const EncCfg& c) {
  EncKernels k;
  k.count_single = encode_count_kernel<V, VEC, MASKB>;
  k.count_batched = encode_count_batched_kernel<V, VEC, MASKB>;
  if (!c.VALS) {
    k.compact_single = encode_compact_kernel<V, VEC, MASKB, false, false>;
    k.compact_batched = encode_compact_batched_kernel<V, VEC, MASKB, false, false>;
    k.fused_batched = encode_fused_batched_kernel<V, VEC, MASKB, false, false>;
  } else if (c.VEC_VALS) {
    k.compact_single = encode_compact_kernel<V, VEC, MASKB, true, true>;
    k.compact_batched = encode_compact_batched_kernel<V, VEC, MASKB, true, true>;
    k.fused_batched = encode_fused_batched_kernel<V, VEC, MASKB, true, true>;
  } else {
    k.compact_single = encode_compact_kernel<V, VEC, MASKB, true, false>;
    k.compact_batched = encode_compact_batched_kernel<V, VEC, MASKB, true, false>;
    k.fused_batched = encode_fused_batched_kernel<V, VEC, MASKB, true, false>;
  }
  return k;
}

template <int V>
static EncKernels enc_kernels_v(const EncCfg& c) {
  if (c.VEC) return c.MASK ? enc_kernels_vm<V, true, true>(c) : enc_kernels_vm<V, true, false>(c);
  return c.MASK ? enc_kernels_vm<V, false, true>(c) : enc_kernels_vm<V, false, false>(c);
}

static EncKernels enc_kernels(const EncCfg& c) {
  switch (c.V) {
    case 1: return enc_kernels_v<1>(c);
    case 2: return enc_kernels_v<2>(c);
    case 4: return enc_kernels_v<4>(c);
    default: return enc_kernels_v<8>(c);
  }
}

// one fill launch + one fused launch for up to kEncMaxBatch full-mode problems of one config
static cudaError_t launch_fused(const EncKernels& k, EncFBatch& b, int64_t tiles, int64_t maxW, cudaStream_t s) {
  b.first_block[b.count] = tiles;
  const dim3 fg((unsigned)std::min<int64_t>(ceil_div64(maxW + 1, 256), 64), (unsigned)b.count);
  encode_fill_kernel<<<fg, 256, 0, s>>>(b);
  k.fused_batched<<<(unsigned)tiles, kEncWarps * 32, 0, s>>>(b);
  return cudaGetLastError();
}
static bool enc_fused_ok(const EncCfg& c, int64_t M, int64_t K, int V) {
  // status words need 2 free high bits: nnz_v < 2^30
  return VS_ENC_FUSED && c.IDX && ceil_div64(M, V) * K < (int64_t(1) << 30);
}

cudaError_t launch_encode(int64_t M, int64_t K, int V, const void* dense, const uint8_t* mask,
                          int32_t* row_ptr, int32_t* col_idx, void* vals, cudaStream_t s) {
  const int64_t W = ceil_div64(M, V);
  if (W == 0) return cudaSuccess;
  if (W > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
  const EncCfg c = enc_config(K, V, dense, mask, col_idx, vals);
  const EncKernels k = enc_kernels(c);
  if (enc_fused_ok(c, M, K, V)) {
    EncFBatch b;
    b.count = 1;
    const int64_t T = enc_tile_windows(K, V, dense != nullptr, mask != nullptr);
    b.d[0] = {M, K, W, T, static_cast<const uint16_t*>(dense), mask, row_ptr, col_idx, static_cast<uint16_t*>(vals)};
    b.first_block[0] = 0;
    return launch_fused(k, b, ceil_div64(W, T), W, s);
  }
  const dim3 grid((unsigned)ceil_div64(W, kEncWarps)), block(kEncWarps * 32);
  const uint16_t* d = static_cast<const uint16_t*>(dense);
  k.count_single<<<grid, block, 0, s>>>(M, K, W, d, mask, row_ptr);
  encode_scan_kernel<<<1, kScanThreads, 0, s>>>(row_ptr, W);
  if (c.IDX)
    k.compact_single<<<grid, block, 0, s>>>(M, K, W, d, mask, row_ptr, col_idx,
                                            static_cast<uint16_t*>(vals));
  return cudaGetLastError();
}

// Problems with W == 0 are handled by the caller.
// Input bytes per batched launch triple (count, scan, compact): VS_ENC_CHUNK_MB (0 = no
// limit, the default).  L2-sized chunks let the compact pass re-read its inputs from L2, but
// measured slower (tools/tune.py, DLMC batch: no limit 247 us, 96 MB 309 us, 48 MB 424 us,
// 24 MB 517 us): fewer, wider launches win.
#ifndef VS_ENC_CHUNK_MB
#define VS_ENC_CHUNK_MB 0
#endif
static constexpr int64_t enc_chunk_bytes() { return (int64_t)VS_ENC_CHUNK_MB * (1LL << 20); }

cudaError_t launch_encode_batched(int64_t count, const int64_t* M, const int64_t* K, const int* V,
                                  const void* const* dense, const uint8_t* const* mask,
                                  int32_t* const* row_ptr, int32_t* const* col_idx,
                                  void* const* vals, int num_sms, cudaStream_t s) {
  std::vector<std::pair<int, int64_t>> order;
  for (int64_t i = 0; i < count; ++i)
    order.push_back({enc_config(K[i], V[i], dense[i], mask[i], col_idx[i], vals[i]).key(), i});
  std::stable_sort(order.begin(), order.end(),
                   [](const auto& a, const auto& b) { return a.first < b.first; });
  EncBatch batch;
  size_t i = 0;
  while (i < order.size()) {
    const int key = order[i].first;
    const int64_t p0 = order[i].second;
    const EncCfg c = enc_config(K[p0], V[p0], dense[p0], mask[p0], col_idx[p0], vals[p0]);
    const EncKernels k = enc_kernels(c);
    if (c.IDX && VS_ENC_FUSED) {
      // full mode: one pass (fill + fused) per group of problems whose counts fit the status
      // encoding; the rest of the group falls through to the two-pass path below
      EncFBatch fb;
      fb.count = 0;
      int64_t tiles = 0, maxW = 0;
      while (i < order.size() && order[i].first == key && fb.count < kEncMaxBatch &&
             enc_fused_ok(c, M[order[i].second], K[order[i].second], V[order[i].second])) {
        const int64_t p = order[i].second;
        const int64_t W = ceil_div64(M[p], V[p]);
        const int64_t T = enc_tile_windows(K[p], V[p], dense[p] != nullptr, mask[p] != nullptr);
        fb.d[fb.count] = {M[p], K[p], W, T, static_cast<const uint16_t*>(dense[p]), mask[p], row_ptr[p],
                          col_idx[p], static_cast<uint16_t*>(vals[p])};
        fb.first_block[fb.count++] = tiles;
        tiles += ceil_div64(W, T);
        maxW = W > maxW ? W : maxW;
        ++i;
      }
      if (fb.count > 0) {
        const cudaError_t e = launch_fused(k, fb, tiles, maxW, s);
        if (e != cudaSuccess) return e;
        continue;
      }
    }
    batch.count = 0;
    int64_t blocks = 0;
    const int threads = kEncWarps * 32;
    int64_t bytes = 0;
    while (i < order.size() && order[i].first == key && batch.count < kEncMaxBatch) {
      const int64_t p = order[i].second;
      const int64_t W = ceil_div64(M[p], V[p]);
      const int64_t nb = ceil_div64(W, kEncWarps);
      if (blocks + nb > 0x7fffffffLL) break;
      // L2-sized chunks: the compact pass re-reads the inputs the count pass just read
      const int64_t pb = M[p] * K[p] * ((dense[p] ? 2 : 0) + (mask[p] ? 1 : 0));
      if (batch.count > 0 && enc_chunk_bytes() > 0 && bytes + pb > enc_chunk_bytes()) break;
      bytes += pb;

      batch.d[batch.count] = {M[p], K[p], W, static_cast<const uint16_t*>(dense[p]), mask[p],
                              row_ptr[p], col_idx[p], static_cast<uint16_t*>(vals[p])};
      batch.first_block[batch.count++] = blocks;
      blocks += nb;
      ++i;
    }
    if (batch.count == 0) return cudaErrorInvalidConfiguration;
    batch.first_block[batch.count] = blocks;
    // one CTA per window (measured slightly faster than a resident-sized grid-stride grid)
    (void)num_sms;
    k.count_batched<<<(unsigned)blocks, threads, 0, s>>>(batch);
    encode_scan_batched_kernel<<<batch.count, kScanThreads, 0, s>>>(batch);
    if (c.IDX) k.compact_batched<<<(unsigned)blocks, threads, 0, s>>>(batch);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace vs
