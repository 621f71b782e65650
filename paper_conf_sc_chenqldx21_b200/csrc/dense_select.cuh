// dense_select.cuh — which 128-row blocks of a problem take the dense-tile tcgen05 kernels
// (dense_tile.cu) instead of the column-vector gather kernels (spmm.cu / sddmm.cu).
//
// B200 cost model.  A stored V x 1 vector costs the gather kernels one
// gathered dense row: 2*L bytes through L2 -> SM (L = N for SpMM, the inner K for SDDMM),
// i.e. V flop per gathered byte.  A dense 128-row tile costs 2 * 128 * Lc * L tensor flops
// (Lc = the padded other dimension: K for SpMM, the mask columns for SDDMM) whatever the
// density.  With the gather at Bg bytes/s and the tcgen05 tiles at Fd flop/s, the dense tile
// is cheaper when  nnz_v(rb) * 2L / Bg  >  2 * 128 * Lc * L / Fd,  i.e.
//     nnz_v(rb) * VS_DENSE_CF  >  128 * Lc,         VS_DENSE_CF = Fd / Bg  (flop per byte).
// The decision depends only on the row block's vectors and the problem's shape, so the gather
// kernels and the dense kernels (and any N-panel or 128-row-aligned row-window shard of the
// problem) take it identically.  Windows of a dense row block whose col_idx is not strictly
// ascending stay with the gather kernels (the dense kernels rely on sorted windows).
#pragma once

#include <stdint.h>

#include "common.cuh"

// Build-time cost-model constants (flop per gathered byte), one per op; 0 = the dense-tile
// kernel of that op is not built and never launched (every row block stays with the gather
// kernel).  VS_SDDMM_DENSE_CF / VS_SDDMM_DENSE_KMIN: the 128 x 128-unit SDDMM kernel
// (dense_tile.cu) takes the 128-row blocks with nnz_v(rb) * 32 > 128 * Lc (stored density
// above V/32) of problems with inner dimension K >= 256.  Tuned on B200 (DESIGN.md §7.8,
// profiles/r03_dense_sddmm.md): over the DLMC batch the step is 0.900 -> 0.830 ms, while the
// single calls keep the per-cell crossovers with cuBLAS Hgemm (a dense-tile launch adds a
// ~1-2 us floor to a single call; rules taking smaller K or lower density made the batch
// faster, 0.816 ms, but single calls up to 1.5x slower).  VS_SPMM_DENSE_CF: the dense-tile
// SpMM, measured slower than the gather kernel at DLMC sizes (profiles/r02_dense_tile.md) -> 0.
#ifndef VS_SDDMM_DENSE_CF
#define VS_SDDMM_DENSE_CF 32
#endif
// smallest inner dimension K the dense-tile SDDMM takes (a shape rule: every shard of a problem
// decides alike)
#ifndef VS_SDDMM_DENSE_KMIN
#define VS_SDDMM_DENSE_KMIN 256
#endif
#ifndef VS_SPMM_DENSE_CF
#define VS_SPMM_DENSE_CF 0
#endif

namespace vs {

constexpr int kDenseRows = 128;  // rows per dense tile (tcgen05 M / N)

// 128-row block rb of a problem with W windows of V rows: window range [w0, w1)
__host__ __device__ __forceinline__ void rb_windows(int64_t rb, int V, int64_t W, int64_t& w0, int64_t& w1) {
  w0 = rb * (kDenseRows / V);
  w1 = w0 + kDenseRows / V;
  if (w1 > W) w1 = W;
}

// dense iff nnz_v(rb) * cf > 128 * Lc (Lc padded to the dense tile granularity)
__device__ __forceinline__ bool rb_is_dense(const int32_t* __restrict__ row_ptr, int64_t W, int V,
                                            int64_t rb, int64_t Lc_padded, int64_t cf) {
  int64_t w0, w1;
  rb_windows(rb, V, W, w0, w1);
  const int64_t nnz = (int64_t)__ldg(row_ptr + w1) - (int64_t)__ldg(row_ptr + w0);
  return nnz * cf > (int64_t)kDenseRows * Lc_padded;
}
// SDDMM [M x N mask]: Lc = the mask columns padded to the 128-column tiles of the dense kernel
__device__ __forceinline__ bool sddmm_rb_dense(const int32_t* __restrict__ row_ptr, int64_t W, int V,
                                               int64_t rb, int64_t N) {
  return rb_is_dense(row_ptr, W, V, rb, ceil_div64(N, 128) * 128, (int64_t)VS_SDDMM_DENSE_CF);
}

// warp-uniform: col_idx[pb, pe) strictly ascending (every lane returns the same answer).
// 128 entries per round trip (4 coalesced loads per lane in flight).
static __device__ __noinline__ bool window_sorted(const int32_t* __restrict__ col_idx, int64_t pb, int64_t pe) {
  const int lane = lane_id();
  int prev_last = -1;  // last entry of the previous row of 32 (entries are >= 0)
  for (int64_t base = pb; base < pe; base += 128) {
    int c[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int64_t p = base + 32 * j + lane;
      c[j] = p < pe ? __ldg(col_idx + p) : 0x7fffffff;
    }
    bool bad = false;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int prev = __shfl_up_sync(0xffffffffu, c[j], 1);
      if (lane == 0) prev = prev_last;
      bad |= (base + 32 * j + lane < pe) && (c[j] <= prev);
      prev_last = __shfl_sync(0xffffffffu, c[j], 31);
    }
    if (__any_sync(0xffffffffu, bad)) return false;
  }
  return true;
}

}  // namespace vs
