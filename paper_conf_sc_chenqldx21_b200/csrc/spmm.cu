// spmm.cu — C[M x N] = A[M x K] * B[K x N], A in column-vector CSR (§5).
//
// Work unit = one warp per (row window w, column panel of 64*NC columns), the paper's
// V x TileN output tile with TileN = 64, here 64 or 128 wide.  The warp walks
// the window's vectors 16 at a time and issues one mma.sync.m16n8k16 (fp16 in, fp32
// accumulate) per 16 panel columns.
//
// Operand switch: the MMA's M dimension is the panel columns, its N dimension
// is V (padded to 8) and its K dimension is the vector index, so C_w^T = Bg^T * vals_w^T.
// Fragment/memory mapping (B200 re-design):
//   lane = 4*g + t.  Thread t owns the 4 vector slots k in {2t, 2t+1, 2t+8, 2t+9} of each
//   16-vector group and loads, for each slot, 16 bytes = 8 consecutive panel columns
//   [8g, 8g+8) of the gathered row B[col_idx[p]] (one LDG.128 per slot and 64-column
//   chunk; the 8 lanes sharing t read one full 128-byte line: four 128B-coalesced
//   transactions per instruction).
//   M-row permutation: MMA tile j (of 4 per 64 columns), row g <-> column 8g+2j and row
//   g+8 <-> column 8g+2j+1, so that the A-fragment words are PRMT pairs of the loaded
//   words and the accumulators of a thread cover 8 consecutive columns of output rows
//   2t and 2t+1: the epilogue stores 16 bytes per row with no shuffles.
//   B fragment (k = vector slot, n = row r < V) is vals[p*V + g].
#include "common.cuh"

namespace vs {

constexpr int kSpmmWarps = 4;

template <int NC, bool VEC>
__device__ __forceinline__ void load_brow(const uint16_t* __restrict__ B, int64_t N, int col,
                                          bool valid, int64_t ncol0, uint4 (&r)[NC]) {
#pragma unroll
  for (int c = 0; c < NC; ++c) {
    const int64_t n = ncol0 + 64 * c;
    if (VEC) {
      r[c] = (valid && n < N) ? ldg128(B + (int64_t)col * N + n) : make_uint4(0, 0, 0, 0);
    } else {
      uint16_t h[8];
#pragma unroll
      for (int e = 0; e < 8; ++e)
        h[e] = (valid && n + e < N) ? ldg16(B + (int64_t)col * N + n + e) : (uint16_t)0;
      r[c] = make_uint4(pack_h2(h[0], h[1]), pack_h2(h[2], h[3]), pack_h2(h[4], h[5]),
                        pack_h2(h[6], h[7]));
    }
  }
}

__device__ __forceinline__ uint32_t word(const uint4& v, int j) {
  return j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w));
}

template <int V, int NC, bool VEC>
__global__ void __launch_bounds__(kSpmmWarps * 32)
    spmm_kernel(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                const uint16_t* __restrict__ vals, const uint16_t* __restrict__ B,
                uint16_t* __restrict__ C) {
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  // panel-major CTA order: consecutive CTAs share a B panel (L1/L2 locality)
  const int64_t bid = blockIdx.x;
  const int64_t pn = bid / n_wgroups;
  const int64_t w = (bid - pn * n_wgroups) * kSpmmWarps + (threadIdx.x >> 5);
  if (w >= W) return;
  const int64_t ncol0 = pn * (64 * NC) + 8 * g;  // this thread's first column
  const int p_begin = row_ptr[w];
  const int p_end = row_ptr[w + 1];

  float acc[NC][4][4];
#pragma unroll
  for (int c = 0; c < NC; ++c)
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int e = 0; e < 4; ++e) acc[c][j][e] = 0.f;

  const int kslot[4] = {2 * t, 2 * t + 1, 2 * t + 8, 2 * t + 9};

  // Main loop: 32 vectors (two 16-vector MMA groups) per iteration, all loads issued
  // before the MMAs (the ILP argument of P:906-914, without the fence trick).
  for (int p0 = p_begin; p0 < p_end; p0 += 32) {
    uint4 rows[2][4][NC];
    uint16_t bv[2][4];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
#pragma unroll
      for (int s = 0; s < 4; ++s) {
        const int p = p0 + 16 * h + kslot[s];
        const bool valid = p < p_end;
        const int col = valid ? ldg32i(col_idx + p) : 0;
        bv[h][s] = (valid && g < V) ? ldg16(vals + (int64_t)p * V + g) : (uint16_t)0;
        load_brow<NC, VEC>(B, N, col, valid, ncol0, rows[h][s]);
      }
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const uint32_t b0 = pack_h2(bv[h][0], bv[h][1]);
      const uint32_t b1 = pack_h2(bv[h][2], bv[h][3]);
#pragma unroll
      for (int c = 0; c < NC; ++c)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint32_t w0 = word(rows[h][0][c], j), w1 = word(rows[h][1][c], j);
          const uint32_t w2 = word(rows[h][2][c], j), w3 = word(rows[h][3][c], j);
          mma_16816(acc[c][j], pack_lo(w0, w1), pack_hi(w0, w1), pack_lo(w2, w3),
                    pack_hi(w2, w3), b0, b1);
        }
    }
  }

  // Epilogue: thread holds rows 2t, 2t+1 x columns [ncol0 + 64c, +8).
#pragma unroll
  for (int rr = 0; rr < 2; ++rr) {
    const int r = 2 * t + rr;
    const int64_t i = w * V + r;
    if (r >= V || i >= M) continue;
#pragma unroll
    for (int c = 0; c < NC; ++c) {
      const int64_t n = ncol0 + 64 * c;
      uint32_t o[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) o[j] = f2_to_h2(acc[c][j][rr], acc[c][j][rr + 2]);
      uint16_t* dst = C + i * N + n;
      if (VEC) {
        if (n < N) stg128(dst, make_uint4(o[0], o[1], o[2], o[3]));
      } else {
#pragma unroll
        for (int e = 0; e < 8; ++e)
          if (n + e < N) dst[e] = (uint16_t)((o[e >> 1] >> (16 * (e & 1))) & 0xFFFF);
      }
    }
  }
}

template <int V>
static cudaError_t launch_spmm_v(int64_t M, int64_t K, int64_t N, const int32_t* row_ptr,
                                 const int32_t* col_idx, const uint16_t* vals, const uint16_t* B,
                                 uint16_t* C, bool vec, cudaStream_t s) {
  (void)K;
  const int64_t W = ceil_div64(M, V);
  const int NC = (N <= 64) ? 1 : 2;
  const int64_t n_panels = ceil_div64(N, 64 * NC);
  const int64_t n_wgroups = ceil_div64(W, kSpmmWarps);
  const int64_t grid = n_panels * n_wgroups;
  if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
  dim3 block(kSpmmWarps * 32);
#define VS_SPMM(NCV, VECB)                                                                 \
  spmm_kernel<V, NCV, VECB><<<(unsigned)grid, block, 0, s>>>(M, N, W, n_wgroups, row_ptr, \
                                                             col_idx, vals, B, C)
  if (NC == 1) {
    if (vec) VS_SPMM(1, true); else VS_SPMM(1, false);
  } else {
    if (vec) VS_SPMM(2, true); else VS_SPMM(2, false);
  }
#undef VS_SPMM
  return cudaGetLastError();
}

cudaError_t launch_spmm(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                        const int32_t* col_idx, const void* vals, const void* B, void* C,
                        cudaStream_t s) {
  const uint16_t* v = static_cast<const uint16_t*>(vals);
  const uint16_t* b = static_cast<const uint16_t*>(B);
  uint16_t* c = static_cast<uint16_t*>(C);
  const bool vec = (N % 8 == 0) && ((reinterpret_cast<uintptr_t>(B) & 15) == 0) &&
                   ((reinterpret_cast<uintptr_t>(C) & 15) == 0);
  switch (V) {
    case 1: return launch_spmm_v<1>(M, K, N, row_ptr, col_idx, v, b, c, vec, s);
    case 2: return launch_spmm_v<2>(M, K, N, row_ptr, col_idx, v, b, c, vec, s);
    case 4: return launch_spmm_v<4>(M, K, N, row_ptr, col_idx, v, b, c, vec, s);
    case 8: return launch_spmm_v<8>(M, K, N, row_ptr, col_idx, v, b, c, vec, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace vs
