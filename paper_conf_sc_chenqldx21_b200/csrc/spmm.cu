// spmm.cu — C[M x N] = A[M x K] * B[K x N], A in column-vector CSR (§5).
//
// Work unit = (row window w, column panel of 64*NC columns), the paper's V x TileN output
// tile with TileN = 64, here 64 or 128 wide, owned by SPLIT warps of one CTA.
// Each warp walks its share of the window's vectors 16 at a time and issues one
// mma.sync.m16n8k16 (fp16 in, fp32 accumulate) per 16 panel columns.
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
#include <cstdlib>

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

// SPLIT warps cooperate on one (window, panel) unit: warp part q takes the 16-vector groups
// q, q + SPLIT, ... and the partial accumulators are summed through shared memory by a
// fixed pairwise tree (deterministic).  A CTA has max(4, SPLIT) warps = max(1, 4/SPLIT) units.
template <int SPLIT>
struct SpmmCta {
  static constexpr int kWarps = SPLIT > kSpmmWarps ? SPLIT : kSpmmWarps;
  static constexpr int kUnits = kWarps / SPLIT;
};

template <int V, int NC, bool VEC, int SPLIT, int UNROLL>
__global__ void __launch_bounds__(SpmmCta<SPLIT>::kWarps * 32)
    spmm_kernel(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                const uint16_t* __restrict__ vals, const uint16_t* __restrict__ B,
                uint16_t* __restrict__ C) {
  constexpr int UPC = SpmmCta<SPLIT>::kUnits;  // units per CTA
  constexpr int NACC = NC * 16;                // accumulator floats per thread
  constexpr int HALF = SPLIT > 1 ? SPLIT / 2 : 1;
  __shared__ float red[UPC * HALF][NACC][32];
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int wid = threadIdx.x >> 5;
  const int part = wid % SPLIT;
  // panel-major CTA order: consecutive CTAs share a B panel (L1/L2 locality)
  const int64_t bid = blockIdx.x;
  const int64_t pn = bid / n_wgroups;
  const int64_t w = (bid - pn * n_wgroups) * UPC + wid / SPLIT;
  const bool active = w < W;
  const int64_t ncol0 = pn * (64 * NC) + 8 * g;  // this thread's first column
  const int p_begin = active ? row_ptr[w] : 0;
  const int p_end = active ? row_ptr[w + 1] : 0;

  float acc[NC][4][4];
#pragma unroll
  for (int c = 0; c < NC; ++c)
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int e = 0; e < 4; ++e) acc[c][j][e] = 0.f;

  const int kslot[4] = {2 * t, 2 * t + 1, 2 * t + 8, 2 * t + 9};

  // group metadata (column index + this thread's vals element per slot), prefetched one
  // iteration ahead so the col_idx -> B-row dependency is not on every iteration's path.
  // An iteration handles UNROLL groups (this warp's groups are p_begin + 16*(part + SPLIT*i)).
  int col[UNROLL][4];
  uint16_t bv[UNROLL][4];
  auto load_meta = [&](int p0, int (&cl)[4], uint16_t (&b)[4]) {
#pragma unroll
    for (int s = 0; s < 4; ++s) {
      const int p = p0 + kslot[s];
      const bool valid = p < p_end;
      cl[s] = valid ? ldg32i(col_idx + p) : -1;
      b[s] = (valid && g < V) ? ldg16(vals + (int64_t)p * V + g) : (uint16_t)0;
    }
  };
  constexpr int kStride = 16 * SPLIT;  // distance between a warp's consecutive groups
  int p0 = p_begin + 16 * part;
#pragma unroll
  for (int u = 0; u < UNROLL; ++u) load_meta(p0 + u * kStride, col[u], bv[u]);
  while (p0 < p_end) {
    uint4 rows[UNROLL][4][NC];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u)
#pragma unroll
      for (int s = 0; s < 4; ++s)
        load_brow<NC, VEC>(B, N, col[u][s] < 0 ? 0 : col[u][s], col[u][s] >= 0, ncol0, rows[u][s]);
    const int p1 = p0 + UNROLL * kStride;
    int coln[UNROLL][4];
    uint16_t bvn[UNROLL][4];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) load_meta(p1 + u * kStride, coln[u], bvn[u]);
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      const uint32_t b0 = pack_h2(bv[u][0], bv[u][1]);
      const uint32_t b1 = pack_h2(bv[u][2], bv[u][3]);
#pragma unroll
      for (int c = 0; c < NC; ++c)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint32_t w0 = word(rows[u][0][c], j), w1 = word(rows[u][1][c], j);
          const uint32_t w2 = word(rows[u][2][c], j), w3 = word(rows[u][3][c], j);
          mma_16816(acc[c][j], pack_lo(w0, w1), pack_hi(w0, w1), pack_lo(w2, w3),
                    pack_hi(w2, w3), b0, b1);
        }
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u)
#pragma unroll
      for (int s = 0; s < 4; ++s) {
        col[u][s] = coln[u][s];
        bv[u][s] = bvn[u][s];
      }
    p0 = p1;
  }

  if constexpr (SPLIT > 1) {
    // pairwise tree over the unit's parts: at each level parts [h, 2h) hand their sums to
    // parts [0, h) (part q adds part q + h)
    const int ubase = (wid / SPLIT) * HALF;
#pragma unroll
    for (int h = HALF; h >= 1; h >>= 1) {
      if (part >= h && part < 2 * h) {
#pragma unroll
        for (int c = 0; c < NC; ++c)
#pragma unroll
          for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) red[ubase + part - h][(c * 4 + j) * 4 + e][lane] = acc[c][j][e];
      }
      __syncthreads();
      if (part < h) {
#pragma unroll
        for (int c = 0; c < NC; ++c)
#pragma unroll
          for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[c][j][e] += red[ubase + part][(c * 4 + j) * 4 + e][lane];
      }
      __syncthreads();
    }
    if (part != 0) return;
  }
  if (!active) return;

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

template <int V, int NC, bool VEC, int SPLIT, int UNROLL>
static void launch_cfg(int64_t M, int64_t N, int64_t W, const int32_t* row_ptr,
                       const int32_t* col_idx, const uint16_t* vals, const uint16_t* B,
                       uint16_t* C, cudaStream_t s) {
  constexpr int UPC = SpmmCta<SPLIT>::kUnits;
  const int64_t n_panels = ceil_div64(N, 64 * NC);
  const int64_t n_wgroups = ceil_div64(W, UPC);
  const int64_t grid = n_panels * n_wgroups;
  spmm_kernel<V, NC, VEC, SPLIT, UNROLL><<<(unsigned)grid, SpmmCta<SPLIT>::kWarps * 32, 0, s>>>(
      M, N, W, n_wgroups, row_ptr, col_idx, vals, B, C);
}

// Tuning knobs (read once from the environment; for experiments only -- the defaults are
// the shipped configuration): VS_SPMM_UNROLL in {1,2}, VS_SPMM_NC in {0 (auto),1,2},
// VS_SPMM_SPLIT_SHIFT (SPLIT = K >> shift, clamped to [1,16] and rounded down to a power of 2).
struct SpmmTune {
  int unroll = 1, nc = 0, split_shift = 8;
};
static const SpmmTune& spmm_tune() {
  static const SpmmTune t = [] {
    SpmmTune r;
    if (const char* e = std::getenv("VS_SPMM_UNROLL")) r.unroll = std::atoi(e) == 1 ? 1 : 2;
    if (const char* e = std::getenv("VS_SPMM_NC")) r.nc = std::atoi(e);
    if (const char* e = std::getenv("VS_SPMM_SPLIT_SHIFT")) r.split_shift = std::atoi(e);
    return r;
  }();
  return t;
}

template <int V, int NC, bool VEC, int UNROLL>
static void launch_split(int64_t M, int64_t K, int64_t N, int64_t W, const int32_t* row_ptr,
                         const int32_t* col_idx, const uint16_t* vals, const uint16_t* B,
                         uint16_t* C, cudaStream_t s) {
  // Warps per (window, panel) unit, from K (the bound on a window's vector count): about
  // one warp per 2^shift possible vectors, up to 16.  It must not depend on N, so that N-panel
  // shards accumulate in exactly the order of the full problem.
  const int64_t q = K >> spmm_tune().split_shift;
  if (q >= 16)
    launch_cfg<V, NC, VEC, 16, UNROLL>(M, N, W, row_ptr, col_idx, vals, B, C, s);
  else if (q >= 8)
    launch_cfg<V, NC, VEC, 8, UNROLL>(M, N, W, row_ptr, col_idx, vals, B, C, s);
  else if (q >= 4)
    launch_cfg<V, NC, VEC, 4, UNROLL>(M, N, W, row_ptr, col_idx, vals, B, C, s);
  else if (q >= 2)
    launch_cfg<V, NC, VEC, 2, UNROLL>(M, N, W, row_ptr, col_idx, vals, B, C, s);
  else
    launch_cfg<V, NC, VEC, 1, UNROLL>(M, N, W, row_ptr, col_idx, vals, B, C, s);
}

template <int V, int NC, bool VEC>
static void launch_unroll(int64_t M, int64_t K, int64_t N, int64_t W, const int32_t* row_ptr,
                          const int32_t* col_idx, const uint16_t* vals, const uint16_t* B,
                          uint16_t* C, cudaStream_t s) {
  if (spmm_tune().unroll == 1)
    launch_split<V, NC, VEC, 1>(M, K, N, W, row_ptr, col_idx, vals, B, C, s);
  else
    launch_split<V, NC, VEC, 2>(M, K, N, W, row_ptr, col_idx, vals, B, C, s);
}

template <int V>
static cudaError_t launch_spmm_v(int64_t M, int64_t K, int64_t N, const int32_t* row_ptr,
                                 const int32_t* col_idx, const uint16_t* vals, const uint16_t* B,
                                 uint16_t* C, bool vec, int num_sms, cudaStream_t s) {
  const int64_t W = ceil_div64(M, V);
  (void)num_sms;
  const int NC = spmm_tune().nc == 0 ? ((N <= 64) ? 1 : 2) : (spmm_tune().nc == 2 && N > 64 ? 2 : 1);
  if (ceil_div64(N, 64 * NC) * W > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
  if (NC == 1) {
    if (vec) launch_unroll<V, 1, true>(M, K, N, W, row_ptr, col_idx, vals, B, C, s);
    else launch_unroll<V, 1, false>(M, K, N, W, row_ptr, col_idx, vals, B, C, s);
  } else {
    if (vec) launch_unroll<V, 2, true>(M, K, N, W, row_ptr, col_idx, vals, B, C, s);
    else launch_unroll<V, 2, false>(M, K, N, W, row_ptr, col_idx, vals, B, C, s);
  }
  return cudaGetLastError();
}

cudaError_t launch_spmm(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                        const int32_t* col_idx, const void* vals, const void* B, void* C,
                        int num_sms, cudaStream_t s) {
  const uint16_t* v = static_cast<const uint16_t*>(vals);
  const uint16_t* b = static_cast<const uint16_t*>(B);
  uint16_t* c = static_cast<uint16_t*>(C);
  const bool vec = (N % 8 == 0) && ((reinterpret_cast<uintptr_t>(B) & 15) == 0) &&
                   ((reinterpret_cast<uintptr_t>(C) & 15) == 0);
  switch (V) {
    case 1: return launch_spmm_v<1>(M, K, N, row_ptr, col_idx, v, b, c, vec, num_sms, s);
    case 2: return launch_spmm_v<2>(M, K, N, row_ptr, col_idx, v, b, c, vec, num_sms, s);
    case 4: return launch_spmm_v<4>(M, K, N, row_ptr, col_idx, v, b, c, vec, num_sms, s);
    case 8: return launch_spmm_v<8>(M, K, N, row_ptr, col_idx, v, b, c, vec, num_sms, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace vs
