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
#include <algorithm>
#include <mutex>
#include <utility>
#include <vector>

#include "common.cuh"
#include "dense_select.cuh"

namespace vs {

constexpr int kSpmmWarps = 4;

// Output destinations of a C tile: ND (compile-time bound) row-major matrices with leading
// dimension ldc, each pointer at element (0, 0) of this launch's C.  ND = 1 is the plain
// vs_spmm output (p[0] = C, ldc = N); vs_spmm_scatter stores every tile into n <= ND
// destinations -- e.g. the symmetric-memory C buffers of all ranks, mapped into this GPU's
// address space, so an N-panel shard lands in every rank's replicated row-major C directly
// from the epilogue (no all-gather, no permute).
constexpr int kMaxScatter = 8;
template <int ND>
struct CDst {
  uint16_t* p[ND];
  int n;
  int64_t ldc;
};

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

// Programmatic dependent launch between the launches of ONE batched call (independent
// problems, disjoint outputs): every block lets the next launch of the batch start as soon as
// it is running (the next kernel fills the SMs this one's last wave leaves idle), and waits
// for the previous launch of the batch to complete before it exits, so a launch completes only
// after all earlier launches of the batch did and whatever follows on the stream sees every
// result.  Both are no-ops for a launch made without the PDL attribute (the batch's first).
// (pdl_launch_dependents / pdl_wait_prior: common.cuh)

// Windows of the 128-row blocks the dense-tile kernel takes (dense_select.cuh; dkp = the
// problem's K padded to 64, 0 = not dense-eligible) are skipped, except windows whose col_idx
// is not strictly ascending: the dense kernel leaves those rows to this kernel.  Warp-uniform.
__device__ __forceinline__ bool spmm_skip_window(int64_t dkp, int V, int64_t W, int64_t w,
                                                 const int32_t* __restrict__ row_ptr,
                                                 const int32_t* __restrict__ col_idx, int pb, int pe) {
  if (dkp == 0 || w >= W) return false;
  if (!rb_is_dense(row_ptr, W, V, (w * V) / kDenseRows, dkp, (int64_t)VS_SPMM_DENSE_CF)) return false;
  return window_sorted(col_idx, pb, pe);
}

// SPLIT warps cooperate on one (window, panel) unit: warp part q takes the 16-vector groups
// q, q + SPLIT, ... and the partial accumulators are summed through shared memory by a
// fixed pairwise tree (deterministic).  A CTA has max(4, SPLIT) warps = max(1, 4/SPLIT) units.
template <int SPLIT>
struct SpmmCta {
  static constexpr int kWarps = SPLIT > kSpmmWarps ? SPLIT : kSpmmWarps;
  static constexpr int kUnits = kWarps / SPLIT;
};

template <int V, int NC, bool VEC, int SPLIT, int UNROLL, int ND>
__device__ __forceinline__ void spmm_body(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                                          int64_t bid, const int32_t* __restrict__ row_ptr,
                                          const int32_t* __restrict__ col_idx,
                                          const uint16_t* __restrict__ vals,
                                          const uint16_t* __restrict__ B, const CDst<ND>& cd,
                                          int64_t dkp) {
  constexpr int UPC = SpmmCta<SPLIT>::kUnits;  // units per CTA
  constexpr int NACC = NC * 16;                // accumulator floats per thread
  constexpr int HALF = SPLIT > 1 ? SPLIT / 2 : 1;
  __shared__ float red[UPC * HALF][NACC][32];
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int wid = threadIdx.x >> 5;
  const int part = wid % SPLIT;
  // panel-major CTA order: consecutive CTAs share a B panel (L1/L2 locality)
  const int64_t pn = bid / n_wgroups;
  const int64_t w = (bid - pn * n_wgroups) * UPC + wid / SPLIT;
  const int64_t ncol0 = pn * (64 * NC) + 8 * g;  // this thread's first column
  const int p_begin = w < W ? row_ptr[w] : 0;
  int p_end = w < W ? row_ptr[w + 1] : 0;
  const bool skip = spmm_skip_window(dkp, V, W, w, row_ptr, col_idx, p_begin, p_end);
  const bool active = w < W && !skip;
  if (!active) p_end = p_begin;

  float acc[NC][4][4];
#pragma unroll
  for (int c = 0; c < NC; ++c)
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int e = 0; e < 4; ++e) acc[c][j][e] = 0.f;

  const int kslot[4] = {2 * t, 2 * t + 1, 2 * t + 8, 2 * t + 9};

  constexpr int kStride = 16 * SPLIT;  // distance between a warp's consecutive groups
  if constexpr (UNROLL == 0) {
    // Pipelined: while the MMAs of group i run, the B rows of group i+1 are in flight, its
    // vals are being fetched and the column indices of group i+2 too (two register sets of
    // rows and vals whose roles alternate; one set of column indices, refilled as soon as
    // it has been turned into row addresses).
    auto load_col = [&](int p0, int (&cl)[4]) {
#pragma unroll
      for (int s = 0; s < 4; ++s) {
        const int p = p0 + kslot[s];
        cl[s] = p < p_end ? ldg32i(col_idx + p) : -1;
      }
    };
    auto load_bv = [&](int p0, uint16_t (&b)[4]) {
#pragma unroll
      for (int s = 0; s < 4; ++s) {
        const int p = p0 + kslot[s];
        b[s] = (p < p_end && g < V) ? ldg16(vals + (int64_t)p * V + g) : (uint16_t)0;
      }
    };
    auto load_rows = [&](const int (&cl)[4], uint4 (&r)[4][NC]) {
#pragma unroll
      for (int s = 0; s < 4; ++s) load_brow<NC, VEC>(B, N, cl[s] < 0 ? 0 : cl[s], cl[s] >= 0, ncol0, r[s]);
    };
    auto mma_group = [&](const uint4 (&r)[4][NC], const uint16_t (&b)[4]) {
      const uint32_t b0 = pack_h2(b[0], b[1]);
      const uint32_t b1 = pack_h2(b[2], b[3]);
#pragma unroll
      for (int c = 0; c < NC; ++c)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint32_t w0 = word(r[0][c], j), w1 = word(r[1][c], j);
          const uint32_t w2 = word(r[2][c], j), w3 = word(r[3][c], j);
          mma_16816(acc[c][j], pack_lo(w0, w1), pack_hi(w0, w1), pack_lo(w2, w3),
                    pack_hi(w2, w3), b0, b1);
        }
    };
    int pc = p_begin + 16 * part;
    int coln[4];
    uint16_t bvA[4], bvB[4];
    uint4 rA[4][NC], rB[4][NC];
    load_col(pc, coln);
    load_rows(coln, rA);
    load_bv(pc, bvA);
    load_col(pc + kStride, coln);
    while (pc < p_end) {
      int pn = pc + kStride;
      if (pn < p_end) load_rows(coln, rB);
      load_col(pn + kStride, coln);
      load_bv(pn, bvB);
      mma_group(rA, bvA);
      pc = pn;
      if (pc >= p_end) break;
      pn = pc + kStride;
      if (pn < p_end) load_rows(coln, rA);
      load_col(pn + kStride, coln);
      load_bv(pn, bvA);
      mma_group(rB, bvB);
      pc = pn;
    }
  } else {
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
  }
  // (no early return: the batched kernel calls this body in a loop with barriers)
  const bool store = part == 0 && active;

  // Epilogue: thread holds rows 2t, 2t+1 x columns [ncol0 + 64c, +8).
#pragma unroll
  for (int rr = 0; rr < 2; ++rr) {
    const int r = 2 * t + rr;
    const int64_t i = w * V + r;
    if (!store || r >= V || i >= M) continue;
#pragma unroll
    for (int c = 0; c < NC; ++c) {
      const int64_t n = ncol0 + 64 * c;
      uint32_t o[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) o[j] = f2_to_h2(acc[c][j][rr], acc[c][j][rr + 2]);
#pragma unroll
      for (int d = 0; d < ND; ++d) {
        if (d >= cd.n) break;
        uint16_t* dst = cd.p[d] + i * cd.ldc + n;
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
}

// ------------------------------------------------------------------ kernels + launch

template <int V, int NC, bool VEC, int SPLIT, int UNROLL>
__global__ void __launch_bounds__(SpmmCta<SPLIT>::kWarps * 32)
    spmm_kernel(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                const uint16_t* __restrict__ vals, const uint16_t* __restrict__ B,
                uint16_t* __restrict__ C, int64_t dkp) {
  const CDst<1> cd = {{C}, 1, N};
  spmm_body<V, NC, VEC, SPLIT, UNROLL, 1>(M, N, W, n_wgroups, blockIdx.x, row_ptr, col_idx, vals, B, cd, dkp);
  pdl_wait_prior();  // completes after a dense-tile launch it overlaps (no-op otherwise)
}

// vs_spmm_scatter, register path (unaligned operands or destinations, V = 1)
template <int V, int NC, bool VEC, int SPLIT>
__global__ void __launch_bounds__(SpmmCta<SPLIT>::kWarps * 32)
    spmm_scatter_kernel(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                        const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                        const uint16_t* __restrict__ vals, const uint16_t* __restrict__ B,
                        const __grid_constant__ CDst<kMaxScatter> cd, int64_t dkp) {
  spmm_body<V, NC, VEC, SPLIT, 1, kMaxScatter>(M, N, W, n_wgroups, blockIdx.x, row_ptr, col_idx,
                                               vals, B, cd, dkp);
  pdl_wait_prior();  // completes after a dense-tile launch it overlaps (no-op otherwise)
}

// Batched launch: one grid over the units of up to kSpmmMaxBatch problems that share a
// kernel configuration; the descriptors travel as a __grid_constant__ kernel parameter and a
// CTA finds its problem by binary search of the per-problem first-block table.
struct SpmmDesc {
  int64_t M, N, W, n_wgroups;
  int64_t dkp;  // dense-tile eligibility: K padded to 64 (0 = not eligible)
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const uint16_t* vals;
  const uint16_t* B;
  uint16_t* C;
};
constexpr int kSpmmMaxBatch = 128;
template <int CAP>
struct SpmmBatchT {
  int count;
  int64_t first_block[CAP + 1];  // register path: CTA blocks; cp path: units (window, panel)
  SpmmDesc d[CAP];
};
using SpmmBatch = SpmmBatchT<kSpmmMaxBatch>;

template <int V, int NC, bool VEC, int SPLIT, int UNROLL>
__global__ void __launch_bounds__(SpmmCta<SPLIT>::kWarps * 32)
    spmm_batched_kernel(const __grid_constant__ SpmmBatch b) {
  // grid-stride over the blocks of all problems (launched with one CTA per block, so usually
  // one iteration); the first problem by binary search, then a forward linear advance
  pdl_launch_dependents();
  const int64_t total = b.first_block[b.count];
  int p = first_problem(b.first_block, b.count, (int64_t)blockIdx.x);
  for (int64_t bid = blockIdx.x; bid < total; bid += gridDim.x) {
    while (b.first_block[p + 1] <= bid) ++p;
    const SpmmDesc& d = b.d[p];
    const CDst<1> cd = {{d.C}, 1, d.N};
    spmm_body<V, NC, VEC, SPLIT, UNROLL, 1>(d.M, d.N, d.W, d.n_wgroups, bid - b.first_block[p],
                                            d.row_ptr, d.col_idx, d.vals, d.B, cd, d.dkp);
  }
  pdl_wait_prior();
}

// ---------------------------------------------------- cp.async-staged kernel (default path)
//
// Why (measured on B200, profiles/r02_gather.md): in the register path above lane 4g+t
// loads row slot t, chunk g, so every 8-lane phase of an LDG.128 touches 4 different
// 128-byte lines: random 128-byte row gathers with that lane mapping top out at 9.2 TB/s,
// against 13-15 TB/s for cp.async with 8 lanes per line feeding ldmatrix (and 20 TB/s for a
// bare LDG.128 with 8 lanes per line, which cannot feed mma.sync fragments directly).
//
// Work unit = (row window, panel of 64*NC columns), owned by SPLIT warps of one CTA (SPLIT
// from K only; fixed-order shared-memory reduction, deterministic), as in the register path.
// Each warp streams its 16-vector groups through a D-stage ring in shared memory:
//  * rows: cp.async.cg 16 B per lane, lanes 8q..8q+7 copy one 128-byte line (one row slot,
//    one 64-column chunk-group), so each phase is one line; slot s of a stage keeps chunk c
//    (of 8 per 64 columns) at position c ^ (s & 7), so the 8 rows read by one ldmatrix phase
//    (slots i..i+7, one chunk) hit 8 distinct bank groups;
//  * the group's vals (16 vectors x V fp16) and the column indices of group j + D ride in the
//    same commit group as the rows of group j: the col_idx -> row-address dependency is D
//    groups ahead of the MMAs;
//  * slots past the window end are zero-filled by the copies (src-size 0): 0 x 0 terms;
//  * MMA m16n8k16, A = gathered rows via ldmatrix.x4.trans (M = 16 panel columns, K = 16
//    vector slots), B = vals (K = slots, N = V rows padded to 8), fp32 accumulate;
//  * epilogue: stmatrix.x4.trans turns the accumulator tiles into row-major 16-byte pieces
//    of the V x 64NC output tile (swizzled, in the drained ring), then 16-byte stores.
// Wider panels (NC = 2, 4) amortise the per-group bookkeeping over more gathered bytes.
// VS_SPMM_CA: gathered B rows copied with cp.async.ca (L1-allocating) instead of .cg
// (measured 1.18x slower over the batched DLMC SpMM: the rings leave little L1)
#ifndef VS_SPMM_CA
#define VS_SPMM_CA 0
#endif
template <int V, int NC, int D>
struct CpRing {
  static constexpr int kRowBytes = 16 * 128 * NC;  // one group: 16 slots x 64NC columns fp16
  static constexpr int kValBytes = 16 * V * 2;
  static constexpr int kColBytes = 16 * 4;
  static constexpr int kRaw = D * (kRowBytes + kValBytes) + 2 * D * kColBytes;
  static constexpr int kWarpBytes = (kRaw + 127) / 128 * 128;
};

template <int V, int NC, int SPLIT, int D, int ND>
__device__ __forceinline__ void spmm_cp_body(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                                             int64_t bid, const int32_t* __restrict__ row_ptr,
                                             const int32_t* __restrict__ col_idx,
                                             const uint16_t* __restrict__ vals,
                                             const uint16_t* __restrict__ B,
                                             const CDst<ND>& cd, unsigned char* smem, int64_t dkp) {
  using R = CpRing<V, NC, D>;
  constexpr int UPC = SpmmCta<SPLIT>::kUnits;
  constexpr int HALF = SPLIT > 1 ? SPLIT / 2 : 1;
  constexpr int PW = 64 * NC;  // panel width
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int wid = threadIdx.x >> 5;
  const int part = wid % SPLIT;
  const int64_t pn = bid / n_wgroups;
  const int64_t w = (bid - pn * n_wgroups) * UPC + wid / SPLIT;
  const int64_t n0 = pn * PW;  // first column of the panel
  const int p_begin = w < W ? row_ptr[w] : 0;
  int p_end = w < W ? row_ptr[w + 1] : 0;
  const bool skip = spmm_skip_window(dkp, V, W, w, row_ptr, col_idx, p_begin, p_end);
  const bool active = w < W && !skip;
  if (!active) p_end = p_begin;
  const uint32_t s_rows = smem_u32(smem + wid * R::kWarpBytes);
  const uint32_t s_vals = s_rows + D * R::kRowBytes;
  const uint32_t s_cols = s_vals + D * R::kValBytes;
  // this warp's groups: vectors [first + 16*SPLIT*j, +16)
  const int first = p_begin + 16 * part;
  const int G = first < p_end ? (p_end - first + 16 * SPLIT - 1) / (16 * SPLIT) : 0;
  const int cq = lane >> 3, cc = lane & 7;  // copy role: slots cq + 4k, chunk cc of each 64
  const uint16_t* Bp = B + n0 + 8 * cc;

  // column indices of group j -> col ring entry j % 2D, permuted so that lane L finds the
  // slots it copies (L>>3) + {0, 4, 8, 12} in one 16-byte word
  auto copy_cols = [&](int j) {
    if (lane < 16) {
      const int p = first + 16 * SPLIT * j + lane;
      const bool ok = p < p_end;
      cp_async_zfill<4>(s_cols + (j % (2 * D)) * R::kColBytes + ((lane & 3) * 4 + (lane >> 2)) * 4,
                        ok ? (const void*)(col_idx + p) : (const void*)col_idx, ok ? 4u : 0u);
    }
  };
  // rows + vals of group j, col indices of group j + D; always one commit group
  auto issue = [&](int j) {
    if (j < G) {
      const int p0 = first + 16 * SPLIT * j;
      const uint4 cl = lds128_u32(s_cols + (j % (2 * D)) * R::kColBytes + cq * 16);
      const int cv[4] = {(int)cl.x, (int)cl.y, (int)cl.z, (int)cl.w};
      const uint32_t rs = s_rows + (j % D) * R::kRowBytes;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int sl = cq + 4 * k;
        const bool okp = p0 + sl < p_end;
        const uint16_t* src = Bp + (int64_t)cv[k] * N;
#pragma unroll
        for (int h = 0; h < NC; ++h) {
          const bool ok = okp && (n0 + 64 * h + 8 * cc < N);
#if VS_SPMM_CA
          cp_async_ca16_zfill(rs + sl * (128 * NC) + ((8 * h + (cc ^ (sl & 7))) * 16),
                              ok ? (const void*)(src + 64 * h) : (const void*)B, ok ? 16u : 0u);
#else
          cp_async_zfill<16>(rs + sl * (128 * NC) + ((8 * h + (cc ^ (sl & 7))) * 16),
                             ok ? (const void*)(src + 64 * h) : (const void*)B, ok ? 16u : 0u);
#endif
        }
      }
      if (lane < 16) {
        const int p = p0 + lane;
        const bool ok = p < p_end;
        cp_async_zfill<2 * V>(s_vals + (j % D) * R::kValBytes + lane * (2 * V),
                              ok ? (const void*)(vals + (int64_t)p * V) : (const void*)vals,
                              ok ? (uint32_t)(2 * V) : 0u);
      }
      if (j + D < G) copy_cols(j + D);
    }
    cp_async_commit();
  };

  float acc[NC][4][4];
#pragma unroll
  for (int h = 0; h < NC; ++h)
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int e = 0; e < 4; ++e) acc[h][j][e] = 0.f;

  const int mi = lane >> 3, ri = lane & 7;  // ldmatrix / stmatrix role
  if (G > 0) {
#pragma unroll 1
    for (int j = 0; j < D && j < G; ++j) copy_cols(j);
    cp_async_commit();
    cp_async_wait<0>();
    __syncwarp();
#pragma unroll
    for (int j = 0; j < D - 1; ++j) issue(j);
    const int slot = ri + 8 * (mi >> 1);
#pragma unroll 1
    for (int j = 0; j < G; ++j) {
      issue(j + D - 1);
      cp_async_wait<D - 1>();
      __syncwarp();
      const uint32_t rs = s_rows + (j % D) * R::kRowBytes + slot * (128 * NC);
      const uint32_t vs = s_vals + (j % D) * R::kValBytes;
      uint32_t b0 = 0, b1 = 0;
      if (g < V) {
        b0 = pack_h2(lds16(vs + ((2 * t) * V + g) * 2), lds16(vs + ((2 * t + 1) * V + g) * 2));
        b1 = pack_h2(lds16(vs + ((2 * t + 8) * V + g) * 2), lds16(vs + ((2 * t + 9) * V + g) * 2));
      }
#pragma unroll
      for (int h = 0; h < NC; ++h)
#pragma unroll
        for (int jj = 0; jj < 4; ++jj) {
          const int chunk = 2 * jj + (mi & 1);
          uint32_t a0, a1, a2, a3;
          ldsm_x4_trans(rs + ((8 * h + (chunk ^ ri)) * 16), a0, a1, a2, a3);
          mma_16816(acc[h][jj], a0, a1, a2, a3, b0, b1);
        }
      __syncwarp();
    }
    cp_async_wait<0>();
    __syncwarp();
  }

  if constexpr (SPLIT > 1) {
    // fixed pairwise tree over the unit's parts through the parts' own (drained) rings
    const uint32_t mine = s_rows;
#pragma unroll
    for (int hh = HALF; hh >= 1; hh >>= 1) {
      if (part >= hh && part < 2 * hh) {
#pragma unroll
        for (int h = 0; h < NC; ++h)
#pragma unroll
          for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e)
              asm volatile("st.shared.f32 [%0], %1;" ::"r"(mine + ((((h * 4 + j) * 4 + e) * 32) + lane) * 4),
                           "f"(acc[h][j][e])
                           : "memory");
      }
      __syncthreads();
      if (part < hh) {
        const uint32_t other = mine + hh * R::kWarpBytes;
#pragma unroll
        for (int h = 0; h < NC; ++h)
#pragma unroll
          for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              float v;
              asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v)
                           : "r"(other + ((((h * 4 + j) * 4 + e) * 32) + lane) * 4));
              acc[h][j][e] += v;
            }
      }
      __syncthreads();
    }
  }
  if (part != 0 || !active) return;  // no barrier follows in this unit

  // epilogue: accumulator tile (h, jj) holds C[r = 2t (+1)][n0 + 64h + 16jj + g (+8)];
  // out tile: 8 rows x 8NC chunks of 16 B, chunk c of row r at (c & ~7) | ((c ^ r) & 7)
  const uint32_t s_out = s_rows;
#pragma unroll
  for (int h = 0; h < NC; ++h)
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const int chunk = 4 * q + mi;
      stsm_x4_trans(s_out + ri * (128 * NC) + ((8 * h + (chunk ^ ri)) * 16),
                    f2_to_h2(acc[h][2 * q][0], acc[h][2 * q][1]),
                    f2_to_h2(acc[h][2 * q][2], acc[h][2 * q][3]),
                    f2_to_h2(acc[h][2 * q + 1][0], acc[h][2 * q + 1][1]),
                    f2_to_h2(acc[h][2 * q + 1][2], acc[h][2 * q + 1][3]));
    }
  __syncwarp();
#pragma unroll
  for (int idx = lane; idx < V * 8 * NC; idx += 32) {
    const int r = idx / (8 * NC), ch = idx % (8 * NC);
    const int64_t i = w * V + r;
    const int64_t n = n0 + 8 * ch;
    const uint4 v = lds128_u32(s_out + r * (128 * NC) + (((ch & ~7) | ((ch ^ r) & 7)) * 16));
    if (i < M && n < N) {
#pragma unroll
      for (int d = 0; d < ND; ++d) {
        if (d >= cd.n) break;
        stg128(cd.p[d] + i * cd.ldc + n, v);
      }
    }
  }
}

// VS_SPMM_CP_WARPS: resident warps per SM the register allocation is sized for (build-time
// knob for tools/tune.py variants; 0 = no cap).  24 (80 registers, with D = 2 stages so the
// rings of 24 warps fit in shared memory): batched DLMC SpMM 443 us, against 621 us
// uncapped (~140 registers, 16 warps/SM) and 469 us at 32 warps.
#ifndef VS_SPMM_CP_WARPS
#define VS_SPMM_CP_WARPS 24
#endif
template <int SPLIT>
struct CpMinBlocks {
  static constexpr int v = VS_SPMM_CP_WARPS / SpmmCta<SPLIT>::kWarps > 0
                               ? VS_SPMM_CP_WARPS / SpmmCta<SPLIT>::kWarps : 1;
};

template <int V, int NC, int SPLIT, int D>
__global__ void __launch_bounds__(SpmmCta<SPLIT>::kWarps * 32, CpMinBlocks<SPLIT>::v)
    spmm_cp_kernel(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                   const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                   const uint16_t* __restrict__ vals, const uint16_t* __restrict__ B,
                   uint16_t* __restrict__ C, int64_t dkp) {
  extern __shared__ __align__(128) unsigned char smem[];
  const CDst<1> cd = {{C}, 1, N};
  spmm_cp_body<V, NC, SPLIT, D, 1>(M, N, W, n_wgroups, blockIdx.x, row_ptr, col_idx, vals, B, cd, smem, dkp);
  pdl_wait_prior();  // completes after a dense-tile launch it overlaps (no-op otherwise)
}

// vs_spmm_scatter, cp.async path: the same body, every output tile stored into cd.n destinations
template <int V, int NC, int SPLIT, int D>
__global__ void __launch_bounds__(SpmmCta<SPLIT>::kWarps * 32, CpMinBlocks<SPLIT>::v)
    spmm_cp_scatter_kernel(int64_t M, int64_t N, int64_t W, int64_t n_wgroups,
                           const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                           const uint16_t* __restrict__ vals, const uint16_t* __restrict__ B,
                           const __grid_constant__ CDst<kMaxScatter> cd, int64_t dkp) {
  extern __shared__ __align__(128) unsigned char smem[];
  spmm_cp_body<V, NC, SPLIT, D, kMaxScatter>(M, N, W, n_wgroups, blockIdx.x, row_ptr, col_idx, vals, B,
                                             cd, smem, dkp);
  pdl_wait_prior();  // completes after a dense-tile launch it overlaps (no-op otherwise)
}

template <int V, int NC, int SPLIT, int D>
__global__ void __launch_bounds__(SpmmCta<SPLIT>::kWarps * 32, CpMinBlocks<SPLIT>::v)
    spmm_cp_batched_kernel(const __grid_constant__ SpmmBatch b) {
  extern __shared__ __align__(128) unsigned char smem[];
  pdl_launch_dependents();
  const int64_t total = b.first_block[b.count];
  int p = first_problem(b.first_block, b.count, (int64_t)blockIdx.x);
  for (int64_t bid = blockIdx.x; bid < total; bid += gridDim.x) {
    while (b.first_block[p + 1] <= bid) ++p;
    const SpmmDesc& d = b.d[p];
    const CDst<1> cd = {{d.C}, 1, d.N};
    spmm_cp_body<V, NC, SPLIT, D, 1>(d.M, d.N, d.W, d.n_wgroups, bid - b.first_block[p], d.row_ptr,
                                     d.col_idx, d.vals, d.B, cd, smem, d.dkp);
  }
  pdl_wait_prior();
}

// Kernel configuration of one problem.  NC (64- or 128-column panels) follows N; SPLIT
// (warps per unit, about one per 256 possible vectors of a window, up to 16) follows K only,
// so N-panel shards of a problem run with exactly the same per-element accumulation order
// as the full problem.  UNROLL = 1 (one 16-vector group in flight per warp and iteration,
// metadata one group ahead) won the sweep of profiles/ (tools/tune.py).
struct SpmmCfg {
  int V, NC, SPLIT;
  bool VEC;
  int CP;  // cp.async ring depth (0 = register path)
  bool operator<(const SpmmCfg& o) const {
    return V != o.V ? V < o.V : NC != o.NC ? NC < o.NC : SPLIT != o.SPLIT ? SPLIT < o.SPLIT
                                                         : VEC != o.VEC ? VEC < o.VEC : CP < o.CP;
  }
};

// cp.async path on/off and its ring depth: VS_SPMM_CP = 0 selects the register path,
// otherwise the number of stages D (2 or 3; default 2, see VS_SPMM_CP_WARPS; 4 was slower).  VS_SPMM_CPNC caps the panel width
// (64 * NC columns, NC in {1, 2, 4}; default 2: tools/tune.py over the DLMC batch, batched
// 502 us (cap 2) vs 569 us (cap 4) vs 650 us (cap 1) vs 629 us for the register path).
// Build-time constants (the shipped library has no run-time knobs; tools/tune.py builds
// variants with -D): VS_SPMM_CP = ring depth (0 = register path only), VS_SPMM_CPNC = panel cap.
#ifndef VS_SPMM_CP
#define VS_SPMM_CP 2
#endif
#ifndef VS_SPMM_CPNC
#define VS_SPMM_CPNC 2
#endif
static constexpr int spmm_cp_stages() {
  return VS_SPMM_CP <= 0 ? 0 : VS_SPMM_CP <= 2 ? 2 : 3;
}
static constexpr int spmm_cp_nc_cap() {
  return VS_SPMM_CPNC >= 4 ? 4 : VS_SPMM_CPNC >= 2 ? 2 : 1;
}
static int64_t cp_smem_bytes(int V, int NC, int SPLIT, int D) {
  const int64_t warps = SPLIT > kSpmmWarps ? SPLIT : kSpmmWarps;
  const int64_t raw = (int64_t)D * (16 * 128 * NC + 32 * V) + 2 * D * 64;
  return warps * ((raw + 127) / 128 * 128);
}

static SpmmCfg spmm_config_al(int64_t K, int64_t N, int V, bool b_al16, bool c_al16);
SpmmCfg spmm_config(int64_t K, int64_t N, int V, const void* B, const void* C) {
  return spmm_config_al(K, N, V, (reinterpret_cast<uintptr_t>(B) & 15) == 0,
                        (reinterpret_cast<uintptr_t>(C) & 15) == 0);
}
static SpmmCfg spmm_config_al(int64_t K, int64_t N, int V, bool b_al16, bool c_al16) {
  SpmmCfg c;
  c.V = V;
  // register path: 64-column panels (a K x 64 panel of B stays L1-resident for K <= ~1500;
  // tools/tune.py: 3% faster than 128-column panels; build with -DVS_SPMM_NC=2 for 128)
#ifndef VS_SPMM_NC
#define VS_SPMM_NC 1
#endif
  c.NC = (N <= 64 || VS_SPMM_NC != 2) ? 1 : 2;
  const int64_t q = K >> 8;
  c.SPLIT = q >= 16 ? 16 : q >= 8 ? 8 : q >= 4 ? 4 : q >= 2 ? 2 : 1;
  c.VEC = (N % 8 == 0) && b_al16 && c_al16;
  // cp.async path: 16-byte row copies and stores (VEC), vals copies of 2V >= 4 bytes; panel
  // width follows N (it does not change any element's accumulation order)
  c.CP = (c.VEC && V >= 2) ? spmm_cp_stages() : 0;
  if (c.CP) {
    int nc = N > 128 ? 4 : N > 64 ? 2 : 1;
    if (nc > spmm_cp_nc_cap()) nc = spmm_cp_nc_cap();
    while (nc > 1 && cp_smem_bytes(V, nc, c.SPLIT, c.CP) > 227 * 1024) nc >>= 1;
    c.NC = nc;
  }
  return c;
}

struct SpmmKernels {
  void (*single)(int64_t, int64_t, int64_t, int64_t, const int32_t*, const int32_t*,
                 const uint16_t*, const uint16_t*, uint16_t*, int64_t);
  void (*batched)(SpmmBatch);
  void (*scatter)(int64_t, int64_t, int64_t, int64_t, const int32_t*, const int32_t*,
                  const uint16_t*, const uint16_t*, CDst<kMaxScatter>, int64_t);
  int threads, units_per_cta, batched_ctas_per_sm;
  int smem;  // dynamic shared memory bytes (cp.async path), 0 otherwise
};

// cp path: raise the dynamic shared memory limit of the instantiation once per device
template <int V, int NC, int SPLIT, int D>
static SpmmKernels cp_kernels_of() {
  constexpr int smem = SpmmCta<SPLIT>::kWarps * CpRing<V, NC, D>::kWarpBytes;
  static_assert(smem <= 227 * 1024 || NC > 1, "cp ring does not fit");
  // once per (instantiation, device), thread-safe (std::call_once)
  static std::once_flag once[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (smem > 48 * 1024 && dev >= 0 && dev < 64) {
    std::call_once(once[dev], [] {
      cudaFuncSetAttribute(spmm_cp_kernel<V, NC, SPLIT, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      cudaFuncSetAttribute(spmm_cp_batched_kernel<V, NC, SPLIT, D>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      cudaFuncSetAttribute(spmm_cp_scatter_kernel<V, NC, SPLIT, D>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    });
  }
  return {spmm_cp_kernel<V, NC, SPLIT, D>, spmm_cp_batched_kernel<V, NC, SPLIT, D>,
          spmm_cp_scatter_kernel<V, NC, SPLIT, D>,
          SpmmCta<SPLIT>::kWarps * 32, SpmmCta<SPLIT>::kUnits, 0, smem};
}

template <int V, int NC, int SPLIT>
static SpmmKernels cp_pick_d(int d) {
  if constexpr (SpmmCta<SPLIT>::kWarps * CpRing<V, NC, 2>::kWarpBytes > 227 * 1024) {
    return cp_kernels_of<V, 1, SPLIT, 2>();  // unreachable: spmm_config shrinks NC first
  } else if constexpr (SpmmCta<SPLIT>::kWarps * CpRing<V, NC, 3>::kWarpBytes > 227 * 1024) {
    return cp_kernels_of<V, NC, SPLIT, 2>();
  } else {
    return d == 2 ? cp_kernels_of<V, NC, SPLIT, 2>() : cp_kernels_of<V, NC, SPLIT, 3>();
  }
}

template <int V, int NC>
static SpmmKernels cp_pick_split(int split, int d) {
  switch (split) {
    case 16: return cp_pick_d<V, NC, 16>(d);
    case 8: return cp_pick_d<V, NC, 8>(d);
    case 4: return cp_pick_d<V, NC, 4>(d);
    case 2: return cp_pick_d<V, NC, 2>(d);
    default: return cp_pick_d<V, NC, 1>(d);
  }
}

template <int V>
static SpmmKernels cp_pick(const SpmmCfg& c) {
  switch (c.NC) {
    case 4: return cp_pick_split<V, 4>(c.SPLIT, c.CP);
    case 2: return cp_pick_split<V, 2>(c.SPLIT, c.CP);
    default: return cp_pick_split<V, 1>(c.SPLIT, c.CP);
  }
}

// Main-loop variant (tools/tune.py): 0 (default) = the plain loop; VS_SPMM_PIPE=1 keeps the
// B rows of the next group in flight during the current group's MMAs -- measured 10% slower,
// the kernel is bound by the L1TEX data pipe (ncu: l1tex__data_pipe_lsu_wavefronts at
// 79-93% of peak), not by latency.
#ifndef VS_SPMM_PIPE
#define VS_SPMM_PIPE 0
#endif
static constexpr int spmm_pipe() { return VS_SPMM_PIPE; }

template <int V, int NC, bool VEC, int SPLIT>
static SpmmKernels kernels_of() {
  constexpr int U = spmm_pipe() ? 0 : 1;
  return {spmm_kernel<V, NC, VEC, SPLIT, U>, spmm_batched_kernel<V, NC, VEC, SPLIT, U>,
          spmm_scatter_kernel<V, NC, VEC, SPLIT>,
          SpmmCta<SPLIT>::kWarps * 32, SpmmCta<SPLIT>::kUnits, 0, 0};
}

template <int V, int NC, bool VEC>
static SpmmKernels pick_split(int split) {
  switch (split) {
    case 16: return kernels_of<V, NC, VEC, 16>();
    case 8: return kernels_of<V, NC, VEC, 8>();
    case 4: return kernels_of<V, NC, VEC, 4>();
    case 2: return kernels_of<V, NC, VEC, 2>();
    default: return kernels_of<V, NC, VEC, 1>();
  }
}

template <int V>
static SpmmKernels pick_v(const SpmmCfg& c) {
  if (c.NC == 1) return c.VEC ? pick_split<V, 1, true>(c.SPLIT) : pick_split<V, 1, false>(c.SPLIT);
  return c.VEC ? pick_split<V, 2, true>(c.SPLIT) : pick_split<V, 2, false>(c.SPLIT);
}

static SpmmKernels pick(const SpmmCfg& c) {
  if (c.CP) {
    switch (c.V) {
      case 2: return cp_pick<2>(c);
      case 4: return cp_pick<4>(c);
      default: return cp_pick<8>(c);
    }
  }
  switch (c.V) {
    case 1: return pick_v<1>(c);
    case 2: return pick_v<2>(c);
    case 4: return pick_v<4>(c);
    default: return pick_v<8>(c);
  }
}

static int64_t spmm_blocks(const SpmmKernels& k, const SpmmCfg& c, int64_t M, int64_t N, int V,
                           int64_t* W_out, int64_t* nwg_out) {
  const int64_t W = ceil_div64(M, V);
  const int64_t nwg = ceil_div64(W, k.units_per_cta);
  *W_out = W;
  *nwg_out = nwg;
  return ceil_div64(N, 64 * c.NC) * nwg;
}

#if VS_SPMM_DENSE_CF > 0
bool spmm_dense_eligible(int64_t M, int64_t K, int64_t N, int V, const void* vals, const void* B);
cudaError_t launch_spmm_dense(int64_t count, const int64_t* M, const int64_t* K, const int64_t* N,
                              const int* V, const int32_t* const* row_ptr, const int32_t* const* col_idx,
                              const void* const* vals, const void* const* B, void* const* const* C_dst,
                              const int* nC, const int64_t* ldc, int num_sms, cudaStream_t s);
#else  // shipped library: no dense-tile path (dense_select.cuh)
static bool spmm_dense_eligible(int64_t, int64_t, int64_t, int, const void*, const void*) { return false; }
static cudaError_t launch_spmm_dense(int64_t, const int64_t*, const int64_t*, const int64_t*, const int*,
                                     const int32_t* const*, const int32_t* const*, const void* const*,
                                     const void* const*, void* const* const*, const int*, const int64_t*, int,
                                     cudaStream_t) {
  return cudaSuccess;
}
#endif
static int64_t spmm_dkp(int64_t M, int64_t K, int64_t N, int V, const void* vals, const void* B) {
  return spmm_dense_eligible(M, K, N, V, vals, B) ? ceil_div64(K, 64) * 64 : 0;
}

// tcgen05 gather-ring SpMM (spmm_tc.cu), build-time variant -DVS_SPMM_TC=1: it takes the problems
// of the cp.async path (V >= 2, 16-byte aligned B and C, N % 8 == 0).
#ifndef VS_SPMM_TC
#define VS_SPMM_TC 0
#endif
#if VS_SPMM_TC
bool spmm_tc_eligible(int64_t K, int64_t N, int V, const void* vals, const void* B);
cudaError_t launch_spmm_tc(int64_t count, const int64_t* M, const int64_t* N, const int* V,
                           const int32_t* const* row_ptr, const int32_t* const* col_idx,
                           const void* const* vals, const void* const* B, void* const* const* C_dst,
                           const int* nC, const int64_t* ldc, int num_sms, cudaStream_t s);
static bool spmm_use_tc(const SpmmCfg& c, int64_t K, int64_t N, int V, const void* vals, const void* B) {
  return c.CP != 0 && spmm_tc_eligible(K, N, V, vals, B);
}
#else
static bool spmm_use_tc(const SpmmCfg&, int64_t, int64_t, int, const void*, const void*) { return false; }
static cudaError_t launch_spmm_tc(int64_t, const int64_t*, const int64_t*, const int*, const int32_t* const*,
                                  const int32_t* const*, const void* const*, const void* const*,
                                  void* const* const*, const int*, const int64_t*, int, cudaStream_t) {
  return cudaErrorNotSupported;
}
#endif

// Launch of a gather kernel overlapped (pdl) with the dense-tile kernel launched just before it.
template <typename... KArgs, typename... Args>
static cudaError_t spmm_launch(bool pdl, void (*kern)(KArgs...), unsigned grid, int threads, int smem,
                               cudaStream_t s, Args... args) {
  if (!pdl) {
    kern<<<grid, threads, smem, s>>>(args...);
    return cudaGetLastError();
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3((unsigned)threads);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

cudaError_t launch_spmm(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                        const int32_t* col_idx, const void* vals, const void* B, void* C,
                        int num_sms, cudaStream_t s) {
  const SpmmCfg c = spmm_config(K, N, V, B, C);
  if (spmm_use_tc(c, K, N, V, vals, B)) {
    void* dst[1] = {C};
    void* const* dsts = dst;
    const int one = 1;
    return launch_spmm_tc(1, &M, &N, &V, &row_ptr, &col_idx, &vals, &B, &dsts, &one, &N, num_sms, s);
  }
  const SpmmKernels k = pick(c);
  int64_t W, nwg;
  const int64_t grid = spmm_blocks(k, c, M, N, V, &W, &nwg);
  if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
  if (grid == 0) return cudaSuccess;
  const int64_t dkp = spmm_dkp(M, K, N, V, vals, B);
  if (dkp != 0) {  // dense row blocks first; the gather launch overlaps it
    void* dst[1] = {C};
    void* const* dsts = dst;
    const int one = 1;
    const cudaError_t de = launch_spmm_dense(1, &M, &K, &N, &V, &row_ptr, &col_idx, &vals, &B, &dsts, &one, &N,
                                             num_sms, s);
    if (de != cudaSuccess) return de;
  }
  return spmm_launch(dkp != 0, k.single, (unsigned)grid, k.threads, k.smem, s, M, N, W, nwg, row_ptr, col_idx,
                     static_cast<const uint16_t*>(vals), static_cast<const uint16_t*>(B), static_cast<uint16_t*>(C),
                     dkp);
}

// vs_spmm_scatter: the launch of vs_spmm, every output tile stored into n_dst destinations
// (row-major, leading dimension ldc).  The 16-byte store path needs every destination and
// ldc * 2 bytes 16-byte aligned (and B aligned, N % 8 == 0), as for vs_spmm.
cudaError_t launch_spmm_scatter(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                                const int32_t* col_idx, const void* vals, const void* B,
                                void* const* C_dst, int n_dst, int64_t ldc, int num_sms, cudaStream_t s) {
  if (n_dst < 1 || n_dst > kMaxScatter) return cudaErrorInvalidValue;
  bool c_al = (ldc % 8) == 0;
  CDst<kMaxScatter> cd = {};
  for (int d = 0; d < n_dst; ++d) {
    cd.p[d] = static_cast<uint16_t*>(C_dst[d]);
    c_al = c_al && ((reinterpret_cast<uintptr_t>(C_dst[d]) & 15) == 0);
  }
  cd.n = n_dst;
  cd.ldc = ldc;
  const SpmmCfg c = spmm_config_al(K, N, V, (reinterpret_cast<uintptr_t>(B) & 15) == 0, c_al);
  if (spmm_use_tc(c, K, N, V, vals, B))
    return launch_spmm_tc(1, &M, &N, &V, &row_ptr, &col_idx, &vals, &B, &C_dst, &n_dst, &ldc, num_sms, s);
  const SpmmKernels k = pick(c);
  int64_t W, nwg;
  const int64_t grid = spmm_blocks(k, c, M, N, V, &W, &nwg);
  if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
  if (grid == 0) return cudaSuccess;
  const int64_t dkp = spmm_dkp(M, K, N, V, vals, B);
  if (dkp != 0) {  // dense row blocks first; the gather launch overlaps it
    const cudaError_t de = launch_spmm_dense(1, &M, &K, &N, &V, &row_ptr, &col_idx, &vals, &B, &C_dst, &n_dst, &ldc,
                                             num_sms, s);
    if (de != cudaSuccess) return de;
  }
  return spmm_launch(dkp != 0, k.scatter, (unsigned)grid, k.threads, k.smem, s, M, N, W, nwg, row_ptr, col_idx,
                     static_cast<const uint16_t*>(vals), static_cast<const uint16_t*>(B), cd, dkp);
}

// VS_SPMM_PDL (build-time, default 1): the launches of one batched call after the first use programmatic
// dependent launch (pdl_*); 0 launches them plainly.  Same kernels, same bits.
#ifndef VS_SPMM_PDL
#define VS_SPMM_PDL 1
#endif
static constexpr bool spmm_pdl_on() { return VS_SPMM_PDL != 0; }

// problems with K == 0 are handled by the caller (zero fill); M == 0 or N == 0 skipped.
cudaError_t launch_spmm_batched(int64_t count, const int64_t* M, const int64_t* K, const int64_t* N,
                                const int* V, const int32_t* const* row_ptr,
                                const int32_t* const* col_idx, const void* const* vals,
                                const void* const* B, void* const* C, int num_sms, cudaStream_t s) {
  // group problem indices by configuration (stable: keeps the caller's order inside a group)
  std::vector<std::pair<SpmmCfg, int64_t>> order;
  order.reserve(count);
  std::vector<int64_t> tcM, tcN, tcL;
  std::vector<int> tcV, tcn;
  std::vector<const int32_t*> tcR, tcI;
  std::vector<const void*> tcA, tcB;
  std::vector<void* const*> tcC;
  for (int64_t i = 0; i < count; ++i) {
    const SpmmCfg c = spmm_config(K[i], N[i], V[i], B[i], C[i]);
    if (spmm_use_tc(c, K[i], N[i], V[i], vals[i], B[i])) {
      tcM.push_back(M[i]); tcN.push_back(N[i]); tcL.push_back(N[i]); tcV.push_back(V[i]); tcn.push_back(1);
      tcR.push_back(row_ptr[i]); tcI.push_back(col_idx[i]); tcA.push_back(vals[i]); tcB.push_back(B[i]);
      tcC.push_back(&C[i]);
      continue;
    }
    order.push_back({c, i});
  }
  if (!tcM.empty()) {
    const cudaError_t e = launch_spmm_tc((int64_t)tcM.size(), tcM.data(), tcN.data(), tcV.data(), tcR.data(),
                                         tcI.data(), tcA.data(), tcB.data(), tcC.data(), tcn.data(), tcL.data(),
                                         num_sms, s);
    if (e != cudaSuccess) return e;
  }
  std::stable_sort(order.begin(), order.end(),
                   [](const auto& a, const auto& b) { return a.first < b.first; });
  // the dense-tile kernel first (it takes the dense row blocks; the gather launches below skip
  // them and start while it runs: programmatic dependent launch, disjoint output rows)
  int launched = 0;
  if (VS_SPMM_DENSE_CF != 0) {
    bool any = false;
    for (const auto& o : order)
      any = any || spmm_dense_eligible(M[o.second], K[o.second], N[o.second], V[o.second], vals[o.second], B[o.second]);
    if (any) {
      std::vector<void* const*> dsts(count);
      std::vector<int> ones(count, 1);
      for (int64_t j = 0; j < count; ++j) dsts[j] = &C[j];
      const cudaError_t e = launch_spmm_dense(count, M, K, N, V, row_ptr, col_idx, vals, B, dsts.data(), ones.data(),
                                              N, num_sms, s);
      if (e != cudaSuccess) return e;
      launched = 1;  // the first gather launch overlaps it
    }
  }
  SpmmBatch batch;
  size_t i = 0;
  while (i < order.size()) {
    const SpmmCfg c = order[i].first;
    const SpmmKernels k = pick(c);
    batch.count = 0;
    int64_t blocks = 0;
    while (i < order.size() && !(c < order[i].first) && !(order[i].first < c) &&
           batch.count < kSpmmMaxBatch) {
      const int64_t p = order[i].second;
      int64_t W, nwg;
      const int64_t nb = spmm_blocks(k, c, M[p], N[p], V[p], &W, &nwg);
      if (blocks + nb > 0x7fffffffLL) break;
      SpmmDesc& d = batch.d[batch.count];
      d = {M[p], N[p], W, nwg, spmm_dkp(M[p], K[p], N[p], V[p], vals[p], B[p]), row_ptr[p], col_idx[p],
           static_cast<const uint16_t*>(vals[p]), static_cast<const uint16_t*>(B[p]),
           static_cast<uint16_t*>(C[p])};
      batch.first_block[batch.count] = blocks;
      blocks += nb;
      ++batch.count;
      ++i;
    }
    if (batch.count == 0) return cudaErrorInvalidConfiguration;
    batch.first_block[batch.count] = blocks;
    // one CTA per block (measured slightly faster than a resident-sized grid-stride grid)
    (void)num_sms;
    if (blocks > 0) {
      if (launched > 0 && spmm_pdl_on()) {
        // later launches of the batch overlap the tail of the previous one (see pdl_*)
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)blocks);
        cfg.blockDim = dim3((unsigned)k.threads);
        cfg.dynamicSmemBytes = (size_t)k.smem;
        cfg.stream = s;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        const cudaError_t le = cudaLaunchKernelEx(&cfg, k.batched, batch);
        if (le != cudaSuccess) return le;
      } else {
        k.batched<<<(unsigned)blocks, k.threads, k.smem, s>>>(batch);
      }
      ++launched;
    }
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace vs
