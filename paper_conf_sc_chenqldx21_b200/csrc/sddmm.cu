// sddmm.cu — out = (A * B) sampled at a column-vector mask (§6).
//
//   out_vals[p*V + r] = sum_k A[wV+r][k] * Bt[col_idx[p]][k]   (p in window w)
//
// Work decomposition (B200 re-design; the paper launches ceil(M/V) x ceil(N/32) CTAs over
// the DENSE N, many of them idle): a persistent grid of warps; the 16-vector
// chunks of every row window are owned by q warps of the launch (warp j takes chunks j,
// j + q, ...), q chosen on the device from nnz_v = row_ptr[W] (no host sync) so that every
// warp gets about the same number of chunks.  Chunks never straddle windows, so the A rows
// of a window are loaded once per warp.
//
// MMA mapping (operand switch as in P:1059-1063): M = 16 vectors of the slice, N = V rows of
// the window (padded to 8), K = the inner dimension.  Both operands are K-contiguous rows
// (Bt rows and A rows), so a thread's two 16-byte loads per row and 64-wide K step feed the
// fragments directly: MMA k-slot pair 2t (resp. 2t+8) of sub-step j <-> inner index
// k0 + 8t + 2j (resp. k0 + 32 + 8t + 2j), the same permutation on both operands.  Every
// partial sum stays inside one MMA accumulator, so the paper's cross-octet shuffle+FADD
// reduction (17-30% of instructions) disappears.
#include <algorithm>
#include <utility>
#include <vector>

#include "common.cuh"
#include "dense_select.cuh"

namespace vs {

constexpr int kSddmmWarps = 4;
// K % 128 == 0 (KC = 2 body) and K == 64 (pair body): unpredicated loads (load_seg2_fast)
#ifndef VS_SDDMM_FAST
#define VS_SDDMM_FAST 1
#endif
// resident CTAs per SM the register allocation is sized for (tools/tune.py over the DLMC batch:
// 4 -> 551 us, 5 -> 516 us (12 B of spills), 6 -> 644 us, 8 -> 782 us: spills in the loop)
#ifndef VS_SDDMM_MINB
#define VS_SDDMM_MINB 5
#endif

template <bool VEC>
__device__ __forceinline__ void load_seg2(const uint16_t* __restrict__ row, int64_t K, int64_t k,
                                          bool valid, uint4& s0, uint4& s1) {
  // row[k .. k+8) and row[k+32 .. k+40): the 4 lanes of a row read 64 contiguous bytes
  // per instruction (two full sectors)
  if (VEC) {
    s0 = (valid && k < K) ? ldg128(row + k) : make_uint4(0, 0, 0, 0);
    s1 = (valid && k + 32 < K) ? ldg128(row + k + 32) : make_uint4(0, 0, 0, 0);
  } else {
    uint16_t h[16];
#pragma unroll
    for (int e = 0; e < 16; ++e) {
      const int64_t kk = k + (e < 8 ? e : 24 + e);
      h[e] = (valid && kk < K) ? ldg16(row + kk) : (uint16_t)0;
    }
    s0 = make_uint4(pack_h2(h[0], h[1]), pack_h2(h[2], h[3]), pack_h2(h[4], h[5]), pack_h2(h[6], h[7]));
    s1 = make_uint4(pack_h2(h[8], h[9]), pack_h2(h[10], h[11]), pack_h2(h[12], h[13]),
                    pack_h2(h[14], h[15]));
  }
}

// K % 64 == 0 fast path: no bounds predicates and no zero fill.  Slots past the window end and
// MMA rows >= V read a valid dummy row (row 0) instead: they only feed accumulator rows / columns
// that store_chunk never writes (rows >= M are written as +0 there), so every stored output is the
// same sum in the same MMA order as the guarded path -> the same bits, with ~6 fewer instructions
// per 16-byte load (the predicates, CS2R zeroing and branch of the guarded loads).
__device__ __forceinline__ void load_seg2_fast(const uint16_t* __restrict__ row, int64_t k, uint4& s0,
                                               uint4& s1) {
  s0 = ldg128(row + k);
  s1 = ldg128(row + k + 32);
}

__device__ __forceinline__ uint32_t wordj(const uint4& v, int j) {
  return j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w));
}

// Stores the two vectors (M rows g, g+8) of a 16-vector chunk held in acc, restricted to
// the vectors below `hi`.
template <int V>
__device__ __forceinline__ void store_chunk(const float (&acc)[4], int64_t v0, int64_t hi,
                                            int64_t w, int64_t M, int g, int t,
                                            uint16_t* __restrict__ out, bool out4) {
#pragma unroll
  for (int q = 0; q < 2; ++q) {
    const int64_t v = v0 + g + 8 * q;
    if (v >= hi) continue;
    const int r = 2 * t;
    const float f0 = (w * V + r < M) ? acc[2 * q] : 0.f;
    const float f1 = (w * V + r + 1 < M) ? acc[2 * q + 1] : 0.f;
    uint16_t* dst = out + v * V + r;
    if (V >= 2 && out4) {
      if (r < V) *reinterpret_cast<uint32_t*>(dst) = f2_to_h2(f0, f1);
    } else {
      if (r < V) dst[0] = f_to_h(f0);
      if (r + 1 < V) dst[1] = f_to_h(f1);
    }
  }
}

// One warp computes the 16-vector chunks j0, j0 + q, j0 + 2q, ... of window w.
// Dependency chain: row_ptr[w], row_ptr[w+1] -> col_idx of the first chunk -> the gathered
// Bt rows; then ONE round trip per chunk and K block of 64*KC: the Bt rows (and, when the
// block is not the whole K, the window's A rows) of all KC 64-wide chunks are loaded
// together, then the KC x 4 MMAs run; the column indices of the warp's next chunk are
// fetched one chunk ahead.  Latency is hidden across warps (no register double buffer:
// measured slower, 628 vs 554 us over the DLMC batch, because of the occupancy it costs).
// (The previous design -- contiguous 16-vector slices straddling windows, one 64-wide chunk
// in flight -- paid a round trip per chunk on the A row and per window of a straddling
// slice: 7 us for a 98%-sparse 512 x 512 mask at K = 256; this one takes 3.3 us.)
template <int V, bool VEC, int KC, bool ARES, int FAST = 0>
__device__ __forceinline__ void sddmm_window(int64_t M, int64_t K,
                                             const int32_t* __restrict__ row_ptr,
                                             const int32_t* __restrict__ col_idx,
                                             const uint16_t* __restrict__ A,
                                             const uint16_t* __restrict__ Bt,
                                             uint16_t* __restrict__ out, bool out4, int64_t w,
                                             int64_t j0, int64_t q) {
  (void)ARES;
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int64_t kt = 8 * t;
  const int64_t pb = row_ptr[w], pe = row_ptr[w + 1];
  int64_t v0 = pb + 16 * j0;
  if (v0 >= pe) return;
  const int64_t arow = w * V + g;
  const bool ok_row = (g < V) && (arow < M);
  const uint16_t* rowA = A + (FAST != 0 && !ok_row ? 0 : arow) * K;
  const bool one_block = K <= 64 * KC;
  int ca = (v0 + g < pe) ? ldg32i(col_idx + v0 + g) : 0;
  int cb = (v0 + g + 8 < pe) ? ldg32i(col_idx + v0 + g + 8) : 0;
  uint4 xx0[KC], xx1[KC];  // A rows of the window, K block
  if (one_block) {
#pragma unroll
    for (int c = 0; c < KC; ++c) {
      if (FAST != 0) load_seg2_fast(rowA, 64 * c + kt, xx0[c], xx1[c]);
      else load_seg2<VEC>(rowA, K, 64 * c + kt, ok_row, xx0[c], xx1[c]);
    }
  }
  for (; v0 < pe; v0 += 16 * q) {
    const bool oka = v0 + g < pe, okb = v0 + g + 8 < pe;
    const int64_t nv0 = v0 + 16 * q;
    const int nca = (nv0 + g < pe) ? ldg32i(col_idx + nv0 + g) : 0;
    const int ncb = (nv0 + g + 8 < pe) ? ldg32i(col_idx + nv0 + g + 8) : 0;
    const uint16_t* rowa = Bt + (int64_t)ca * K;
    const uint16_t* rowb = Bt + (int64_t)cb * K;
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
    for (int64_t kb = 0; kb < K; kb += 64 * KC) {
      uint4 xa0[KC], xa1[KC], xb0[KC], xb1[KC];
#pragma unroll
      for (int c = 0; c < KC; ++c) {
        const int64_t k = kb + 64 * c + kt;
        // FAST 1: every chunk unpredicated (slots past the window end read row 0); FAST 2: only
        // full chunks (warp-uniform test), the tail chunk keeps the guarded loads
        if (FAST == 1 || (FAST == 2 && v0 + 16 <= pe)) {
          load_seg2_fast(rowa, k, xa0[c], xa1[c]);
          load_seg2_fast(rowb, k, xb0[c], xb1[c]);
          if (!one_block) load_seg2_fast(rowA, k, xx0[c], xx1[c]);
        } else {
          load_seg2<VEC>(rowa, K, k, oka, xa0[c], xa1[c]);
          load_seg2<VEC>(rowb, K, k, okb, xb0[c], xb1[c]);
          if (!one_block) load_seg2<VEC>(rowA, K, k, ok_row, xx0[c], xx1[c]);
        }
      }
#pragma unroll
      for (int c = 0; c < KC; ++c)
#pragma unroll
        for (int j = 0; j < 4; ++j)
          mma_16816(acc, wordj(xa0[c], j), wordj(xb0[c], j), wordj(xa1[c], j), wordj(xb1[c], j),
                    wordj(xx0[c], j), wordj(xx1[c], j));
    }
    store_chunk<V>(acc, v0, pe, w, M, g, t, out, out4);
    ca = nca;
    cb = ncb;
  }
}

// K <= 64 body with TWO of the warp's chunks in flight per round trip (v0 and v0 + 16q):
// 8 LDG.128 per thread before the first MMA instead of 4, so a warp keeps twice the gather
// bytes in flight at the same occupancy (register cost = the KC = 2 body's).  Each chunk's
// accumulation order is the KC = 1 body's, so the bits are identical.
template <int V, int FAST = 0>
__device__ __forceinline__ void sddmm_window_pair(int64_t M, int64_t K,
                                                  const int32_t* __restrict__ row_ptr,
                                                  const int32_t* __restrict__ col_idx,
                                                  const uint16_t* __restrict__ A,
                                                  const uint16_t* __restrict__ Bt,
                                                  uint16_t* __restrict__ out, bool out4, int64_t w,
                                                  int64_t j0, int64_t q) {
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int64_t kt = 8 * t;
  const int64_t pb = row_ptr[w], pe = row_ptr[w + 1];
  int64_t v0 = pb + 16 * j0;
  if (v0 >= pe) return;
  const int64_t arow = w * V + g;
  const bool ok_row = (g < V) && (arow < M);
  const int64_t sq = 16 * q;
  auto col = [&](int64_t v) { return (v < pe) ? ldg32i(col_idx + v) : 0; };
  int c0a = col(v0 + g), c0b = col(v0 + g + 8), c1a = col(v0 + sq + g), c1b = col(v0 + sq + g + 8);
  // K == 64: see load_seg2_fast (absent slots read row 0, never stored); FAST 2 only for pairs
  // of full chunks
  uint4 xx0, xx1;
  if (FAST != 0) load_seg2_fast(A + (ok_row ? arow : 0) * K, kt, xx0, xx1);
  else load_seg2<true>(A + arow * K, K, kt, ok_row, xx0, xx1);
  for (; v0 < pe; v0 += 2 * sq) {
    const int64_t v1 = v0 + sq, n0 = v0 + 2 * sq, n1 = n0 + sq;
    const int n0a = col(n0 + g), n0b = col(n0 + g + 8), n1a = col(n1 + g), n1b = col(n1 + g + 8);
    uint4 a0[2], a1[2], b0[2], b1[2];
    if (FAST == 1 || (FAST == 2 && v1 + 16 <= pe)) {
      load_seg2_fast(Bt + (int64_t)c0a * K, kt, a0[0], a1[0]);
      load_seg2_fast(Bt + (int64_t)c0b * K, kt, b0[0], b1[0]);
      load_seg2_fast(Bt + (int64_t)c1a * K, kt, a0[1], a1[1]);
      load_seg2_fast(Bt + (int64_t)c1b * K, kt, b0[1], b1[1]);
    } else {
      load_seg2<true>(Bt + (int64_t)c0a * K, K, kt, v0 + g < pe, a0[0], a1[0]);
      load_seg2<true>(Bt + (int64_t)c0b * K, K, kt, v0 + g + 8 < pe, b0[0], b1[0]);
      load_seg2<true>(Bt + (int64_t)c1a * K, K, kt, v1 + g < pe, a0[1], a1[1]);
      load_seg2<true>(Bt + (int64_t)c1b * K, K, kt, v1 + g + 8 < pe, b0[1], b1[1]);
    }
    float acc0[4] = {0.f, 0.f, 0.f, 0.f}, acc1[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int j = 0; j < 4; ++j)
      mma_16816(acc0, wordj(a0[0], j), wordj(b0[0], j), wordj(a1[0], j), wordj(b1[0], j),
                wordj(xx0, j), wordj(xx1, j));
#pragma unroll
    for (int j = 0; j < 4; ++j)
      mma_16816(acc1, wordj(a0[1], j), wordj(b0[1], j), wordj(a1[1], j), wordj(b1[1], j),
                wordj(xx0, j), wordj(xx1, j));
    store_chunk<V>(acc0, v0, pe, w, M, g, t, out, out4);
    if (v1 < pe) store_chunk<V>(acc1, v1, pe, w, M, g, t, out, out4);
    c0a = n0a; c0b = n0b; c1a = n1a; c1b = n1b;
  }
}

// ARES slot = "mixed K blocks": one kernel serves both K <= 64 (KC = 1 body) and K > 64
// (KC = 2 body), chosen per problem at run time, so a batch needs one launch per V instead of
// one per (V, KC) group (no tail between the two launches).  Same bodies, same bits.
template <int V, bool VEC, int KC, bool ARES, int FAST = 0>
__device__ __forceinline__ void sddmm_window_any(int64_t M, int64_t K,
                                                 const int32_t* __restrict__ row_ptr,
                                                 const int32_t* __restrict__ col_idx,
                                                 const uint16_t* __restrict__ A,
                                                 const uint16_t* __restrict__ Bt,
                                                 uint16_t* __restrict__ out, bool out4, int64_t w,
                                                 int64_t j0, int64_t q, bool pair) {
  if constexpr (ARES && VEC && FAST != 0) {
    // only K == 64 or K % 128 == 0 problems reach this instantiation (sddmm_fast_ok)
    (void)pair;
    if (K <= 64)
      sddmm_window_pair<V, FAST>(M, K, row_ptr, col_idx, A, Bt, out, out4, w, j0, q);
    else
      sddmm_window<V, VEC, 2, false, FAST>(M, K, row_ptr, col_idx, A, Bt, out, out4, w, j0, q);
  } else if constexpr (ARES && VEC) {
    if (K <= 64 && pair)
      sddmm_window_pair<V>(M, K, row_ptr, col_idx, A, Bt, out, out4, w, j0, q);
    else if (K <= 64)
      sddmm_window<V, VEC, 1, false>(M, K, row_ptr, col_idx, A, Bt, out, out4, w, j0, q);
    else
      sddmm_window<V, VEC, 2, false>(M, K, row_ptr, col_idx, A, Bt, out, out4, w, j0, q);
  } else {
    sddmm_window<V, VEC, KC, ARES>(M, K, row_ptr, col_idx, A, Bt, out, out4, w, j0, q);
  }
}

// Row blocks the dense-tile kernel takes (dense_select.cuh) are skipped here, except windows
// whose col_idx is not strictly ascending: the dense kernel finds a window's vectors of each
// column tile by a search that assumes ascending order, so such a window (rare: the encoder
// emits ascending windows) is computed here in full by the warp of its first item, after the
// dense kernel has completed (this kernel follows it on the stream; when the two overlap by
// programmatic dependent launch the warp waits for it with griddepcontrol.wait), overwriting its
// writes.
// Returns the q to use for the item, 0 to skip it, or -1 for such a window.
__device__ __forceinline__ int64_t sddmm_gather_q(bool dense_ok, int64_t N, int V, int64_t W,
                                                  const int32_t* __restrict__ row_ptr,
                                                  const int32_t* __restrict__ col_idx, int64_t w,
                                                  int64_t j0, int64_t q) {
  if (!dense_ok) return q;
  const int64_t rb = (w * V) / kDenseRows;
  if (!sddmm_rb_dense(row_ptr, W, V, rb, N)) return q;
  if (j0 != 0) return 0;
  return window_sorted(col_idx, __ldg(row_ptr + w), __ldg(row_ptr + w + 1)) ? 0 : -1;
}

// Work items of one problem: W windows x q warps per window (warp j of window w takes the
// window's 16-vector chunks j, j + q, ...); q = the number of warps per window that gives
// every warp of the launch about the same number of chunks.
__device__ __forceinline__ int64_t sddmm_q(int64_t chunks, int64_t W, int64_t per_warp) {
  const int64_t q = ceil_div64(chunks, W * per_warp);
  return q < 1 ? 1 : (q > 64 ? 64 : q);
}

template <int V, bool VEC, int KC, bool ARES, bool FAST = false>
__global__ void __launch_bounds__(kSddmmWarps * 32, VS_SDDMM_MINB)
    sddmm_kernel(int64_t M, int64_t K, int64_t W, const int32_t* __restrict__ row_ptr,
                 const int32_t* __restrict__ col_idx, const uint16_t* __restrict__ A,
                 const uint16_t* __restrict__ Bt, uint16_t* __restrict__ out, bool out4,
                 bool pair, int64_t N, bool dense_ok) {
  const int64_t nnz = row_ptr[W];
  const int64_t n_warps = (int64_t)gridDim.x * kSddmmWarps;
  const int64_t gw = (int64_t)blockIdx.x * kSddmmWarps + (threadIdx.x >> 5);
  const int64_t chunks = ceil_div64(nnz, 16) + W;  // upper bound of sum_w ceil(nnz_w / 16)
  const int64_t q = sddmm_q(chunks, W, ceil_div64(chunks, n_warps));
  const int64_t items = W * q;
  for (int64_t it = gw; it < items; it += n_warps) {
    const int64_t w = it / q;
    int64_t qq = sddmm_gather_q(dense_ok, N, V, W, row_ptr, col_idx, w, it - w * q, q);
    if (qq == 0) continue;
    if (qq < 0) {  // non-ascending window of a dense row block: after the dense kernel, in full
      pdl_wait_prior();
      qq = 1;
    }
    // single-problem kernel: FAST mode 1 (measured best per call, profiles/r02_sddmm_variants.md)
    sddmm_window_any<V, VEC, KC, ARES, FAST ? 1 : 0>(M, K, row_ptr, col_idx, A, Bt, out, out4, w,
                                                     qq == q ? it - w * q : 0, qq, pair);
  }
  pdl_wait_prior();  // completes only after a dense-tile kernel it overlaps (no-op otherwise)
}

// Batched launch over up to kSddmmMaxBatch problems of one configuration: every problem
// gets W_p x q_p work items (q_p from its nnz, read on the device, so every warp gets about
// the same number of chunks); the items of all problems are dealt round-robin to the
// persistent warps in problem order, so at any time the warps work on one or two problems
// (L2 locality).
struct SddmmDesc {
  int64_t M, K, W, N;
  int64_t dense_ok;  // sddmm_dense_eligible: row blocks may be taken by the dense-tile kernel
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const uint16_t* A;
  const uint16_t* Bt;
  uint16_t* out;
  int64_t out4;
};
constexpr int kSddmmMaxBatch = 128;
struct SddmmBatch {
  int count;
  int pair;  // K <= 64 problems take two chunks per round trip (sddmm_window_pair)
  SddmmDesc d[kSddmmMaxBatch];
};

template <int V, bool VEC, int KC, bool ARES, bool FAST = false>
__global__ void __launch_bounds__(kSddmmWarps * 32, VS_SDDMM_MINB)
    sddmm_batched_kernel(const __grid_constant__ SddmmBatch b) {
  __shared__ int64_t pre[kSddmmMaxBatch + 1];  // prefix of work items
  __shared__ int64_t qs[kSddmmMaxBatch];
  const int lane = lane_id();
  const int64_t n_warps = (int64_t)gridDim.x * kSddmmWarps;
  if (threadIdx.x < 32) {
    // pass 1: total chunks -> chunks per warp
    int64_t tot = 0;
    for (int base = 0; base < b.count; base += 32) {
      const int p = base + lane;
      int64_t ch = 0;
      if (p < b.count) ch = ceil_div64((int64_t)b.d[p].row_ptr[b.d[p].W], 16) + b.d[p].W;
#pragma unroll
      for (int o = 16; o >= 1; o >>= 1) ch += __shfl_xor_sync(0xffffffffu, ch, o);
      tot += ch;
    }
    const int64_t per_warp = ceil_div64(tot, n_warps) > 0 ? ceil_div64(tot, n_warps) : 1;
    // pass 2: items per problem, exclusive prefix
    int64_t carry = 0;
    for (int base = 0; base < b.count; base += 32) {
      const int p = base + lane;
      int64_t items = 0, q = 1;
      if (p < b.count) {
        const int64_t W = b.d[p].W;
        const int64_t ch = ceil_div64((int64_t)b.d[p].row_ptr[W], 16) + W;
        q = sddmm_q(ch, W, per_warp);
        items = W * q;
      }
      int64_t incl = items;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t x = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += x;
      }
      if (p < b.count) {
        pre[p] = carry + incl - items;
        qs[p] = q;
      }
      carry += __shfl_sync(0xffffffffu, incl, 31);
    }
    if (lane == 0) pre[b.count] = carry;
  }
  __syncthreads();
  const int64_t n_items = pre[b.count];
  const int64_t gw = (int64_t)blockIdx.x * kSddmmWarps + (threadIdx.x >> 5);
  int p = 0;
  for (int64_t it = gw; it < n_items; it += n_warps) {
    while (pre[p + 1] <= it) ++p;
    const SddmmDesc& d = b.d[p];
    const int64_t q = qs[p];
    const int64_t loc = it - pre[p];
    const int64_t w = loc / q;
    int64_t qq = sddmm_gather_q(d.dense_ok != 0, d.N, V, d.W, d.row_ptr, d.col_idx, w, loc - w * q, q);
    if (qq == 0) continue;
    if (qq < 0) {  // non-ascending window of a dense row block: after the dense kernel, in full
      pdl_wait_prior();
      qq = 1;
    }
    // batched kernel: FAST mode 2 (full chunks only: many short windows in a batch)
    sddmm_window_any<V, VEC, KC, ARES, FAST ? 2 : 0>(d.M, d.K, d.row_ptr, d.col_idx, d.A, d.Bt, d.out,
                                                     d.out4 != 0, w, qq == q ? loc - w * q : 0, qq,
                                                     b.pair != 0);
  }
  pdl_wait_prior();  // completes only after a dense-tile kernel it overlaps (no-op otherwise)
}

// Persistent grid: as many CTAs as can be resident at once (occupancy queried once per
// kernel instantiation), so every warp's contiguous share of slices runs concurrently.
template <typename Kern>
static int ctas_per_sm(Kern k) {
  int b = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k, kSddmmWarps * 32, 0) != cudaSuccess || b < 1)
    b = 1;
  return b;
}

// Kernel variant of a problem: K block 64 * KC (KC = 2 for K > 64: measured faster than
// KC = 4 over the DLMC set, tools/tune.py; VS_SDDMM_KC caps it) and whether the A row of a
// window stays in registers -- the ARES slot now selects the mixed-K kernel (sddmm_window_any).  Encoded as
// KC * 2 + ARES.
// Build-time constants (no run-time knobs in the shipped library; tools/tune.py builds
// variants with -D): VS_SDDMM_KC caps the K block, VS_SDDMM_MIX = one mixed-K kernel per V,
// VS_SDDMM_PAIR = two chunks in flight for K <= 64.
#ifndef VS_SDDMM_KC
#define VS_SDDMM_KC 2
#endif
#ifndef VS_SDDMM_MIX
#define VS_SDDMM_MIX 1
#endif
#ifndef VS_SDDMM_PAIR
#define VS_SDDMM_PAIR 1
#endif
static int sddmm_variant(int64_t K, bool vec) {
  constexpr int cap = VS_SDDMM_KC >= 2 ? 2 : 1;
  int kc = (!vec || K <= 64) ? 1 : 2;
  if (kc > cap) kc = cap;
  // vector-path problems of any K share the mixed kernel; K == 64 and K % 128 == 0 take its
  // unpredicated-load instantiation (code 6)
  if (vec && VS_SDDMM_MIX && cap == 2) return (VS_SDDMM_FAST && K > 0 && (K == 64 || K % 128 == 0)) ? 6 : 2 * 2 + 1;
  return kc * 2;
}

// K <= 64 problems of the mixed-K kernel keep two chunks in flight per warp
// (sddmm_window_pair); VS_SDDMM_PAIR=0 selects the one-chunk body.  Same bits either way.
static constexpr bool sddmm_pair_on() { return VS_SDDMM_PAIR != 0; }

template <int V, bool VEC, int KC, bool ARES, bool FAST = false>
static int sddmm_ctas_per_sm() {
  static const int n = ctas_per_sm(sddmm_kernel<V, VEC, KC, ARES, FAST>);
  return n;
}
template <int V, bool VEC, int KC, bool ARES, bool FAST = false>
static int sddmm_batched_ctas_per_sm() {
  static const int n = ctas_per_sm(sddmm_batched_kernel<V, VEC, KC, ARES, FAST>);
  return n;
}

// Launch after the dense-tile kernel just launched on the stream: overlapped with it by
// programmatic dependent launch (pdl: the gather kernel's blocks start while it runs and
// complete after it, see sddmm_gather_q), or plainly (stream order).
// VS_SDDMM_PDL (build time, default 1): the gather kernel follows a dense-tile launch of at most
// kSddmmPdlMaxUnits units (CTAs) with programmatic dependent launch.  Measured (profiles/
// r03_dense_sddmm.md): single calls ~5 % faster and the ResNet-50 layer step 0.954 -> ~0.90 ms,
// but back-to-back C5 steps (a 65536-CTA dense grid ahead of the persistent gather grid)
// 110 -> 171 ms, so launches with larger dense grids follow plainly (stream order).
#ifndef VS_SDDMM_PDL
#define VS_SDDMM_PDL 1
#endif
constexpr int64_t kSddmmPdlMaxUnits = 4096;  // DLMC V groups 1088, ResNet-50 layers 1532; C5 >= 8192 per rank
static int64_t sddmm_dense_units(int64_t M, int64_t N) { return ceil_div64(M, 128) * ceil_div64(N, 128); }
template <typename... KArgs, typename... Args>
static void launch_maybe_pdl(bool pdl, void (*kern)(KArgs...), dim3 grid, dim3 block, cudaStream_t s,
                             Args... args) {
  if (!pdl || !VS_SDDMM_PDL) {
    kern<<<grid, block, 0, s>>>(args...);
    return;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  (void)cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

template <int V, bool VEC, int KC, bool ARES, bool FAST = false>
static void launch_sddmm_one(int64_t M, int64_t K, const int32_t* row_ptr, const int32_t* col_idx,
                             const uint16_t* A, const uint16_t* Bt, uint16_t* out, int num_sms,
                             cudaStream_t s, int64_t N, bool dense_ok, bool pdl) {
  const int64_t W = ceil_div64(M, V);
  const bool out4 = (reinterpret_cast<uintptr_t>(out) & 3) == 0;
  dim3 grid((unsigned)(num_sms * sddmm_ctas_per_sm<V, VEC, KC, ARES, FAST>()));
  launch_maybe_pdl(pdl, sddmm_kernel<V, VEC, KC, ARES, FAST>, grid, dim3(kSddmmWarps * 32), s, M, K, W,
                   row_ptr, col_idx, A, Bt, out, out4, sddmm_pair_on(), N, dense_ok);
}

#if VS_SDDMM_DENSE_CF > 0
bool sddmm_dense_eligible(int64_t M, int64_t N, int64_t K, int V, const void* A, const void* Bt);
cudaError_t launch_sddmm_dense(int64_t count, const int64_t* M, const int64_t* N, const int64_t* K,
                               const int* V, const int32_t* const* row_ptr, const int32_t* const* col_idx,
                               const void* const* A, const void* const* Bt, void* const* out, int num_sms,
                               cudaStream_t s);
#else  // shipped library: no dense-tile path (dense_select.cuh)
static bool sddmm_dense_eligible(int64_t, int64_t, int64_t, int, const void*, const void*) { return false; }
static cudaError_t launch_sddmm_dense(int64_t, const int64_t*, const int64_t*, const int64_t*, const int*,
                                      const int32_t* const*, const int32_t* const*, const void* const*,
                                      const void* const*, void* const*, int, cudaStream_t) {
  return cudaSuccess;
}
#endif

template <int V>
static cudaError_t launch_sddmm_v(int64_t M, int64_t N, int64_t K, const int32_t* row_ptr,
                                  const int32_t* col_idx, const uint16_t* A, const uint16_t* Bt,
                                  uint16_t* out, bool vec, int num_sms, cudaStream_t s) {
  const int V_ = V;
  const bool dok = sddmm_dense_eligible(M, N, K, V, A, Bt);
  const bool pdl = dok && sddmm_dense_units(M, N) <= kSddmmPdlMaxUnits;
  if (dok) {
    // dense row blocks first (short non-persistent CTAs); the persistent gather grid then
    // takes the remaining row blocks
    const void* a = A;
    const void* bt = Bt;
    void* o = out;
    const cudaError_t de = launch_sddmm_dense(1, &M, &N, &K, &V_, &row_ptr, &col_idx, &a, &bt, &o, num_sms, s);
    if (de != cudaSuccess) return de;
  }
  switch ((vec ? 8 : 0) + sddmm_variant(K, vec)) {
    case 8 + 2: launch_sddmm_one<V, true, 1, false>(M, K, row_ptr, col_idx, A, Bt, out, num_sms, s, N, dok, pdl); break;
    case 8 + 3: launch_sddmm_one<V, true, 1, true>(M, K, row_ptr, col_idx, A, Bt, out, num_sms, s, N, dok, pdl); break;
    case 8 + 4: launch_sddmm_one<V, true, 2, false>(M, K, row_ptr, col_idx, A, Bt, out, num_sms, s, N, dok, pdl); break;
    case 8 + 5: launch_sddmm_one<V, true, 2, true>(M, K, row_ptr, col_idx, A, Bt, out, num_sms, s, N, dok, pdl); break;
    case 8 + 6: launch_sddmm_one<V, true, 2, true, true>(M, K, row_ptr, col_idx, A, Bt, out, num_sms, s, N, dok, pdl); break;
    case 3: launch_sddmm_one<V, false, 1, true>(M, K, row_ptr, col_idx, A, Bt, out, num_sms, s, N, dok, pdl); break;
    default: launch_sddmm_one<V, false, 1, false>(M, K, row_ptr, col_idx, A, Bt, out, num_sms, s, N, dok, pdl); break;
  }
  return cudaGetLastError();
}

template <int V, bool VEC, int KC, bool ARES, bool FAST = false>
static void launch_sddmm_batch(const SddmmBatch& b, int num_sms, cudaStream_t s, bool pdl) {
  // VS_SDDMM_OVERSUB (build time): grid = that many times the resident CTAs.  2 is 5% faster
  // for the SDDMM batch alone but 2% slower for the bench step, where the oversubscribed grid
  // competes with the concurrent SpMM / encode branches; default 1.
#ifndef VS_SDDMM_OVERSUB
#define VS_SDDMM_OVERSUB 1
#endif
  constexpr int over = VS_SDDMM_OVERSUB < 1 ? 1 : VS_SDDMM_OVERSUB;
  dim3 grid((unsigned)(num_sms * sddmm_batched_ctas_per_sm<V, VEC, KC, ARES, FAST>() * over));
  launch_maybe_pdl(pdl, sddmm_batched_kernel<V, VEC, KC, ARES, FAST>, grid, dim3(kSddmmWarps * 32), s, b);
}

template <int V>
static void launch_sddmm_batch_v(const SddmmBatch& b, int code, int num_sms, cudaStream_t s, bool pdl) {
  switch (code) {
    case 8 + 2: return launch_sddmm_batch<V, true, 1, false>(b, num_sms, s, pdl);
    case 8 + 3: return launch_sddmm_batch<V, true, 1, true>(b, num_sms, s, pdl);
    case 8 + 4: return launch_sddmm_batch<V, true, 2, false>(b, num_sms, s, pdl);
    case 8 + 5: return launch_sddmm_batch<V, true, 2, true>(b, num_sms, s, pdl);
    case 8 + 6: return launch_sddmm_batch<V, true, 2, true, true>(b, num_sms, s, pdl);
    case 3: return launch_sddmm_batch<V, false, 1, true>(b, num_sms, s, pdl);
    default: return launch_sddmm_batch<V, false, 1, false>(b, num_sms, s, pdl);
  }
}

// tcgen05 path (sddmm_tc.cu), compiled only into a library built with -DVS_WITH_SDDMM_TC=1:
// such a build sends problems with K % 8 == 0, K > 0 and 16-byte aligned A, Bt and out_vals
// to the tensor-core kernel, single and batched calls alike.  Not in the shipped library:
// measured 1.8-2.5x slower than the mma.sync kernels below over the DLMC set (DESIGN.md 7.4,
// profiles/r01b_tcgen05.md) -- the cp.async shared-memory staging that tcgen05 operands need
// caps the row gather at ~60 B/clk/SM, below the register path.
#ifndef VS_WITH_SDDMM_TC
#define VS_WITH_SDDMM_TC 0
#endif
static constexpr bool sddmm_tc_on() { return VS_WITH_SDDMM_TC != 0; }
#if VS_WITH_SDDMM_TC
bool sddmm_tc_eligible(int64_t K, const void* A, const void* Bt, const void* out);
cudaError_t launch_sddmm_tc_batched(int64_t count, const int64_t* M, const int64_t* N, const int64_t* K, const int* V,
                                    const int32_t* const* row_ptr, const int32_t* const* col_idx,
                                    const void* const* A, const void* const* Bt, void* const* out,
                                    int num_sms, cudaStream_t s);
#else
static bool sddmm_tc_eligible(int64_t, const void*, const void*, const void*) { return false; }
static cudaError_t launch_sddmm_tc_batched(int64_t, const int64_t*, const int64_t*, const int64_t*,
                                           const int*, const int32_t* const*, const int32_t* const*,
                                           const void* const*, const void* const*, void* const*,
                                           int, cudaStream_t) {
  return cudaErrorNotSupported;
}
#endif

static cudaError_t launch_sddmm_mma_batched(int64_t count, const int64_t* M, const int64_t* N,
                                            const int64_t* K, const int* V,
                                            const int32_t* const* row_ptr,
                                            const int32_t* const* col_idx, const void* const* A,
                                            const void* const* Bt, void* const* out, int num_sms,
                                            cudaStream_t s, bool pdl_first = false);

cudaError_t launch_sddmm_batched(int64_t count, const int64_t* M, const int64_t* N, const int64_t* K,
                                 const int* V, const int32_t* const* row_ptr,
                                 const int32_t* const* col_idx, const void* const* A,
                                 const void* const* Bt, void* const* out, int num_sms,
                                 cudaStream_t s) {
  if (!sddmm_tc_on()) {
    // the dense-tile kernel (taking the dense row blocks), then the gather kernels (skipping them)
    bool dense = false;
    int64_t units = 0;
    for (int64_t i = 0; i < count && VS_SDDMM_DENSE_CF != 0; ++i)
      if (sddmm_dense_eligible(M[i], N[i], K[i], V[i], A[i], Bt[i])) {
        dense = true;
        units += sddmm_dense_units(M[i], N[i]);
      }
    if (dense) {
      const cudaError_t e = launch_sddmm_dense(count, M, N, K, V, row_ptr, col_idx, A, Bt, out, num_sms, s);
      if (e != cudaSuccess) return e;
    }
    return launch_sddmm_mma_batched(count, M, N, K, V, row_ptr, col_idx, A, Bt, out, num_sms, s,
                                    dense && units <= kSddmmPdlMaxUnits);
  }
  std::vector<int64_t> sel[2];
  for (int64_t i = 0; i < count; ++i) sel[sddmm_tc_eligible(K[i], A[i], Bt[i], out[i]) ? 1 : 0].push_back(i);
  for (int path = 0; path < 2; ++path) {
    if (sel[path].empty()) continue;
    std::vector<int64_t> m, n, k;
    std::vector<int> v;
    std::vector<const int32_t*> rp, ci;
    std::vector<const void*> a, bt;
    std::vector<void*> o;
    for (int64_t i : sel[path]) {
      m.push_back(M[i]); n.push_back(N[i]); k.push_back(K[i]); v.push_back(V[i]); rp.push_back(row_ptr[i]);
      ci.push_back(col_idx[i]); a.push_back(A[i]); bt.push_back(Bt[i]); o.push_back(out[i]);
    }
    const cudaError_t e =
        path ? launch_sddmm_tc_batched((int64_t)m.size(), m.data(), n.data(), k.data(), v.data(),
                                       rp.data(), ci.data(), a.data(), bt.data(), o.data(), num_sms, s)
             : launch_sddmm_mma_batched((int64_t)m.size(), m.data(), n.data(), k.data(), v.data(), rp.data(),
                                        ci.data(), a.data(), bt.data(), o.data(), num_sms, s);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

static cudaError_t launch_sddmm_mma_batched(int64_t count, const int64_t* M, const int64_t* N,
                                            const int64_t* K, const int* V,
                                            const int32_t* const* row_ptr,
                                            const int32_t* const* col_idx, const void* const* A,
                                            const void* const* Bt, void* const* out, int num_sms,
                                            cudaStream_t s, bool pdl_first) {
  // group by (V, vector path); keep the caller's order inside a group
  std::vector<std::pair<int, int64_t>> order;
  for (int64_t i = 0; i < count; ++i) {
    const bool vec = (K[i] % 8 == 0) && ((reinterpret_cast<uintptr_t>(A[i]) & 15) == 0) &&
                     ((reinterpret_cast<uintptr_t>(Bt[i]) & 15) == 0);
    // key: V, vector path, kernel variant
    order.push_back({V[i] * 16 + (vec ? 8 : 0) + sddmm_variant(K[i], vec), i});
  }
  std::stable_sort(order.begin(), order.end(),
                   [](const auto& a, const auto& b) { return a.first < b.first; });
  SddmmBatch batch;
  batch.pair = sddmm_pair_on() ? 1 : 0;
  size_t i = 0;
  while (i < order.size()) {
    const int key = order[i].first;
    batch.count = 0;
    while (i < order.size() && order[i].first == key && batch.count < kSddmmMaxBatch) {
      const int64_t p = order[i].second;
      SddmmDesc& d = batch.d[batch.count++];
      d = {M[p], K[p], ceil_div64(M[p], V[p]), N[p],
           sddmm_dense_eligible(M[p], N[p], K[p], V[p], A[p], Bt[p]) ? 1 : 0, row_ptr[p], col_idx[p],
           static_cast<const uint16_t*>(A[p]), static_cast<const uint16_t*>(Bt[p]),
           static_cast<uint16_t*>(out[p]), (reinterpret_cast<uintptr_t>(out[p]) & 3) == 0 ? 1 : 0};
      ++i;
    }
    const int code = key & 15;
    switch (key >> 4) {
      case 1: launch_sddmm_batch_v<1>(batch, code, num_sms, s, pdl_first); break;
      case 2: launch_sddmm_batch_v<2>(batch, code, num_sms, s, pdl_first); break;
      case 4: launch_sddmm_batch_v<4>(batch, code, num_sms, s, pdl_first); break;
      default: launch_sddmm_batch_v<8>(batch, code, num_sms, s, pdl_first); break;
    }
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    pdl_first = false;  // later launches follow the gather launch before them plainly
  }
  return cudaSuccess;
}

cudaError_t launch_sddmm(int64_t M, int64_t N, int64_t K, int V, const int32_t* row_ptr,
                         const int32_t* col_idx, const void* A, const void* Bt, void* out,
                         int num_sms, cudaStream_t s) {
  if (sddmm_tc_on() && sddmm_tc_eligible(K, A, Bt, out))
    return launch_sddmm_tc_batched(1, &M, &N, &K, &V, &row_ptr, &col_idx, &A, &Bt, &out, num_sms, s);
  const uint16_t* a = static_cast<const uint16_t*>(A);
  const uint16_t* b = static_cast<const uint16_t*>(Bt);
  uint16_t* o = static_cast<uint16_t*>(out);
  const bool vec = (K % 8 == 0) && ((reinterpret_cast<uintptr_t>(A) & 15) == 0) &&
                   ((reinterpret_cast<uintptr_t>(Bt) & 15) == 0);
  switch (V) {
    case 1: return launch_sddmm_v<1>(M, N, K, row_ptr, col_idx, a, b, o, vec, num_sms, s);
    case 2: return launch_sddmm_v<2>(M, N, K, row_ptr, col_idx, a, b, o, vec, num_sms, s);
    case 4: return launch_sddmm_v<4>(M, N, K, row_ptr, col_idx, a, b, o, vec, num_sms, s);
    case 8: return launch_sddmm_v<8>(M, N, K, row_ptr, col_idx, a, b, o, vec, num_sms, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace vs
