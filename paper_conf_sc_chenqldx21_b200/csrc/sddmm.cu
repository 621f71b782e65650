// sddmm.cu — out = (A * B) sampled at a column-vector mask (§6).
//
//   out_vals[p*V + r] = sum_k A[wV+r][k] * Bt[col_idx[p]][k]   (p in window w)
//
// Work decomposition (B200 re-design; the paper launches ceil(M/V) x ceil(N/32) CTAs over
// the DENSE N, many of them idle): a persistent grid of warps splits the
// stored vectors 0..nnz_v-1 (nnz_v = row_ptr[W], read on the device, so no host sync) into
// 16-vector slices; every warp owns a contiguous run of slices, finds the window of its
// first vector once by a warp-cooperative search of row_ptr and then walks forward.  A
// slice that straddles windows is finished window by window (rows of other windows are
// computed and dropped).
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

namespace vs {

constexpr int kSddmmWarps = 4;

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

__device__ __forceinline__ uint32_t wordj(const uint4& v, int j) {
  return j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w));
}

// Largest w in [0, W) with row_ptr[w] <= v (the window owning vector v; empty windows
// before it are skipped).  Warp-cooperative 32-ary search; all lanes get the result.
__device__ __forceinline__ int64_t find_window(const int32_t* __restrict__ row_ptr, int64_t W,
                                               int64_t v) {
  int64_t lo = 0, hi = W;  // answer in [lo, hi)
  const int lane = lane_id();
  while (hi - lo > 1) {
    const int64_t span = hi - lo;
    const int64_t step = (span + 31) / 32;
    const int64_t probe = lo + (int64_t)lane * step;
    const bool le = (probe < hi) && (row_ptr[probe] <= v);
    const unsigned ballot = __ballot_sync(0xffffffffu, le);
    // lanes 0..(n-1) satisfy le (row_ptr non-decreasing); lane 0 always (row_ptr[lo] <= v)
    const int last = 31 - __clz(ballot);
    const int64_t nlo = lo + (int64_t)last * step;
    const int64_t nhi = (last == 31) ? hi : (lo + (int64_t)(last + 1) * step);
    lo = nlo;
    hi = nhi < hi ? nhi : hi;
  }
  return lo;
}

// Stores the two vectors (M rows g, g+8) of a 16-vector slice held in acc, restricted to the
// vectors [lo, hi) of window w.
template <int V>
__device__ __forceinline__ void store_slice(const float (&acc)[4], int64_t v0, int64_t lo,
                                            int64_t hi, int64_t w, int64_t M, int g, int t,
                                            uint16_t* __restrict__ out, bool out4) {
#pragma unroll
  for (int q = 0; q < 2; ++q) {
    const int64_t v = v0 + g + 8 * q;
    if (v < lo || v >= hi) continue;
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

// One warp computes the 16-vector slices [s_begin, s_end) of one problem (nnz stored
// vectors in total); s_begin < s_end.  The work is one stream of 64-wide K chunks (slice by
// slice; a slice that straddles windows is finished window by window, re-reading its rows),
// software-pipelined one chunk ahead: while the MMAs of a chunk run, the gathered Bt rows of
// the next chunk -- possibly the first chunk of the next segment or slice -- are in flight,
// and the column indices of the next slice are fetched one slice ahead.  The first loads are
// issued before the window search, which does not affect them.  (Processing 2 or 4 slices of
// one window together to share the A fragment measured no faster, tools/tune.py.)
template <int V, bool VEC>
__device__ __forceinline__ void sddmm_range(int64_t M, int64_t K, int64_t W,
                                            const int32_t* __restrict__ row_ptr,
                                            const int32_t* __restrict__ col_idx,
                                            const uint16_t* __restrict__ A,
                                            const uint16_t* __restrict__ Bt,
                                            uint16_t* __restrict__ out, bool out4, int64_t s_begin,
                                            int64_t s_end, int64_t nnz) {
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int64_t kt = 8 * t;
  int64_t v0 = s_begin * 16;
  int64_t v_hi = (v0 + 16 < nnz) ? v0 + 16 : nnz;
  bool oka = v0 + g < v_hi, okb = v0 + g + 8 < v_hi;
  const uint16_t* rowa = Bt + (int64_t)(oka ? ldg32i(col_idx + v0 + g) : 0) * K;
  const uint16_t* rowb = Bt + (int64_t)(okb ? ldg32i(col_idx + v0 + g + 8) : 0) * K;
  uint4 a0, a1, b0, b1;  // Bt chunk [k0, k0 + 64) of vectors g and g+8 (the next one to use)
  load_seg2<VEC>(rowa, K, kt, oka, a0, a1);
  load_seg2<VEC>(rowb, K, kt, okb, b0, b1);
  int64_t w = find_window(row_ptr, W, v0);
  int64_t w_end_p = row_ptr[w + 1];

  for (int64_t s = s_begin; s < s_end; ++s) {
    // next slice's column indices, one slice ahead
    const bool has_next = s + 1 < s_end;
    const int64_t nv0 = v0 + 16;
    const int64_t nv_hi = (nv0 + 16 < nnz) ? nv0 + 16 : nnz;
    const bool noka = has_next && nv0 + g < nv_hi, nokb = has_next && nv0 + g + 8 < nv_hi;
    const int nca = noka ? ldg32i(col_idx + nv0 + g) : 0;
    const int ncb = nokb ? ldg32i(col_idx + nv0 + g + 8) : 0;

    int64_t v_cur = v0;
    while (v_cur < v_hi) {
      while (w_end_p <= v_cur) {  // advance to the window owning v_cur
        ++w;
        w_end_p = row_ptr[w + 1];
      }
      const int64_t seg_hi = w_end_p < v_hi ? w_end_p : v_hi;  // vectors [v_cur, seg_hi) in w
      const bool last_seg = seg_hi == v_hi;
      const int64_t arow = w * V + g;
      const bool ok_row = (g < V) && (arow < M);
      const uint16_t* rowA = A + arow * K;
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      for (int64_t k0 = 0; k0 < K; k0 += 64) {
        uint4 x0, x1;  // A row g of the window, same K permutation
        load_seg2<VEC>(rowA, K, k0 + kt, ok_row, x0, x1);
        const uint4 ca0 = a0, ca1 = a1, cb0 = b0, cb1 = b1;
        if (k0 + 64 < K) {  // next chunk of the same rows
          load_seg2<VEC>(rowa, K, k0 + 64 + kt, oka, a0, a1);
          load_seg2<VEC>(rowb, K, k0 + 64 + kt, okb, b0, b1);
        } else if (!last_seg) {  // the same rows again, for the slice's next window
          load_seg2<VEC>(rowa, K, kt, oka, a0, a1);
          load_seg2<VEC>(rowb, K, kt, okb, b0, b1);
        } else if (has_next) {  // first chunk of the next slice
          load_seg2<VEC>(Bt + (int64_t)nca * K, K, kt, noka, a0, a1);
          load_seg2<VEC>(Bt + (int64_t)ncb * K, K, kt, nokb, b0, b1);
        }
#pragma unroll
        for (int j = 0; j < 4; ++j)
          mma_16816(acc, wordj(ca0, j), wordj(cb0, j), wordj(ca1, j), wordj(cb1, j),
                    wordj(x0, j), wordj(x1, j));
      }
      store_slice<V>(acc, v0, v_cur, seg_hi, w, M, g, t, out, out4);
      v_cur = seg_hi;
    }
    v0 = nv0;
    v_hi = nv_hi;
    oka = noka;
    okb = nokb;
    rowa = Bt + (int64_t)nca * K;
    rowb = Bt + (int64_t)ncb * K;
  }
}

template <int V, bool VEC>
__global__ void __launch_bounds__(kSddmmWarps * 32)
    sddmm_kernel(int64_t M, int64_t K, int64_t W, const int32_t* __restrict__ row_ptr,
                 const int32_t* __restrict__ col_idx, const uint16_t* __restrict__ A,
                 const uint16_t* __restrict__ Bt, uint16_t* __restrict__ out, bool out4) {
  const int64_t nnz = row_ptr[W];
  const int64_t n_slices = ceil_div64(nnz, 16);
  const int64_t n_warps = (int64_t)gridDim.x * kSddmmWarps;
  const int64_t gw = (int64_t)blockIdx.x * kSddmmWarps + (threadIdx.x >> 5);
  const int64_t per = ceil_div64(n_slices, n_warps);
  const int64_t s_begin = gw * per;
  const int64_t s_end = (s_begin + per < n_slices) ? s_begin + per : n_slices;
  if (s_begin >= s_end) return;
  sddmm_range<V, VEC>(M, K, W, row_ptr, col_idx, A, Bt, out, out4, s_begin, s_end, nnz);
}

// Batched launch over up to kSddmmMaxBatch problems of one configuration.  Each problem's
// slices (count from its row_ptr[W], read on the device and prefix-summed per CTA in shared
// memory) are cut into chunks of kSliceChunk slices; the chunks of all problems are dealt
// round-robin to the persistent warps.
struct SddmmDesc {
  int64_t M, K, W;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const uint16_t* A;
  const uint16_t* Bt;
  uint16_t* out;
  int64_t out4;
};
constexpr int kSddmmMaxBatch = 128;
constexpr int kSliceChunk = 8;  // slices per work chunk of the batched kernel
struct SddmmBatch {
  int count;
  SddmmDesc d[kSddmmMaxBatch];
};

template <int V, bool VEC>
__global__ void __launch_bounds__(kSddmmWarps * 32)
    sddmm_batched_kernel(const __grid_constant__ SddmmBatch b) {
  __shared__ int64_t pre[kSddmmMaxBatch + 1];  // prefix of slice-chunk counts
  __shared__ int64_t nnzs[kSddmmMaxBatch];
  const int lane = lane_id();
  if (threadIdx.x < 32) {
    int64_t carry = 0;
    for (int base = 0; base < b.count; base += 32) {
      const int p = base + lane;
      const int64_t nz = p < b.count ? (int64_t)b.d[p].row_ptr[b.d[p].W] : 0;
      const int64_t v = ceil_div64(ceil_div64(nz, 16), kSliceChunk);  // chunks of slices
      int64_t incl = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t x = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += x;
      }
      if (p < b.count) {
        pre[p] = carry + incl - v;
        nnzs[p] = nz;
      }
      carry += __shfl_sync(0xffffffffu, incl, 31);
    }
    if (lane == 0) pre[b.count] = carry;
  }
  __syncthreads();
  // Work is dealt in rounds of chunks of kSliceChunk slices: chunk c of the global chunk
  // sequence goes to warp c % n_warps, so at any time the warps work on neighbouring chunks
  // (one or two problems resident in L2), instead of every warp touching its own problem.
  const int64_t n_chunks = pre[b.count];
  const int64_t n_warps = (int64_t)gridDim.x * kSddmmWarps;
  const int64_t gw = (int64_t)blockIdx.x * kSddmmWarps + (threadIdx.x >> 5);
  int p = 0;
  for (int64_t c = gw; c < n_chunks; c += n_warps) {
    while (pre[p + 1] <= c) ++p;
    const int64_t s0 = (c - pre[p]) * kSliceChunk;
    const int64_t slices = ceil_div64(nnzs[p], 16);
    const int64_t s1 = s0 + kSliceChunk < slices ? s0 + kSliceChunk : slices;
    const SddmmDesc& d = b.d[p];
    sddmm_range<V, VEC>(d.M, d.K, d.W, d.row_ptr, d.col_idx, d.A, d.Bt, d.out, d.out4 != 0, s0, s1,
                        nnzs[p]);
  }
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

template <int V, bool VEC>
static int sddmm_ctas_per_sm() {
  static const int n = ctas_per_sm(sddmm_kernel<V, VEC>);
  return n;
}
template <int V, bool VEC>
static int sddmm_batched_ctas_per_sm() {
  static const int n = ctas_per_sm(sddmm_batched_kernel<V, VEC>);
  return n;
}

template <int V>
static cudaError_t launch_sddmm_v(int64_t M, int64_t N, int64_t K, const int32_t* row_ptr,
                                  const int32_t* col_idx, const uint16_t* A, const uint16_t* Bt,
                                  uint16_t* out, bool vec, int num_sms, cudaStream_t s) {
  (void)N;
  const int64_t W = ceil_div64(M, V);
  dim3 block(kSddmmWarps * 32);
  const bool out4 = (reinterpret_cast<uintptr_t>(out) & 3) == 0;
  if (vec) {
    dim3 grid((unsigned)(num_sms * sddmm_ctas_per_sm<V, true>()));
    sddmm_kernel<V, true><<<grid, block, 0, s>>>(M, K, W, row_ptr, col_idx, A, Bt, out, out4);
  } else {
    dim3 grid((unsigned)(num_sms * sddmm_ctas_per_sm<V, false>()));
    sddmm_kernel<V, false><<<grid, block, 0, s>>>(M, K, W, row_ptr, col_idx, A, Bt, out, out4);
  }
  return cudaGetLastError();
}

template <int V, bool VEC>
static void launch_sddmm_batch(const SddmmBatch& b, int num_sms, cudaStream_t s) {
  dim3 grid((unsigned)(num_sms * sddmm_batched_ctas_per_sm<V, VEC>()));
  sddmm_batched_kernel<V, VEC><<<grid, kSddmmWarps * 32, 0, s>>>(b);
}

cudaError_t launch_sddmm_batched(int64_t count, const int64_t* M, const int64_t* K, const int* V,
                                 const int32_t* const* row_ptr, const int32_t* const* col_idx,
                                 const void* const* A, const void* const* Bt, void* const* out,
                                 int num_sms, cudaStream_t s) {
  // group by (V, vector path); keep the caller's order inside a group
  std::vector<std::pair<int, int64_t>> order;
  for (int64_t i = 0; i < count; ++i) {
    const bool vec = (K[i] % 8 == 0) && ((reinterpret_cast<uintptr_t>(A[i]) & 15) == 0) &&
                     ((reinterpret_cast<uintptr_t>(Bt[i]) & 15) == 0);
    order.push_back({V[i] * 2 + (vec ? 1 : 0), i});
  }
  std::stable_sort(order.begin(), order.end(),
                   [](const auto& a, const auto& b) { return a.first < b.first; });
  SddmmBatch batch;
  size_t i = 0;
  while (i < order.size()) {
    const int key = order[i].first;
    batch.count = 0;
    while (i < order.size() && order[i].first == key && batch.count < kSddmmMaxBatch) {
      const int64_t p = order[i].second;
      SddmmDesc& d = batch.d[batch.count++];
      d = {M[p], K[p], ceil_div64(M[p], V[p]), row_ptr[p], col_idx[p],
           static_cast<const uint16_t*>(A[p]), static_cast<const uint16_t*>(Bt[p]),
           static_cast<uint16_t*>(out[p]), (reinterpret_cast<uintptr_t>(out[p]) & 3) == 0 ? 1 : 0};
      ++i;
    }
    const bool vec = key & 1;
    switch (key >> 1) {
      case 1: vec ? launch_sddmm_batch<1, true>(batch, num_sms, s) : launch_sddmm_batch<1, false>(batch, num_sms, s); break;
      case 2: vec ? launch_sddmm_batch<2, true>(batch, num_sms, s) : launch_sddmm_batch<2, false>(batch, num_sms, s); break;
      case 4: vec ? launch_sddmm_batch<4, true>(batch, num_sms, s) : launch_sddmm_batch<4, false>(batch, num_sms, s); break;
      default: vec ? launch_sddmm_batch<8, true>(batch, num_sms, s) : launch_sddmm_batch<8, false>(batch, num_sms, s); break;
    }
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

cudaError_t launch_sddmm(int64_t M, int64_t N, int64_t K, int V, const int32_t* row_ptr,
                         const int32_t* col_idx, const void* A, const void* Bt, void* out,
                         int num_sms, cudaStream_t s) {
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
