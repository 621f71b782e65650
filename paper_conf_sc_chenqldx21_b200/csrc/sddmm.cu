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

template <int V, bool VEC>
__global__ void __launch_bounds__(kSddmmWarps * 32)
    sddmm_kernel(int64_t M, int64_t K, int64_t W, const int32_t* __restrict__ row_ptr,
                 const int32_t* __restrict__ col_idx, const uint16_t* __restrict__ A,
                 const uint16_t* __restrict__ Bt, uint16_t* __restrict__ out, bool out4) {
  const int lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int64_t nnz = row_ptr[W];
  const int64_t n_slices = ceil_div64(nnz, 16);
  const int64_t n_warps = (int64_t)gridDim.x * kSddmmWarps;
  const int64_t gw = (int64_t)blockIdx.x * kSddmmWarps + (threadIdx.x >> 5);
  const int64_t per = ceil_div64(n_slices, n_warps);
  const int64_t s_begin = gw * per;
  const int64_t s_end = (s_begin + per < n_slices) ? s_begin + per : n_slices;
  if (s_begin >= s_end) return;

  int64_t w = find_window(row_ptr, W, s_begin * 16);
  int64_t w_end_p = row_ptr[w + 1];  // first vector after window w

  for (int64_t s = s_begin; s < s_end; ++s) {
    const int64_t v0 = s * 16;
    const int64_t v_hi = (v0 + 16 < nnz) ? v0 + 16 : nnz;
    // the two vectors (M rows g and g+8) this thread loads Bt rows for
    const int64_t va = v0 + g, vb = v0 + g + 8;
    const bool oka = va < v_hi, okb = vb < v_hi;
    const int ca = oka ? ldg32i(col_idx + va) : 0;
    const int cb = okb ? ldg32i(col_idx + vb) : 0;
    const uint16_t* rowa = Bt + (int64_t)ca * K;
    const uint16_t* rowb = Bt + (int64_t)cb * K;

    int64_t v_cur = v0;
    while (v_cur < v_hi) {
      while (w_end_p <= v_cur) {  // advance to the window owning v_cur
        ++w;
        w_end_p = row_ptr[w + 1];
      }
      const int64_t seg_hi = w_end_p < v_hi ? w_end_p : v_hi;  // vectors [v_cur, seg_hi) in w
      const int64_t arow = w * V + g;
      const bool oka_row = (g < V) && (arow < M);
      const uint16_t* rowA = A + arow * K;

      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      for (int64_t k0 = 0; k0 < K; k0 += 128) {
        uint4 a0[2], a1[2], b0[2], b1[2], x0[2], x1[2];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int64_t k = k0 + 64 * h + 8 * t;
          load_seg2<VEC>(rowa, K, k, oka, a0[h], a1[h]);      // Bt row of vector g
          load_seg2<VEC>(rowb, K, k, okb, b0[h], b1[h]);      // Bt row of vector g+8
          load_seg2<VEC>(rowA, K, k, oka_row, x0[h], x1[h]);  // A row g of the window
        }
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
          for (int j = 0; j < 4; ++j)
            mma_16816(acc, wordj(a0[h], j), wordj(b0[h], j), wordj(a1[h], j), wordj(b1[h], j),
                      wordj(x0[h], j), wordj(x1[h], j));
      }
      // acc[0..1]: vector v0+g, rows 2t, 2t+1; acc[2..3]: vector v0+g+8, rows 2t, 2t+1.
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const int64_t v = v0 + g + 8 * q;
        if (v < v_cur || v >= seg_hi) continue;
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
      v_cur = seg_hi;
    }
  }
}

template <int V>
static cudaError_t launch_sddmm_v(int64_t M, int64_t N, int64_t K, const int32_t* row_ptr,
                                  const int32_t* col_idx, const uint16_t* A, const uint16_t* Bt,
                                  uint16_t* out, bool vec, int num_sms, cudaStream_t s) {
  (void)N;
  const int64_t W = ceil_div64(M, V);
  dim3 block(kSddmmWarps * 32);
  dim3 grid((unsigned)(num_sms * 8));  // persistent: 8 CTAs (32 warps) per SM
  const bool out4 = (reinterpret_cast<uintptr_t>(out) & 3) == 0;
  if (vec)
    sddmm_kernel<V, true><<<grid, block, 0, s>>>(M, K, W, row_ptr, col_idx, A, Bt, out, out4);
  else
    sddmm_kernel<V, false><<<grid, block, 0, s>>>(M, K, W, row_ptr, col_idx, A, Bt, out, out4);
  return cudaGetLastError();
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
