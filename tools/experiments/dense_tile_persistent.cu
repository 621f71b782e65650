// dense_tile.cu — dense-tile tcgen05 kernels for the 128-row blocks the B200 cost model
// (dense_select.cuh) sends away from the column-vector gather kernels.
//
// Why: a stored V x 1 vector gives the gather kernels V flop per gathered byte
// (AL1), and B200 moves ~8-20 TB/s of random rows from L2 into the SMs against
// ~1.5-2 PFLOP/s of dense fp16 tensor throughput.  Where a 128-row block holds more than
// 128 * Lc / CF stored vectors, computing its whole dense tile on the tensor cores costs less
// than gathering its vectors.  The results are the same sums (fp32 accumulate, fp16
// round-to-nearest-even output); absent vectors only add exact zero products (SpMM) or are not
// stored (SDDMM).
//
// SDDMM  out[p*V + r] = sum_k A[wV+r][k] * Bt[col_idx[p]][k]   (§6)
//   Unit = (problem, 128-row block rb of A, 128-column tile ct of the mask): one CTA of 4 warps,
//   non-persistent (3 resident per SM, so one CTA's loads overlap another's MMAs / epilogue).
//   D[128 mask cols x 128 A rows] (fp32, TMEM, 128 columns) = Bt[c0:c0+128, :] * A[r0:r0+128, :]^T
//   with tcgen05.mma M = 128, N = 128, K = 16 (the operand switch of P:1059-1063: mask columns on
//   the MMA M side), both operands K-contiguous rows loaded by TMA 2-D tile copies (SWIZZLE_128B
//   = the canonical K-major layout), a 2-stage ring of 64-wide K slabs (any inner K).  Warp 0
//   lane 0 issues the TMA copies, warp 1 lane 0 the MMAs; then every warp drains its TMEM lane
//   quarter (thread = mask column c) into a shared tile Tt[c][r] (fp16 RN, rows >= M are +0;
//   each c a 256-byte row, 16-byte chunks XOR-swizzled by c), so the V rows of a window at
//   column c are 2V contiguous bytes.  Sampling: warp j takes windows j, j+4, ... of the row
//   block and walks each window's col_idx (16-byte loads); every stored vector whose column
//   falls in the tile gets one 2V-byte shared load and one 2V-byte global store -- any col_idx
//   order, duplicates included.
//
// SpMM  C[i][n] = sum_p vals[p*V + i%V] * B[col_idx[p]][n]   (§5)  [opt-in build]
//   Unit = (problem, 32-row block of A / C).  The unit's stored vectors (contiguous: the
//   windows of the 32 rows) are decoded once into a dense [32 rows x K] fp16 tile in shared
//   memory (K-major, 128-byte swizzle; K <= 2048), then for every 128-column panel of B:
//   D[128 panel cols x 32 rows] (fp32, TMEM) = B[:, n0:n0+128]^T * A_tile^T with tcgen05.mma
//   M = 128, N = 32, K = 16 (the operand switch of P:858-871: B columns on the MMA M side, B
//   MN-major straight from TMA 2-D tiles), and the epilogue stores the tile into C (fp16 RN;
//   to every destination of vs_spmm_scatter).  Absent vectors are exact zeros of the tile.
//   A window whose col_idx is not strictly ascending (duplicates, any order) is not taken here:
//   its rows are left to the gather kernel, which checks the same condition.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>
#include <vector>

#include "common.cuh"
#include "dense_select.cuh"
#include "tc_common.cuh"

#if VS_SDDMM_DENSE_CF > 0 || VS_SPMM_DENSE_CF > 0
namespace vs {
namespace dt {

constexpr int kMaxProb = 32;  // problems per launch (tensor maps travel as kernel parameters)

static PFN_cuTensorMapEncodeTiled_v12000 tmap_encoder();
static bool make_kmajor_map(CUtensorMap* m, const void* base, int64_t rows, int64_t K, int box_rows);
static bool make_mnmajor_map(CUtensorMap* m, const void* base, int64_t K, int64_t N);

}  // namespace dt
}  // namespace vs
#endif

#if VS_SDDMM_DENSE_CF > 0
namespace vs {
namespace dt {

// ================================================================================ SDDMM
// Persistent warp-specialised kernel, one CTA per SM walking the units blockIdx.x, + gridDim.x, ...
// Roles (each walks the same unit sequence and skips the gather kernel's row blocks by the same
// predicate, so the per-role counters of dense units agree):
//   warp 0      TMA producer: Bt slab + A slab of every 64-wide K block into a kSdStages ring
//   warp 1      MMA issuer: D[acc] (two 128-column TMEM accumulators) += Bt slab * A slab^T
//   warps 2-5   search: warp s takes dense units j with j % 4 == s and writes, per window, the
//               range [lo, hi) of its vectors in the tile's column range into slot s
//   warps 6-13  epilogue, two groups of 4 warps: group g takes dense units j with j % 2 == g
//               (= accumulator g): TMEM -> Tt[g] (fp16), then the store pass from Tt[g]
// so the TMA stream, the searches and the store passes of different units overlap.
constexpr int kSdU = 128;                      // A rows per unit (MMA N; TMEM columns per accumulator)
constexpr int kSdBtSlab = 128 * 128;           // bytes: 128 mask columns x 64 k fp16 (16 KB)
constexpr int kSdASlab = kSdU * 128;           // bytes: 128 A rows x 64 k fp16 (16 KB)
constexpr int kSdStage = kSdBtSlab + kSdASlab;
constexpr int kSdStages = 2;
constexpr int kSdSearchWarps = 4;
constexpr int kSdEpiGroups = 4;
constexpr int kSdTt = 128 * kSdU * 2;          // 32 KB fp16 tile per epilogue group
constexpr int kSdThreads = 32 * (2 + kSdSearchWarps + 4 * kSdEpiGroups);  // 448
constexpr int kSdSmem = kSdStages * kSdStage + kSdEpiGroups * kSdTt + 1024;  // + alignment slack
constexpr uint32_t kIdescSd = tc::idesc_f16(128, kSdU, 0, 0);
constexpr int kSdSwz = kSdU / 8 - 1;           // Tt chunk swizzle mask (chunks per 2*kSdU-byte row - 1)

struct alignas(64) SdDesc {
  CUtensorMap tmA;   // A [M x K] fp16, box {64, kSdU}, SWIZZLE_128B
  CUtensorMap tmBt;  // Bt [N x K] fp16, box {64, 128}, SWIZZLE_128B
  int64_t M, N, K, W, n_ct;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  uint16_t* out;
  int32_t V, out_vec, col16;  // out_vec: out is 2V-byte aligned; col16: col_idx 16-byte aligned
};
struct SdBatch {
  int count;
  int64_t unit_begin, unit_end;  // the launch's unit range (<= gridDim.x * kSdListCap units)
  int64_t first_unit[kMaxProb + 1];
  SdDesc d[kMaxProb];
};

// out[e*V .. e*V + V) = the V fp16 values at shared address a (2V contiguous bytes)
__device__ __forceinline__ void sd_sample_store(uint32_t a, uint16_t* dst, int V, bool vec) {
  if (vec && V == 8) {
    *reinterpret_cast<uint4*>(dst) = lds128_u32(a);
  } else if (vec && V == 4) {
    uint32_t x, y;
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(x), "=r"(y) : "r"(a));
    *reinterpret_cast<uint2*>(dst) = make_uint2(x, y);
  } else if (vec && V == 2) {
    uint32_t x;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(x) : "r"(a));
    *reinterpret_cast<uint32_t*>(dst) = x;
  } else {
    for (int r = 0; r < V; ++r) dst[r] = lds16(a + 2 * r);
  }
}

// Smallest i in [lo, hi] with a[i] >= x, for two targets at once (a[lo, hi) ascending, a[hi]
// taken as +inf): 9-ary search, 8 independent probes per target per round trip (a 1024-entry
// window takes 3 rounds + one of <= 8 loads), so the latency of one thread's search is ~4 L2
// round trips.  On a window that is not ascending the result is some index in [lo, hi].
__device__ __forceinline__ void kary_lower_bound2(const int32_t* __restrict__ a, int lo, int hi, int x1, int x2,
                                                  int& r1, int& r2) {
  int l1 = lo, h1 = hi, l2 = lo, h2 = hi;
  while (h1 - l1 > 8 || h2 - l2 > 8) {
    const int s1 = (h1 - l1) / 9, s2 = (h2 - l2) / 9;
    int c1 = 0, c2 = 0;
#pragma unroll
    for (int i = 1; i <= 8; ++i) {
      c1 += (s1 > 0 && __ldg(a + l1 + s1 * i) < x1) ? 1 : 0;
      c2 += (s2 > 0 && __ldg(a + l2 + s2 * i) < x2) ? 1 : 0;
    }
    if (s1 > 0) {
      const int nh = c1 < 8 ? l1 + s1 * (c1 + 1) : h1;
      l1 = c1 > 0 ? l1 + s1 * c1 + 1 : l1;
      h1 = nh;
    }
    if (s2 > 0) {
      const int nh = c2 < 8 ? l2 + s2 * (c2 + 1) : h2;
      l2 = c2 > 0 ? l2 + s2 * c2 + 1 : l2;
      h2 = nh;
    }
  }
  int c1 = 0, c2 = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    c1 += (l1 + i < h1 && __ldg(a + l1 + i) < x1) ? 1 : 0;
    c2 += (l2 + i < h2 && __ldg(a + l2 + i) < x2) ? 1 : 0;
  }
  r1 = l1 + c1;
  r2 = l2 + c2;
}

// Store pass of one unit: warp j takes windows j, j + 4, ... of the unit, eight windows per
// round with their first 64 vectors' col_idx loads in flight together (lane = vector: coalesced
// loads, 2V-byte shared load + 2V-byte global store each); the window's vectors in the tile's
// column range are [lo, hi) (searched before the drain).  A vector whose column is outside the
// range (possible only in a window that is not ascending) is not stored.
// Tt[c][r]: 2*kSdU-byte row per mask column c, 16-byte chunk j of it at j ^ (c & kSdSwz).
__device__ __forceinline__ void sd_store1(const SdDesc& d, uint32_t tt, uint32_t rofs, int e, int col, int c0, int V,
                                          bool vec) {
  const uint32_t c = (uint32_t)(col - c0);
  if (col >= 0 && c < 128u)
    sd_sample_store(tt + c * (2 * kSdU) + (((rofs >> 3) ^ (c & kSdSwz)) << 4) + (rofs & 7) * 2, d.out + (int64_t)e * V, V,
                    vec);
}
constexpr int kSdStoreWin = 4;  // windows per warp round of the store pass
constexpr int kSdWarps = 4;     // warps of an epilogue group
__device__ __forceinline__ void sd_store(const SdDesc& d, uint32_t tt, const int32_t* lo_s, const int32_t* hi_s,
                                         int nwin, int c0, int V, int warp, int lane) {
  const bool vec = d.out_vec != 0;
  const int32_t* __restrict__ ci = d.col_idx;
  for (int wb = warp; wb < nwin; wb += kSdWarps * kSdStoreWin) {
    int lo[kSdStoreWin], hi[kSdStoreWin], ca[kSdStoreWin], cb[kSdStoreWin];
#pragma unroll
    for (int u = 0; u < kSdStoreWin; ++u) {
      const int wl = wb + kSdWarps * u;
      lo[u] = wl < nwin ? lo_s[wl] : 0;
      hi[u] = wl < nwin ? hi_s[wl] : 0;
    }
#pragma unroll
    for (int u = 0; u < kSdStoreWin; ++u) {
      ca[u] = lo[u] + lane < hi[u] ? __ldg(ci + lo[u] + lane) : -1;
      cb[u] = lo[u] + 32 + lane < hi[u] ? __ldg(ci + lo[u] + 32 + lane) : -1;
    }
#pragma unroll
    for (int u = 0; u < kSdStoreWin; ++u) {
      const uint32_t rofs = (uint32_t)((wb + kSdWarps * u) * V);
      sd_store1(d, tt, rofs, lo[u] + lane, ca[u], c0, V, vec);
      sd_store1(d, tt, rofs, lo[u] + 32 + lane, cb[u], c0, V, vec);
    }
#pragma unroll
    for (int u = 0; u < kSdStoreWin; ++u) {  // windows with more than 64 vectors in the tile (dense ones)
      const uint32_t rofs = (uint32_t)((wb + kSdWarps * u) * V);
      for (int e0 = lo[u] + 64; e0 < hi[u]; e0 += 64) {
        const int e1 = e0 + lane, e2 = e0 + 32 + lane;
        const int c1 = e1 < hi[u] ? __ldg(ci + e1) : -1;
        const int c2 = e2 < hi[u] ? __ldg(ci + e2) : -1;
        sd_store1(d, tt, rofs, e1, c1, c0, V, vec);
        sd_store1(d, tt, rofs, e2, c2, c0, V, vec);
      }
    }
  }
}

// Store pass, 16-byte col_idx loads (col_idx 16-byte aligned; sd_store otherwise): lane l of warp
// j loads entries [4l, 4l + 4) of the 16-byte groups covering [lo, hi) of windows j, j + 4, ...,
// eight windows per round (eight 16-byte loads per lane in flight), and stores the in-range
// ones; Tt is read with plain shared-memory loads (the compiler hoists them ahead of the
// stores).  Windows with more than 125 vectors in the tile continue in a loop.
constexpr int kSdStoreWin4 = 8;
template <int V>
__device__ __forceinline__ void sd_out(const SdDesc& d, const uint8_t* tt, uint32_t rofs, int e, int col, int c0,
                                       bool vec) {
  const uint32_t c = (uint32_t)(col - c0);
  if (col < 0 || c >= 128u) return;
  const uint8_t* a = tt + c * (2 * kSdU) + ((((rofs >> 3) ^ (c & kSdSwz))) << 4) + (rofs & 7) * 2;
  uint16_t* dst = d.out + (int64_t)e * V;
  if (vec && V == 8) {
    *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(a);
  } else if (vec && V == 4) {
    *reinterpret_cast<uint2*>(dst) = *reinterpret_cast<const uint2*>(a);
  } else if (vec && V == 2) {
    *reinterpret_cast<uint32_t*>(dst) = *reinterpret_cast<const uint32_t*>(a);
  } else {
#pragma unroll
    for (int r = 0; r < V; ++r) dst[r] = reinterpret_cast<const uint16_t*>(a)[r];
  }
}
// col_idx[e, e + 4) with entries >= h as -1; one 16-byte load when all four are below h (no
// read past h: the last group of col_idx may end mid-way through a 16-byte block)
__device__ __forceinline__ int4 sd_ld4(const int32_t* __restrict__ ci, int e, int h) {
  if (e + 3 < h) return __ldg(reinterpret_cast<const int4*>(ci + e));
  return make_int4(e < h ? __ldg(ci + e) : -1, e + 1 < h ? __ldg(ci + e + 1) : -1, e + 2 < h ? __ldg(ci + e + 2) : -1, -1);
}
template <int V>
__device__ __forceinline__ void sd_store4(const SdDesc& d, const uint8_t* tt, const int32_t* lo_s, const int32_t* hi_s,
                                          int nwin, int c0, int warp, int lane) {
  const bool vec = d.out_vec != 0;
  const int32_t* __restrict__ ci = d.col_idx;
  for (int wb = warp; wb < nwin; wb += kSdWarps * kSdStoreWin4) {
    int lo[kSdStoreWin4], hi[kSdStoreWin4];
    int4 cv[kSdStoreWin4];
#pragma unroll
    for (int u = 0; u < kSdStoreWin4; ++u) {
      const int wl = wb + kSdWarps * u;
      lo[u] = wl < nwin ? lo_s[wl] : 0;
      hi[u] = wl < nwin ? hi_s[wl] : 0;
    }
#pragma unroll
    for (int u = 0; u < kSdStoreWin4; ++u) cv[u] = sd_ld4(ci, (lo[u] & ~3) + 4 * lane, hi[u]);
#pragma unroll
    for (int u = 0; u < kSdStoreWin4; ++u) {
      const uint32_t rofs = (uint32_t)((wb + kSdWarps * u) * V);
      const int e = (lo[u] & ~3) + 4 * lane;
      sd_out<V>(d, tt, rofs, e, e >= lo[u] && e < hi[u] ? cv[u].x : -1, c0, vec);
      sd_out<V>(d, tt, rofs, e + 1, e + 1 >= lo[u] && e + 1 < hi[u] ? cv[u].y : -1, c0, vec);
      sd_out<V>(d, tt, rofs, e + 2, e + 2 >= lo[u] && e + 2 < hi[u] ? cv[u].z : -1, c0, vec);
      sd_out<V>(d, tt, rofs, e + 3, e + 3 >= lo[u] && e + 3 < hi[u] ? cv[u].w : -1, c0, vec);
    }
#pragma unroll 1
    for (int u = 0; u < kSdStoreWin4; ++u) {  // windows with vectors past the first 128-entry group row
      const int wl = wb + kSdWarps * u;
      if (wl >= nwin) break;
      const int l = lo_s[wl], h = hi_s[wl];
      const uint32_t rofs = (uint32_t)(wl * V);
      for (int g = (l & ~3) + 128; g < h; g += 128) {
        const int e = g + 4 * lane;
        const int4 x = sd_ld4(ci, e, h);
        sd_out<V>(d, tt, rofs, e, e < h ? x.x : -1, c0, vec);
        sd_out<V>(d, tt, rofs, e + 1, e + 1 < h ? x.y : -1, c0, vec);
        sd_out<V>(d, tt, rofs, e + 2, e + 2 < h ? x.z : -1, c0, vec);
        sd_out<V>(d, tt, rofs, e + 3, e + 3 < h ? x.w : -1, c0, vec);
      }
    }
  }
}

// Unit u of the batch: problem, 128-row block, 128-column tile, and whether the row block is
// the dense kernel's (dense_select.cuh: the same predicate as sddmm_rb_dense).
struct SdUnit {
  int p, rb, ct, nwin;
  int64_t w0;
};
__device__ __forceinline__ void sd_decode(const SdBatch& b, int64_t u, SdUnit& x) {
  x.p = first_problem(b.first_unit, b.count, u);
  const SdDesc& d = b.d[x.p];
  const int loc = (int)(u - b.first_unit[x.p]);  // < 2^31 (sddmm_dense_eligible)
  const int n_ct = (int)d.n_ct;
  x.rb = loc / n_ct;
  x.ct = loc - x.rb * n_ct;
  int64_t w1;
  rb_windows(x.rb, d.V, d.W, x.w0, w1);
  x.nwin = (int)(w1 - x.w0);
}
__device__ __forceinline__ bool sd_dense(const SdBatch& b, const SdUnit& x) {
  const SdDesc& d = b.d[x.p];
  const int64_t nnz = (int64_t)__ldg(d.row_ptr + x.w0 + x.nwin) - (int64_t)__ldg(d.row_ptr + x.w0);
  return nnz * (int64_t)VS_SDDMM_DENSE_CF > (int64_t)kDenseRows * (d.n_ct * 128);
}
constexpr int kSdListCap = 2048;  // dense units per CTA per launch (the host splits larger launches)

__global__ void __launch_bounds__(kSdThreads, 1) sddmm_dense_kernel(const __grid_constant__ SdBatch b) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t full_bar[kSdStages], empty_bar[kSdStages];
  __shared__ __align__(8) uint64_t tfull_bar[kSdEpiGroups], tempty_bar[kSdEpiGroups];
  __shared__ __align__(8) uint64_t sfull_bar[kSdSearchWarps], sempty_bar[kSdSearchWarps];
  __shared__ uint32_t tmem_base_sh;
  __shared__ int32_t lo_s[kSdSearchWarps][kSdU], hi_s[kSdSearchWarps][kSdU];
  __shared__ int32_t ulist[kSdListCap];  // the CTA's dense units (offsets from b.unit_begin)
  __shared__ int n_dense_sh;
  const uint32_t smem = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t s_ring = smem, s_tt = smem + kSdStages * kSdStage;
  const int warp = threadIdx.x >> 5, lane = lane_id();

  if (threadIdx.x == 0) {
    for (int s = 0; s < kSdStages; ++s) {
      tc::mbar_init(smem_u32(&full_bar[s]), 1);
      tc::mbar_init(smem_u32(&empty_bar[s]), 1);
    }
    for (int a = 0; a < kSdEpiGroups; ++a) {
      tc::mbar_init(smem_u32(&tfull_bar[a]), 1);
      tc::mbar_init(smem_u32(&tempty_bar[a]), 4);  // one arrive per warp of the epilogue group
    }
    for (int s = 0; s < kSdSearchWarps; ++s) {
      tc::mbar_init(smem_u32(&sfull_bar[s]), 1);
      tc::mbar_init(smem_u32(&sempty_bar[s]), 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(kSdEpiGroups * kSdU));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  // ---- the CTA's dense units (ascending), evaluated in parallel: one round trip per 448 units
  // instead of one per unit in every role
  {
    const int64_t mine = b.unit_end > b.unit_begin + blockIdx.x
                             ? ceil_div64(b.unit_end - b.unit_begin - blockIdx.x, gridDim.x) : 0;
    __shared__ int wcnt[kSdThreads / 32];
    int running = 0;
    for (int64_t base = 0; base < mine; base += kSdThreads) {
      const int64_t idx = base + threadIdx.x;
      const int64_t u = b.unit_begin + blockIdx.x + idx * gridDim.x;
      bool dense = false;
      if (idx < mine) {
        SdUnit x;
        sd_decode(b, u, x);
        dense = sd_dense(b, x);
      }
      const unsigned bal = __ballot_sync(0xffffffffu, dense);
      if (lane == 0) wcnt[warp] = __popc(bal);
      __syncthreads();
      int before = running, tot = 0;
      for (int w = 0; w < kSdThreads / 32; ++w) {
        if (w < warp) before += wcnt[w];
        tot += wcnt[w];
      }
      if (dense) ulist[before + __popc(bal & ((1u << lane) - 1u))] = (int32_t)(u - b.unit_begin);
      running += tot;
      __syncthreads();
    }
    if (threadIdx.x == 0) n_dense_sh = running;
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = tmem_base_sh;
  const int n_dense = n_dense_sh;

  if (warp == 0) {
    // ================================ TMA producer ================================
    if (lane == 0) {
      uint32_t it = 0;
      SdUnit x;
      for (int li = 0; li < n_dense; ++li) {
        sd_decode(b, b.unit_begin + ulist[li], x);
        const SdDesc& d = b.d[x.p];
        const int KB = (int)ceil_div64(d.K, 64);
        for (int kb = 0; kb < KB; ++kb, ++it) {
          const uint32_t s = it % kSdStages, use = it / kSdStages;
          if (use > 0) tc::mbar_wait(smem_u32(&empty_bar[s]), (use - 1) & 1);
          const uint32_t st = s_ring + s * kSdStage;
          tc::mbar_expect_tx(smem_u32(&full_bar[s]), kSdStage);
          tc::tma_load_2d(st, &d.tmBt, kb * 64, x.ct * 128, smem_u32(&full_bar[s]));
          tc::tma_load_2d(st + kSdBtSlab, &d.tmA, kb * 64, x.rb * kSdU, smem_u32(&full_bar[s]));
        }
      }
    }
  } else if (warp == 1) {
    // ================================ MMA issuer ================================
    if (lane == 0) {
      uint32_t it = 0, seq = 0;
      SdUnit x;
      for (int li = 0; li < n_dense; ++li) {
        sd_decode(b, b.unit_begin + ulist[li], x);
        const SdDesc& d = b.d[x.p];
        const int KB = (int)ceil_div64(d.K, 64);
        const uint32_t acc = seq % kSdEpiGroups;
        tc::mbar_wait(smem_u32(&tempty_bar[acc]), ((seq / kSdEpiGroups) & 1) ^ 1);
        tc::fence_after();
        for (int kb = 0; kb < KB; ++kb, ++it) {
          const uint32_t s = it % kSdStages, use = it / kSdStages;
          tc::mbar_wait(smem_u32(&full_bar[s]), use & 1);
          tc::fence_after();
          const uint32_t st = s_ring + s * kSdStage;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            tc::mma(tmem + acc * kSdU, tc::sdesc(st + 32 * k, 16, 1024), tc::sdesc(st + kSdBtSlab + 32 * k, 16, 1024),
                    kIdescSd, (kb > 0 || k > 0) ? 1u : 0u);
          tc::commit(smem_u32(&empty_bar[s]));
        }
        tc::commit(smem_u32(&tfull_bar[acc]));
        ++seq;
      }
    }
  } else if (warp < 2 + kSdSearchWarps) {
    // ================================ search ================================
#ifndef VS_SD_EXP
#define VS_SD_EXP 0
#endif
    const int sw = warp - 2;
    uint32_t seq = 0;
    SdUnit x;
    for (int li = 0; li < n_dense; ++li) {
      if ((int)(seq % kSdSearchWarps) == sw) {
        sd_decode(b, b.unit_begin + ulist[li], x);
        const uint32_t use = seq / kSdSearchWarps;
        tc::mbar_wait(smem_u32(&sempty_bar[sw]), (use & 1) ^ 1);
        const SdDesc& d = b.d[x.p];
        const int c0 = x.ct * 128;
        for (int i = lane; i < (VS_SD_EXP >= 2 ? 0 : x.nwin); i += 32) {
          int lo, hi;
          kary_lower_bound2(d.col_idx, __ldg(d.row_ptr + x.w0 + i), __ldg(d.row_ptr + x.w0 + i + 1), c0, c0 + 128, lo,
                            hi);
          lo_s[sw][i] = lo;
          hi_s[sw][i] = hi > lo ? hi : lo;
        }
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(smem_u32(&sfull_bar[sw]));
      }
      ++seq;
    }
  } else {
    // ================================ epilogue ================================
    const int ew = warp - 2 - kSdSearchWarps;  // 0 .. 4 * kSdEpiGroups - 1
    const int g = ew >> 2, gw = ew & 3;         // group, warp within the group
    const int q = warp & 3;                     // TMEM lane quarter (tcgen05.ld: warp % 4)
    const uint32_t tt = s_tt + g * kSdTt;
    const int c = 32 * q + lane;                // mask column of this thread in the drain
    const uint32_t trow = tt + (uint32_t)c * (2 * kSdU);
    uint32_t seq = 0;
    SdUnit x;
    for (int li = 0; li < n_dense; ++li) {
      if ((int)(seq % kSdEpiGroups) == g) {
        sd_decode(b, b.unit_begin + ulist[li], x);
        const SdDesc& d = b.d[x.p];
        const uint32_t use = seq / kSdEpiGroups;  // this group's use of accumulator g
        // ---- drain: Tt[c][r] fp16 (RN), rows >= M +0, 16-byte chunks XOR-swizzled by c
        tc::mbar_wait(smem_u32(&tfull_bar[g]), use & 1);
        tc::fence_after();
        const int64_t rows_valid = d.M - (int64_t)x.rb * kSdU;
#pragma unroll 1
        for (int j = 0; j < kSdU / 32; ++j) {
          uint32_t v[32];
          tc::ld32(tmem + g * kSdU + ((uint32_t)(32 * q) << 16) + 32 * j, v);
          tc::ld_wait();
          uint32_t h[16];
#pragma unroll
          for (int xx = 0; xx < 16; ++xx) {
            const int r = 32 * j + 2 * xx;
            const float f0 = r < rows_valid ? __uint_as_float(v[2 * xx]) : 0.f;
            const float f1 = r + 1 < rows_valid ? __uint_as_float(v[2 * xx + 1]) : 0.f;
            h[xx] = f2_to_h2(f0, f1);
          }
#pragma unroll
          for (int m = 0; m < 4; ++m)
            asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(
                             trow + ((((uint32_t)(4 * j + m)) ^ (c & kSdSwz)) << 4)),
                         "r"(h[4 * m]), "r"(h[4 * m + 1]), "r"(h[4 * m + 2]), "r"(h[4 * m + 3])
                         : "memory");
        }
        tc::fence_before();
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(smem_u32(&tempty_bar[g]));
        tc::named_bar(1 + g, 128);  // Tt[g] complete
        // ---- store pass (slot of the search warp that took this unit)
        const uint32_t slot = seq % kSdSearchWarps, suse = seq / kSdSearchWarps;
        tc::mbar_wait(smem_u32(&sfull_bar[slot]), suse & 1);
#ifndef VS_SD_EXP
#define VS_SD_EXP 0
#endif
        if (VS_SD_EXP == 0) {
          if (d.col16) {
            const uint8_t* ttp = smem_raw + (tt - smem_u32(smem_raw));
            switch (d.V) {
              case 1: sd_store4<1>(d, ttp, lo_s[slot], hi_s[slot], x.nwin, x.ct * 128, gw, lane); break;
              case 2: sd_store4<2>(d, ttp, lo_s[slot], hi_s[slot], x.nwin, x.ct * 128, gw, lane); break;
              case 4: sd_store4<4>(d, ttp, lo_s[slot], hi_s[slot], x.nwin, x.ct * 128, gw, lane); break;
              default: sd_store4<8>(d, ttp, lo_s[slot], hi_s[slot], x.nwin, x.ct * 128, gw, lane); break;
            }
          } else {
            sd_store(d, tt, lo_s[slot], hi_s[slot], x.nwin, x.ct * 128, d.V, gw, lane);
          }
        }
        tc::named_bar(1 + g, 128);  // Tt[g] and the slot read by the whole group
        if (gw == 0 && lane == 0) tc::mbar_arrive(smem_u32(&sempty_bar[slot]));
      }
      ++seq;
    }
  }

  tc::fence_before();
  __syncthreads();
  if (warp == 0) {
    tc::fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kSdEpiGroups * kSdU));
  }
}

static cudaError_t launch_sd(SdBatch& b, int num_sms, cudaStream_t s) {
  static std::once_flag once[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64)
    std::call_once(once[dev], [] {
      cudaFuncSetAttribute(sddmm_dense_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSdSmem);
    });
  const int64_t units = b.first_unit[b.count];
  const int grid = (int)std::min<int64_t>(num_sms, units);
  if (grid <= 0) return cudaSuccess;
  const int64_t per_launch = (int64_t)grid * kSdListCap;
  for (int64_t u0 = 0; u0 < units; u0 += per_launch) {
    b.unit_begin = u0;
    b.unit_end = std::min<int64_t>(units, u0 + per_launch);
    sddmm_dense_kernel<<<grid, kSdThreads, kSdSmem, s>>>(b);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace dt

// Problems the dense SDDMM path can take at all (the per-row-block choice is made on the
// device): 0 < K with K % 8 == 0 (16-byte TMA row stride), 16-byte aligned A and Bt, row and
// column counts that fit the int32 TMA coordinates.
bool sddmm_dense_eligible(int64_t M, int64_t N, int64_t K, int V, const void* A, const void* Bt) {
  return M > 0 && N > 0 && K > 0 && V >= 1 && V <= 8 && K % 8 == 0 &&
         ((reinterpret_cast<uintptr_t>(A) & 15) == 0) && ((reinterpret_cast<uintptr_t>(Bt) & 15) == 0) &&
         N < (int64_t(1) << 31) && M < (int64_t(1) << 31) && K < (int64_t(1) << 31) &&
         ceil_div64(M, dt::kSdU) * ceil_div64(N, 128) < (int64_t(1) << 31);
}

// Launches the dense-tile SDDMM over the eligible problems (units of row blocks the cost
// model leaves to the gather kernel exit at once on the device).
cudaError_t launch_sddmm_dense(int64_t count, const int64_t* M, const int64_t* N, const int64_t* K,
                               const int* V, const int32_t* const* row_ptr, const int32_t* const* col_idx,
                               const void* const* A, const void* const* Bt, void* const* out, int num_sms,
                               cudaStream_t s) {
  using namespace dt;
  SdBatch batch;
  batch.count = 0;
  batch.first_unit[0] = 0;
  auto flush = [&]() -> cudaError_t {
    if (batch.count == 0) return cudaSuccess;
    const cudaError_t e = launch_sd(batch, num_sms, s);
    batch.count = 0;
    batch.first_unit[0] = 0;
    return e;
  };
  for (int64_t i = 0; i < count; ++i) {
    if (!sddmm_dense_eligible(M[i], N[i], K[i], V[i], A[i], Bt[i])) continue;
    if (batch.first_unit[batch.count] + ceil_div64(M[i], dt::kSdU) * ceil_div64(N[i], 128) >= (int64_t(1) << 31)) {
      const cudaError_t e = flush();  // one launch's grid stays below 2^31 CTAs
      if (e != cudaSuccess) return e;
    }
    SdDesc& d = batch.d[batch.count];
    if (!make_kmajor_map(&d.tmA, A[i], M[i], K[i], kSdU) || !make_kmajor_map(&d.tmBt, Bt[i], N[i], K[i], 128))
      return cudaErrorInvalidValue;
    d.M = M[i];
    d.N = N[i];
    d.K = K[i];
    d.V = V[i];
    d.W = ceil_div64(M[i], V[i]);
    d.n_ct = ceil_div64(N[i], 128);
    d.row_ptr = row_ptr[i];
    d.col_idx = col_idx[i];
    d.out = static_cast<uint16_t*>(out[i]);
    d.out_vec = (reinterpret_cast<uintptr_t>(out[i]) & (uintptr_t)(2 * V[i] - 1)) == 0 ? 1 : 0;
    d.col16 = (reinterpret_cast<uintptr_t>(col_idx[i]) & 15) == 0 ? 1 : 0;
    batch.first_unit[batch.count + 1] = batch.first_unit[batch.count] + ceil_div64(M[i], kSdU) * d.n_ct;
    ++batch.count;
    if (batch.count == kMaxProb) {
      const cudaError_t e = flush();
      if (e != cudaSuccess) return e;
    }
  }
  return flush();
}

}  // namespace vs
#endif  // VS_SDDMM_DENSE_CF > 0

#if VS_SPMM_DENSE_CF > 0  // opt-in build only (dense_select.cuh)
namespace vs {
namespace dt {

// ================================================================================ SpMM
constexpr int kSpRows = 32;            // A / C rows per unit (MMA N)
constexpr int kATile = kSpRows * 128;  // 32 rows x 64 k fp16 (4 KB)
constexpr int kSpThreads = 320;        // 10 warps
constexpr int kSpEpi = 256;            // decode / epilogue threads (warps 2-9)
constexpr int kSpKbMax = 32;           // K <= 2048: the decoded A tile stays resident
constexpr int kSpStages = 4;
constexpr int kBPanel = 64 * 128 * 2;  // B tile: 64 k x 128 n fp16 = 2 slabs of 64 n (16 KB)
constexpr int kSpSmem = kSpKbMax * kATile + kSpStages * kBPanel + 1024;
constexpr uint32_t kIdescSp = tc::idesc_f16(128, kSpRows, 1, 0);
constexpr int kMaxDst = 8;

struct alignas(64) SpDesc {
  CUtensorMap tmB;  // B [K x N] fp16 (N contiguous), box {64 n, 64 k}, SWIZZLE_128B
  int64_t M, K, N, W, n_rb;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const uint16_t* vals;
  uint16_t* C[kMaxDst];
  int64_t ldc;
  int32_t V, nC;
};
struct SpBatch {
  int count;
  int64_t first_unit[kMaxProb + 1];
  SpDesc d[kMaxProb];
};

__device__ __forceinline__ bool sp_unit_dense(const SpDesc& d, int64_t rb32) {
  return rb_is_dense(d.row_ptr, d.W, d.V, rb32 / (kDenseRows / kSpRows), ceil_div64(d.K, 64) * 64,
                     (int64_t)VS_SPMM_DENSE_CF);
}

// byte offset of element (row, k) in the decoded K-major 128-byte-swizzled A tile
__device__ __forceinline__ uint32_t adec_off(int row, int k) {
  const int kb = k >> 6, kk = k & 63, rr = row & 7;
  return (uint32_t)(kb * kATile + (row >> 3) * 1024 + rr * 128 + ((((kk >> 3) ^ rr)) << 4) + (kk & 7) * 2);
}

__global__ void __launch_bounds__(kSpThreads, 1) spmm_dense_kernel(const __grid_constant__ SpBatch b) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t full_bar[kSpStages], empty_bar[kSpStages];
  __shared__ __align__(8) uint64_t tfull_bar[2], tempty_bar[2], afull_bar, aempty_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ int32_t wptr[kSpRows + 1];
  __shared__ int32_t unsorted[kSpRows];
  const uint32_t smem = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t s_adec = smem;                          // decoded A tile (kSpKbMax x 4 KB)
  const uint32_t s_stage = smem + kSpKbMax * kATile;     // B stage ring
  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int64_t total = b.first_unit[b.count];

  if (threadIdx.x == 0) {
    for (int s = 0; s < kSpStages; ++s) {
      tc::mbar_init(smem_u32(&full_bar[s]), 1);
      tc::mbar_init(smem_u32(&empty_bar[s]), 1);
    }
    for (int a = 0; a < 2; ++a) {
      tc::mbar_init(smem_u32(&tfull_bar[a]), 1);
      tc::mbar_init(smem_u32(&tempty_bar[a]), 8);
    }
    tc::mbar_init(smem_u32(&afull_bar), 1);   // the decoders (one elected arrive)
    tc::mbar_init(smem_u32(&aempty_bar), 1);  // MMA commit after the unit's last MMA
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(
        smem_u32(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = tmem_base_sh;

  int p = 0;  // problem cursor
  auto locate = [&](int64_t u) -> int64_t {
    while (b.first_unit[p + 1] <= u) ++p;
    return u - b.first_unit[p];
  };
  if (warp == 0) {
    // ================================ TMA producer (B tiles) ================================
    uint32_t s = 0, ph = 0;
    for (int64_t u = blockIdx.x; u < total; u += gridDim.x) {
      const int64_t rb = locate(u);
      const SpDesc& d = b.d[p];
      if (!sp_unit_dense(d, rb)) continue;
      const int KB = (int)ceil_div64(d.K, 64);
      for (int64_t n0 = 0; n0 < d.N; n0 += 128) {
        for (int kb = 0; kb < KB; ++kb) {
          tc::mbar_wait(smem_u32(&empty_bar[s]), ph ^ 1);
          if (lane == 0) {
            const uint32_t st = s_stage + s * kBPanel;
            tc::mbar_expect_tx(smem_u32(&full_bar[s]), kBPanel);
            tc::tma_load_2d(st, &d.tmB, (int)n0, kb * 64, smem_u32(&full_bar[s]));
            tc::tma_load_2d(st + kBPanel / 2, &d.tmB, (int)n0 + 64, kb * 64, smem_u32(&full_bar[s]));
          }
          __syncwarp();
          if (++s == kSpStages) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ================================ MMA issuer ================================
    uint32_t s = 0, ph = 0, au = 0, tile = 0;
    for (int64_t u = blockIdx.x; u < total; u += gridDim.x) {
      const int64_t rb = locate(u);
      const SpDesc& d = b.d[p];
      if (!sp_unit_dense(d, rb)) continue;
      const int KB = (int)ceil_div64(d.K, 64);
      tc::mbar_wait(smem_u32(&afull_bar), au & 1);  // decoded A tile of this unit
      tc::fence_after();
      for (int64_t n0 = 0; n0 < d.N; n0 += 128) {
        const uint32_t acc = tile & 1;
        tc::mbar_wait(smem_u32(&tempty_bar[acc]), ((tile >> 1) & 1) ^ 1);
        tc::fence_after();
        for (int kb = 0; kb < KB; ++kb) {
          tc::mbar_wait(smem_u32(&full_bar[s]), ph);
          tc::fence_after();
          if (lane == 0) {
            const uint32_t st = s_stage + s * kBPanel;
            const uint32_t at = s_adec + kb * kATile;
#pragma unroll
            for (int k = 0; k < 4; ++k)
              tc::mma(tmem + acc * kSpRows, tc::sdesc(st + 2048 * k, kBPanel / 2, 1024),
                      tc::sdesc(at + 32 * k, 16, 1024), kIdescSp, (kb > 0 || k > 0) ? 1u : 0u);
            tc::commit(smem_u32(&empty_bar[s]));
          }
          __syncwarp();
          if (++s == kSpStages) { s = 0; ph ^= 1; }
        }
        if (lane == 0) tc::commit(smem_u32(&tfull_bar[acc]));
        __syncwarp();
        ++tile;
      }
      if (lane == 0) tc::commit(smem_u32(&aempty_bar));  // A tile free once these MMAs complete
      __syncwarp();
      ++au;
    }
  } else {
    // ================================ decode + epilogue ================================
    const int et = threadIdx.x - 64;  // 0..255
    const int q = warp & 3, h = (warp - 2) >> 2;
    uint32_t au = 0, tile = 0;
    for (int64_t u = blockIdx.x; u < total; u += gridDim.x) {
      const int64_t rb = locate(u);
      const SpDesc& d = b.d[p];
      if (!sp_unit_dense(d, rb)) continue;
      const int V = d.V;
      const int KB = (int)ceil_div64(d.K, 64);
      const int64_t i0 = rb * kSpRows;
      const int64_t w0 = i0 / V;
      const int64_t w1 = (i0 + kSpRows) / V < d.W ? (i0 + kSpRows) / V : d.W;
      const int nwin = (int)(w1 - w0);
      // ---- wait until the previous unit's MMAs released the A tile, then zero it
      tc::mbar_wait(smem_u32(&aempty_bar), (au & 1) ^ 1);
      for (int x = et; x < KB * kATile / 16; x += kSpEpi)
        asm volatile("st.shared.v4.u32 [%0], {%1,%1,%1,%1};" ::"r"(s_adec + x * 16), "r"(0) : "memory");
      if (et <= nwin) wptr[et] = __ldg(d.row_ptr + w0 + et);
      if (et < kSpRows) unsorted[et] = 0;
      tc::named_bar(1, kSpEpi);
      // ---- decode: one flat pass over the unit's vectors [P0, P1)
      const int64_t P0 = wptr[0], P1 = wptr[nwin];
      const int64_t off = (int64_t)((reinterpret_cast<uintptr_t>(d.col_idx) >> 2) & 3);
      const int64_t Pa = ((P0 + off) & ~(int64_t)3) - off;
      for (int64_t base = Pa + 4 * et; base < P1; base += 4 * kSpEpi) {
        int c4[4];
        if (base >= P0 && base + 3 < P1) {
          const int4 t = __ldg(reinterpret_cast<const int4*>(d.col_idx + base));
          c4[0] = t.x; c4[1] = t.y; c4[2] = t.z; c4[3] = t.w;
        } else {
#pragma unroll
          for (int j = 0; j < 4; ++j) c4[j] = (base + j >= P0 && base + j < P1) ? __ldg(d.col_idx + base + j) : -1;
        }
        const int64_t pf = base < P0 ? P0 : base;
        int lo = 0, hi = nwin - 1;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (wptr[mid] <= pf) lo = mid; else hi = mid - 1;
        }
        int wl = lo;
        int prev = (pf > wptr[wl] && pf < P1) ? __ldg(d.col_idx + pf - 1) : -1;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int64_t pp = base + j;
          if (pp < P0 || pp >= P1) continue;
          while (wptr[wl + 1] <= pp) { ++wl; prev = -1; }
          const int c = c4[j];
          if (c <= prev) atomicOr(&unsorted[wl], 1);
          prev = c;
          const uint16_t* src = d.vals + pp * V;
          uint16_t hv[8];
          if (V == 8) {
            const uint4 t = __ldg(reinterpret_cast<const uint4*>(src));
            hv[0] = t.x & 0xFFFF; hv[1] = t.x >> 16; hv[2] = t.y & 0xFFFF; hv[3] = t.y >> 16;
            hv[4] = t.z & 0xFFFF; hv[5] = t.z >> 16; hv[6] = t.w & 0xFFFF; hv[7] = t.w >> 16;
          } else if (V == 4) {
            const uint2 t = __ldg(reinterpret_cast<const uint2*>(src));
            hv[0] = t.x & 0xFFFF; hv[1] = t.x >> 16; hv[2] = t.y & 0xFFFF; hv[3] = t.y >> 16;
          } else {
            const uint32_t t = __ldg(reinterpret_cast<const unsigned int*>(src));
            hv[0] = t & 0xFFFF; hv[1] = t >> 16;
          }
#pragma unroll
          for (int r = 0; r < 8; ++r)
            if (r < V)
              asm volatile("st.shared.u16 [%0], %1;" ::"r"(s_adec + adec_off(wl * V + r, c)), "h"(hv[r]) : "memory");
        }
      }
      // generic-proxy stores -> visible to the tensor core (async proxy), then hand over
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      tc::named_bar(1, kSpEpi);
      if (et == 0) tc::mbar_arrive(smem_u32(&afull_bar));
      ++au;
      // ---- epilogue per 128-column panel: TMEM -> fp16 (RN) -> C rows (every destination)
      for (int64_t n0 = 0; n0 < d.N; n0 += 128) {
        const uint32_t acc = tile & 1;
        tc::mbar_wait(smem_u32(&tfull_bar[acc]), (tile >> 1) & 1);
        tc::fence_after();
        uint32_t v[16];
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
            : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
              "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
              "=r"(v[15])
            : "r"(tmem + ((uint32_t)(32 * q) << 16) + acc * kSpRows + 16 * h));
        tc::ld_wait();
        tc::fence_before();
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(smem_u32(&tempty_bar[acc]));
        const int64_t n = n0 + 32 * q + lane;
        if (n < d.N) {
#pragma unroll
          for (int x = 0; x < 16; ++x) {
            const int r = 16 * h + x;
            const int64_t i = i0 + r;
            if (i >= d.M || unsorted[r / V]) continue;
            const uint16_t hv = f_to_h(__uint_as_float(v[x]));
            for (int dd = 0; dd < d.nC; ++dd) d.C[dd][i * d.ldc + n] = hv;
          }
        }
        ++tile;
      }
    }
  }

  tc::fence_before();
  __syncthreads();
  if (warp == 1) {
    tc::fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tmem));
  }
}

static cudaError_t launch_sp(const SpBatch& b, int num_sms, cudaStream_t s) {
  static std::once_flag once[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64)
    std::call_once(once[dev], [] {
      cudaFuncSetAttribute(spmm_dense_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSpSmem);
    });
  const int64_t units = b.first_unit[b.count];
  const int grid = (int)std::min<int64_t>(num_sms, units);
  if (grid > 0) spmm_dense_kernel<<<grid, kSpThreads, kSpSmem, s>>>(b);
  return cudaGetLastError();
}

}  // namespace dt

// Problems the dense SpMM path can take at all (the per-row-block choice is made on the
// device): V >= 2, 0 < K <= 2048 (decoded A tile resident), N % 8 == 0 and 16-byte aligned B
// (TMA), vals aligned to 2V bytes (one load per vector).
bool spmm_dense_eligible(int64_t M, int64_t K, int64_t N, int V, const void* vals, const void* B) {
  return M > 0 && N > 0 && K > 0 && K <= 64 * dt::kSpKbMax && V >= 2 && N % 8 == 0 &&
         ((reinterpret_cast<uintptr_t>(B) & 15) == 0) &&
         ((reinterpret_cast<uintptr_t>(vals) & (uintptr_t)(2 * V - 1)) == 0) && N < (int64_t(1) << 31) &&
         M < (int64_t(1) << 31);
}

// dense-tile SpMM over the eligible problems; C_dst[i] holds nC[i] destinations (ldc[i])
cudaError_t launch_spmm_dense(int64_t count, const int64_t* M, const int64_t* K, const int64_t* N,
                              const int* V, const int32_t* const* row_ptr, const int32_t* const* col_idx,
                              const void* const* vals, const void* const* B, void* const* const* C_dst,
                              const int* nC, const int64_t* ldc, int num_sms, cudaStream_t s) {
  using namespace dt;
  SpBatch batch;
  batch.count = 0;
  batch.first_unit[0] = 0;
  auto flush = [&]() -> cudaError_t {
    if (batch.count == 0) return cudaSuccess;
    const cudaError_t e = launch_sp(batch, num_sms, s);
    batch.count = 0;
    batch.first_unit[0] = 0;
    return e;
  };
  for (int64_t i = 0; i < count; ++i) {
    if (!spmm_dense_eligible(M[i], K[i], N[i], V[i], vals[i], B[i]) || nC[i] < 1 || nC[i] > kMaxDst) continue;
    SpDesc& d = batch.d[batch.count];
    if (!make_mnmajor_map(&d.tmB, B[i], K[i], N[i])) return cudaErrorInvalidValue;
    d.M = M[i];
    d.K = K[i];
    d.N = N[i];
    d.V = V[i];
    d.W = ceil_div64(M[i], V[i]);
    d.n_rb = ceil_div64(M[i], kSpRows);
    d.row_ptr = row_ptr[i];
    d.col_idx = col_idx[i];
    d.vals = static_cast<const uint16_t*>(vals[i]);
    for (int k = 0; k < kMaxDst; ++k) d.C[k] = k < nC[i] ? static_cast<uint16_t*>(C_dst[i][k]) : nullptr;
    d.nC = nC[i];
    d.ldc = ldc[i];
    batch.first_unit[batch.count + 1] = batch.first_unit[batch.count] + d.n_rb;
    ++batch.count;
    if (batch.count == kMaxProb) {
      const cudaError_t e = flush();
      if (e != cudaSuccess) return e;
    }
  }
  return flush();
}

}  // namespace vs
#endif  // VS_SPMM_DENSE_CF > 0

#if VS_SDDMM_DENSE_CF > 0 || VS_SPMM_DENSE_CF > 0
namespace vs {
namespace dt {

static PFN_cuTensorMapEncodeTiled_v12000 tmap_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      p = nullptr;
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }();
  return fn;
}

// K-major fp16 [rows x K] operand, box {64, box_rows}, 128-byte swizzle, OOB -> zero
static bool make_kmajor_map(CUtensorMap* m, const void* base, int64_t rows, int64_t K, int box_rows) {
  auto enc = tmap_encoder();
  if (enc == nullptr) return false;
  cuuint64_t gdim[2] = {(cuuint64_t)K, (cuuint64_t)rows};
  cuuint64_t gstride[1] = {(cuuint64_t)K * 2};
  cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(base), gdim, gstride, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// MN-major fp16 B [K x N] (N contiguous), box {64 n, 64 k}, 128-byte swizzle, OOB -> zero
static bool make_mnmajor_map(CUtensorMap* m, const void* base, int64_t K, int64_t N) {
  auto enc = tmap_encoder();
  if (enc == nullptr) return false;
  cuuint64_t gdim[2] = {(cuuint64_t)N, (cuuint64_t)K};
  cuuint64_t gstride[1] = {(cuuint64_t)N * 2};
  cuuint32_t box[2] = {64, 64};
  cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(base), gdim, gstride, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace dt
}  // namespace vs
#endif
