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
//   non-persistent (4 resident per SM, so one CTA's loads overlap another's MMAs / epilogue).
//   D[128 mask cols x 128 A rows] (fp32, TMEM, 128 columns) = Bt[c0:c0+128, :] * A[r0:r0+128, :]^T
//   with tcgen05.mma M = 128, N = 128, K = 16 (the operand switch of P:1059-1063: mask columns on
//   the MMA M side), both operands K-contiguous rows loaded by TMA 2-D tile copies (SWIZZLE_128B
//   = the canonical K-major layout), a ring of 64-wide K slabs (any inner K; one stage, 4 CTAs per SM).  Warp 0
//   lane 0 issues the TMA copies, warp 1 lane 0 the MMAs; then every warp drains its TMEM lane
//   quarter (thread = mask column c) into a shared tile Tt[c][r] (fp16 RN, rows >= M are +0;
//   each c a 256-byte row, 16-byte chunks XOR-swizzled by c), so the V rows of a window at
//   column c are 2V contiguous bytes.  While the TMA / MMA run, warps 2-3 find per window the
//   range [lo, hi) of its vectors whose column falls in the tile (9-ary search on the ascending
//   col_idx); the store pass (warp j: windows j, j+4, ...; lanes = consecutive vectors) gives
//   each of them one 2V-byte shared load and one 2V-byte global store.  A window that is not
//   strictly ascending is recomputed afterwards by the gather kernel (sddmm.cu).
//
// SpMM  C[i][n] = sum_p vals[p*V + i%V] * B[col_idx[p]][n]   (§5)  [opt-in build]
//   Unit = (problem, 128-row block of A / C), K <= 512: the block's stored vectors are decoded
//   into a dense K-major [128 x K] fp16 tile in shared memory (windows that are not strictly
//   ascending are flagged and left to the gather kernel), then per panel of <= 256 columns
//   tcgen05.mma M = 128 rows x N = panel with B MN-major from TMA, epilogue to every
//   vs_spmm_scatter destination (details at spmm_dense_kernel).

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
constexpr int kSdThreads = 128;              // 4 warps = the 4 TMEM lane quarters
constexpr int kSdSlab = 128 * 128;           // bytes: 128 rows x 64 k fp16 (16 KB)
constexpr int kSdStage = 2 * kSdSlab;        // Bt slab + A slab
// Ring depth, chosen per launch from the launch's largest K (two instantiations): problems with
// K <= 256 (<= 4 slabs) one stage, 4 CTAs per SM (TMEM: 4 x 128 columns) -- they hide the serial
// slab round trips better than 2 stages at 3 CTAs per SM (DLMC step 0.830 -> 0.824 ms); longer K
// (e.g. the ResNet-50 layers' 3136) three stages at 2 CTAs per SM, so slabs stream instead of one
// round trip each (profiles/r03_dense_sddmm.md).
constexpr int kSdStagesShort = 1;
constexpr int kSdStagesLong = 3;
constexpr int kSdShortKB = 4;  // slabs a one-stage launch takes (K <= 256)
template <int S>
struct SdCfg {
  static constexpr int kSmem = S * kSdStage + 1024;  // + 1024-byte alignment slack (SWIZZLE_128B)
  static constexpr int kCtasPerSm = S == 1 ? 4 : (S == 2 ? 3 : 2);
};
static_assert(128 * 256 <= kSdStagesShort * kSdStage, "Tt tile reuses the stage ring");  // 32 KB
constexpr uint32_t kIdescSd = tc::idesc_f16(128, 128, 0, 0);

struct alignas(64) SdDesc {
  CUtensorMap tmA;   // A [M x K] fp16, box {64, 128}, SWIZZLE_128B
  CUtensorMap tmBt;  // Bt [N x K] fp16, box {64, 128}, SWIZZLE_128B
  int64_t M, N, K, W, n_ct;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  uint16_t* out;
  int32_t V, out_vec;  // out_vec: out is 2V-byte aligned
};
struct SdBatch {
  int count;
  int64_t first_unit[kMaxProb + 1];
  SdDesc d[kMaxProb];
};

template <int V>
__device__ __forceinline__ void sd_sample_store(uint32_t a, uint16_t* dst, bool vec) {
  if (V == 8) {
    const uint4 t = lds128_u32(a);
    if (vec) {
      *reinterpret_cast<uint4*>(dst) = t;
    } else {
      const uint32_t w[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
      for (int r = 0; r < 8; ++r) dst[r] = (uint16_t)(w[r >> 1] >> (16 * (r & 1)));
    }
  } else if (V == 4) {
    uint32_t x, y;
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(x), "=r"(y) : "r"(a));
    if (vec) {
      *reinterpret_cast<uint2*>(dst) = make_uint2(x, y);
    } else {
      dst[0] = (uint16_t)x; dst[1] = (uint16_t)(x >> 16); dst[2] = (uint16_t)y; dst[3] = (uint16_t)(y >> 16);
    }
  } else if (V == 2) {
    uint32_t x;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(x) : "r"(a));
    if (vec) {
      *reinterpret_cast<uint32_t*>(dst) = x;
    } else {
      dst[0] = (uint16_t)x; dst[1] = (uint16_t)(x >> 16);
    }
  } else {
    dst[0] = lds16(a);
  }
}

// Smallest i in [lo, hi] with a[i] >= x, for two targets at once (a[lo, hi) ascending, a[hi]
// taken as +inf): 9-ary search, 8 independent probes per target per round trip.  The first
// round is placed around a guess of each answer (g1, g2: where x would sit if the window's
// columns were spread evenly), 8 probes dd apart with dd ~ sqrt(n) / 4, so on a random mask it
// brackets the answer to dd entries and one more round of <= 8 loads finishes: ~2 L2 round
// trips instead of ~4 for a 1024-entry window.  Any placement of the probes keeps the search
// exact (it counts the probes below x).  On a window that is not ascending the result is some
// index in [lo, hi].
__device__ __forceinline__ void kary_lower_bound2(const int32_t* __restrict__ a, int lo, int hi, int x1, int x2,
                                                  int g1, int g2, int& r1, int& r2) {
  int l1 = lo, h1 = hi, l2 = lo, h2 = hi;
  const int n = hi - lo;
  int dd = (int)(sqrtf((float)n) * 0.25f);
  dd = dd < 1 ? 1 : dd;
  if (8 * dd <= n && n > 16) {  // guided first round: probes base + dd * i, i = 1..8, inside [lo, hi)
    auto place = [&](int g) {
      int base = g - 4 * dd;
      base = base < lo - 1 ? lo - 1 : base;
      base = base > hi - 1 - 8 * dd ? hi - 1 - 8 * dd : base;
      return base;
    };
    const int b1 = place(g1), b2 = place(g2);
    int c1 = 0, c2 = 0;
#pragma unroll
    for (int i = 1; i <= 8; ++i) {
      c1 += __ldg(a + b1 + dd * i) < x1 ? 1 : 0;
      c2 += __ldg(a + b2 + dd * i) < x2 ? 1 : 0;
    }
    const int nh1 = c1 < 8 ? b1 + dd * (c1 + 1) : h1;
    l1 = c1 > 0 ? b1 + dd * c1 + 1 : l1;
    h1 = nh1;
    const int nh2 = c2 < 8 ? b2 + dd * (c2 + 1) : h2;
    l2 = c2 > 0 ? b2 + dd * c2 + 1 : l2;
    h2 = nh2;
  }
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

// Store pass of one unit: warp j takes windows j, j + 4, ... of the block, four windows per
// round with their first 64 vectors' col_idx loads in flight together (lane = vector: coalesced
// loads, 2V-byte shared load + 2V-byte global store each); the window's vectors in the tile's
// column range are [lo, hi) (searched before the drain).  A vector whose column is outside the
// range (possible only in a window that is not ascending) is not stored.
template <int V>
__device__ __forceinline__ void sd_store1(const SdDesc& d, uint32_t tt, uint32_t rofs, int e, int col, int c0,
                                          bool vec) {
  const uint32_t c = (uint32_t)(col - c0);
  if (col >= 0 && c < 128u)
    sd_sample_store<V>(tt + c * 256 + (((rofs >> 3) ^ (c & 15)) << 4) + (rofs & 7) * 2, d.out + (int64_t)e * V, vec);
}
template <int V>
__device__ __forceinline__ void sd_store(const SdDesc& d, uint32_t tt, const int32_t* lo_s, const int32_t* hi_s,
                                         int nwin, int c0, int warp, int lane) {
  const bool vec = d.out_vec != 0;
  const int32_t* __restrict__ ci = d.col_idx;
  for (int wb = warp; wb < nwin; wb += 16) {
    int lo[4], hi[4], ca[4], cb[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int wl = wb + 4 * u;
      lo[u] = wl < nwin ? lo_s[wl] : 0;
      hi[u] = wl < nwin ? hi_s[wl] : 0;
    }
    // an ascending window has at most 128 vectors in the tile: four 32-vector chunks per window,
    // all sixteen loads of the round in flight together
    int cc[4][2];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      ca[u] = lo[u] + lane < hi[u] ? __ldg(ci + lo[u] + lane) : -1;
      cb[u] = lo[u] + 32 + lane < hi[u] ? __ldg(ci + lo[u] + 32 + lane) : -1;
#pragma unroll
      for (int q = 0; q < 2; ++q)
        cc[u][q] = lo[u] + 64 + 32 * q + lane < hi[u] ? __ldg(ci + lo[u] + 64 + 32 * q + lane) : -1;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t rofs = (uint32_t)((wb + 4 * u) * V);
      sd_store1<V>(d, tt, rofs, lo[u] + lane, ca[u], c0, vec);
      sd_store1<V>(d, tt, rofs, lo[u] + 32 + lane, cb[u], c0, vec);
#pragma unroll
      for (int q = 0; q < 2; ++q) sd_store1<V>(d, tt, rofs, lo[u] + 64 + 32 * q + lane, cc[u][q], c0, vec);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {  // past 128 vectors: only a window that is not ascending
      const uint32_t rofs = (uint32_t)((wb + 4 * u) * V);
      for (int e0 = lo[u] + 128; e0 < hi[u]; e0 += 64) {
        const int e1 = e0 + lane, e2 = e0 + 32 + lane;
        const int c1 = e1 < hi[u] ? __ldg(ci + e1) : -1;
        const int c2 = e2 < hi[u] ? __ldg(ci + e2) : -1;
        sd_store1<V>(d, tt, rofs, e1, c1, c0, vec);
        sd_store1<V>(d, tt, rofs, e2, c2, c0, vec);
      }
    }
  }
}

// Phase timing of the dense SDDMM CTAs (tuning builds only, -DVS_SD_TIMING=1): clock64 at the
// phase boundaries of the first kSdTimed CTAs of a launch, read back with vs_debug_sd_timing.
#ifndef VS_SD_TIMING
#define VS_SD_TIMING 0
#endif
#if VS_SD_TIMING
constexpr int kSdTimed = 8192;
__device__ unsigned long long g_sd_t[kSdTimed][8];
#define SD_T(slot) do { if (blockIdx.x < kSdTimed) g_sd_t[blockIdx.x][slot] = clock64(); } while (0)
#else
#define SD_T(slot) do { } while (0)
#endif

template <int kSdStages>
__global__ void __launch_bounds__(kSdThreads, SdCfg<kSdStages>::kCtasPerSm)
    sddmm_dense_kernel(const __grid_constant__ SdBatch b) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t full_bar[kSdStages], empty_bar[kSdStages], done_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ int32_t lo_s[128], hi_s[128];  // per window: its vectors in the tile's column range
  __shared__ int32_t wptr[129];              // row_ptr of the block's windows
  pdl_launch_dependents();  // the gather kernel that follows may start at once (sddmm.cu)
  if (threadIdx.x == 0) SD_T(0);
  const int64_t u = blockIdx.x;
  const int p = first_problem(b.first_unit, b.count, u);
  const SdDesc& d = b.d[p];
  const int loc = (int)(u - b.first_unit[p]);  // < 2^31: units = ceil(M/128) * ceil(N/128), both < 2^24
  const int n_ct = (int)d.n_ct;
  const int rb = loc / n_ct, ct = loc - rb * n_ct;
  const int64_t w0 = rb * (128 / d.V);
  const int nwin = (int)((w0 + 128 / d.V < d.W ? w0 + 128 / d.V : d.W) - w0);
  // one round trip: the block's window pointers (the dense / gather decision and the searches)
  for (int i = threadIdx.x; i <= nwin; i += kSdThreads) wptr[i] = __ldg(d.row_ptr + w0 + i);
  __syncthreads();
  // CTA-uniform: a row block of the gather kernel (the predicate of sddmm_rb_dense)
  if ((int64_t)(wptr[nwin] - wptr[0]) * (int64_t)VS_SDDMM_DENSE_CF <= (int64_t)kDenseRows * (n_ct * 128)) return;
  if (threadIdx.x == 0) SD_T(1);

  const uint32_t smem = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const int warp = threadIdx.x >> 5, lane = lane_id();
  if (threadIdx.x == 0) {
    for (int s = 0; s < kSdStages; ++s) {
      tc::mbar_init(smem_u32(&full_bar[s]), 1);
      tc::mbar_init(smem_u32(&empty_bar[s]), 1);
    }
    tc::mbar_init(smem_u32(&done_bar), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(
        smem_u32(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = tmem_base_sh;
  const int KB = (int)ceil_div64(d.K, 64);
  const int r0 = (int)(rb * 128), c0 = (int)(ct * 128);
  if (threadIdx.x == 0) SD_T(2);

  if (warp == 0) {
    // ---- TMA producer: slab kb -> stage kb % kSdStages (Bt slab, then A slab)
    if (lane == 0) {
      for (int kb = 0; kb < KB; ++kb) {
        const int s = kb % kSdStages, use = kb / kSdStages;
        if (use > 0) tc::mbar_wait(smem_u32(&empty_bar[s]), (use - 1) & 1);
        const uint32_t st = smem + s * kSdStage;
        tc::mbar_expect_tx(smem_u32(&full_bar[s]), kSdStage);
        tc::tma_load_2d(st, &d.tmBt, kb * 64, c0, smem_u32(&full_bar[s]));
        tc::tma_load_2d(st + kSdSlab, &d.tmA, kb * 64, r0, smem_u32(&full_bar[s]));
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ---- MMA issuer
    if (lane == 0) {
      for (int kb = 0; kb < KB; ++kb) {
        const int s = kb % kSdStages, use = kb / kSdStages;
        tc::mbar_wait(smem_u32(&full_bar[s]), use & 1);
        tc::fence_after();
        const uint32_t st = smem + s * kSdStage;
#pragma unroll
        for (int k = 0; k < 4; ++k)
          tc::mma(tmem, tc::sdesc(st + 32 * k, 16, 1024), tc::sdesc(st + kSdSlab + 32 * k, 16, 1024), kIdescSd,
                  (kb > 0 || k > 0) ? 1u : 0u);
        tc::commit(smem_u32(&empty_bar[s]));
      }
      tc::commit(smem_u32(&done_bar));
    }
    __syncwarp();
  } else {
    // ---- warps 2-3, while the TMA / MMA run: per window (thread = window), its vectors with a
    // column in [c0, c0 + 128) are the range [lo, hi) of its (ascending) col_idx
    for (int i = threadIdx.x - 64; i < nwin; i += kSdThreads - 64) {
      const int pb = wptr[i], pe = wptr[i + 1];
      const int64_t nn = pe - pb;
      int lo, hi;
      kary_lower_bound2(d.col_idx, pb, pe, c0, c0 + 128, pb + (int)(nn * c0 / d.N),
                        pb + (int)(nn * (c0 + 128) / d.N), lo, hi);
      lo_s[i] = lo;
      hi_s[i] = hi > lo ? hi : lo;
    }
    if (threadIdx.x == 64) SD_T(3);
  }

  // ---- drain: thread = mask column c = TMEM lane 32 * warp + lane; Tt[c][r] fp16 over the ring
  tc::mbar_wait(smem_u32(&done_bar), 0);
  tc::fence_after();
  if (threadIdx.x == 0) SD_T(4);
  const int c = 32 * warp + lane;
  const uint32_t trow = smem + (uint32_t)c * 256;
  const int64_t rows_valid = d.M - r0;  // rows >= M are stored as +0
#pragma unroll 1
  for (int j = 0; j < 4; ++j) {
    uint32_t v[32];
    tc::ld32(tmem + ((uint32_t)(32 * warp) << 16) + 32 * j, v);
    tc::ld_wait();
    uint32_t h[16];
#pragma unroll
    for (int x = 0; x < 16; ++x) {
      const int r = 32 * j + 2 * x;
      const float f0 = r < rows_valid ? __uint_as_float(v[2 * x]) : 0.f;
      const float f1 = r + 1 < rows_valid ? __uint_as_float(v[2 * x + 1]) : 0.f;
      h[x] = f2_to_h2(f0, f1);
    }
#pragma unroll
    for (int m = 0; m < 4; ++m)
      asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(trow + ((((uint32_t)(4 * j + m)) ^ (c & 15)) << 4)),
                   "r"(h[4 * m]), "r"(h[4 * m + 1]), "r"(h[4 * m + 2]), "r"(h[4 * m + 3])
                   : "memory");
  }
  tc::fence_before();
  __syncthreads();  // Tt complete, TMEM drained
  if (threadIdx.x == 0) SD_T(5);
  if (warp == 0) {
    tc::fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
  }
  switch (d.V) {
    case 1: sd_store<1>(d, smem, lo_s, hi_s, nwin, c0, warp, lane); break;
    case 2: sd_store<2>(d, smem, lo_s, hi_s, nwin, c0, warp, lane); break;
    case 4: sd_store<4>(d, smem, lo_s, hi_s, nwin, c0, warp, lane); break;
    default: sd_store<8>(d, smem, lo_s, hi_s, nwin, c0, warp, lane); break;
  }
#if VS_SD_TIMING
  __syncthreads();
  if (threadIdx.x == 0) SD_T(6);
#endif
}

template <int S>
static void launch_sd_s(const SdBatch& b, int64_t units, cudaStream_t s) {
  static std::once_flag once[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64)
    std::call_once(once[dev], [] {
      cudaFuncSetAttribute(sddmm_dense_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, SdCfg<S>::kSmem);
    });
  sddmm_dense_kernel<S><<<(unsigned)units, kSdThreads, SdCfg<S>::kSmem, s>>>(b);
}

static cudaError_t launch_sd(const SdBatch& b, cudaStream_t s) {
  const int64_t units = b.first_unit[b.count];
  if (units <= 0) return cudaSuccess;
  int64_t kb_max = 0;
  for (int i = 0; i < b.count; ++i) kb_max = std::max<int64_t>(kb_max, ceil_div64(b.d[i].K, 64));
  if (kb_max <= kSdShortKB) launch_sd_s<kSdStagesShort>(b, units, s);
  else launch_sd_s<kSdStagesLong>(b, units, s);
  return cudaGetLastError();
}

}  // namespace dt

#if VS_SD_TIMING
// tuning builds only: copies the phase clocks of the last dense SDDMM launch (n CTAs x 8)
extern "C" int vs_debug_sd_timing(void* host, int n) {
  if (n > dt::kSdTimed) n = dt::kSdTimed;
  return (int)cudaMemcpyFromSymbol(host, dt::g_sd_t, (size_t)n * 8 * sizeof(unsigned long long));
}
#endif

// Problems the dense SDDMM path can take at all (the per-row-block choice is made on the
// device): 0 < K with K % 8 == 0 (16-byte TMA row stride), 16-byte aligned A and Bt, row and
// column counts that fit the int32 TMA coordinates.
bool sddmm_dense_eligible(int64_t M, int64_t N, int64_t K, int V, const void* A, const void* Bt) {
  return M > 0 && N > 0 && K >= VS_SDDMM_DENSE_KMIN && K > 0 && V >= 1 && V <= 8 && K % 8 == 0 &&
         ((reinterpret_cast<uintptr_t>(A) & 15) == 0) && ((reinterpret_cast<uintptr_t>(Bt) & 15) == 0) &&
         N < (int64_t(1) << 31) && M < (int64_t(1) << 31) && K < (int64_t(1) << 31) &&
         ceil_div64(M, 128) * ceil_div64(N, 128) < (int64_t(1) << 31);
}

// Launches the dense-tile SDDMM over the eligible problems (units of row blocks the cost
// model leaves to the gather kernel exit at once on the device).
cudaError_t launch_sddmm_dense(int64_t count, const int64_t* M, const int64_t* N, const int64_t* K,
                               const int* V, const int32_t* const* row_ptr, const int32_t* const* col_idx,
                               const void* const* A, const void* const* Bt, void* const* out, int num_sms,
                               cudaStream_t s) {
  using namespace dt;
  (void)num_sms;
  SdBatch batch;
  batch.count = 0;
  batch.first_unit[0] = 0;
  auto flush = [&]() -> cudaError_t {
    if (batch.count == 0) return cudaSuccess;
    const cudaError_t e = launch_sd(batch, s);
    batch.count = 0;
    batch.first_unit[0] = 0;
    return e;
  };
  for (int64_t i = 0; i < count; ++i) {
    if (!sddmm_dense_eligible(M[i], N[i], K[i], V[i], A[i], Bt[i])) continue;
    if (batch.first_unit[batch.count] + ceil_div64(M[i], 128) * ceil_div64(N[i], 128) >= (int64_t(1) << 31)) {
      const cudaError_t e = flush();  // one launch's grid stays below 2^31 CTAs
      if (e != cudaSuccess) return e;
    }
    SdDesc& d = batch.d[batch.count];
    if (!make_kmajor_map(&d.tmA, A[i], M[i], K[i], 128) || !make_kmajor_map(&d.tmBt, Bt[i], N[i], K[i], 128))
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
    batch.first_unit[batch.count + 1] = batch.first_unit[batch.count] + ceil_div64(M[i], 128) * d.n_ct;
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

#if VS_SPMM_DENSE_CF > 0
namespace vs {
namespace dt {

// ================================================================================ SpMM
// Unit = (problem, 128-row block): one CTA of 8 warps, one per SM (193 KB of shared memory).
//  1. decode: the block's stored vectors [P0, P1) (contiguous in col_idx: the windows of the
//     block) are streamed by all 256 threads (coalesced col_idx / vals loads, a per-thread window
//     cursor over the block's row_ptr) and scattered into a zeroed dense A tile [128 rows x K]
//     in shared memory, K-major SWIZZLE_128B (K <= 512: the tile stays resident); a window whose
//     col_idx is not strictly ascending is flagged (the gather kernel computes it: duplicates
//     sum there, spmm_skip_window);
//  2. per N panel of <= 256 columns: D[128 rows x Np] (fp32, TMEM) = A tile * B panel with
//     tcgen05.mma M = 128, N = Np, K = 16, B MN-major straight from TMA boxes {64 n, 64 k}
//     (2-stage ring), warp 0 lane 0 issuing the copies, warp 1 lane 0 the MMAs;
//  3. epilogue: warp w drains TMEM lane quarter w % 4 (thread = row), column half w / 4, fp16
//     (RN), 16-byte stores of the row into every destination (vs_spmm_scatter), rows >= M and
//     rows of flagged windows skipped.
constexpr int kSpU = 128;
constexpr int kSpKMax = 512;
constexpr int kSpASlab = kSpU * 128;        // 128 rows x 64 k fp16 (16 KB)
constexpr int kSpNP = 256;                  // N panel (MMA N, TMEM columns)
constexpr int kSpBBox = 64 * 128;           // one TMA box: 64 k x 64 n fp16 (8 KB)
constexpr int kSpBStage = (kSpNP / 64) * kSpBBox;
constexpr int kSpStages = 2;
constexpr int kSpThreads = 256;
constexpr int kSpSmem = (kSpKMax / 64) * kSpASlab + kSpStages * kSpBStage + 1024;
constexpr int kMaxDst = 8;
constexpr int kSpUnroll = 4;

struct alignas(64) SpDesc {
  CUtensorMap tmB;  // B [K x N] fp16 (N contiguous), box {64 n, 64 k}, SWIZZLE_128B
  int64_t M, K, N, W;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const uint16_t* vals;
  uint16_t* C[kMaxDst];
  int64_t ldc;
  int32_t V, nC, c16, in16;  // c16: every destination and ldc * 2 bytes 16-byte aligned;
                              // in16: col_idx and vals 16-byte aligned
};
struct SpBatch {
  int count;
  int64_t first_unit[kMaxProb + 1];
  SpDesc d[kMaxProb];
};

// byte offset of element (row, k) in the decoded K-major 128-byte-swizzled A tile
__device__ __forceinline__ uint32_t sp_adec(int row, int k) {
  const int kk = k & 63, rr = row & 7;
  return (uint32_t)((k >> 6) * kSpASlab + (row >> 3) * 1024 + rr * 128 + ((((kk >> 3) ^ rr)) << 4) + (kk & 7) * 2);
}

template <int V>
__device__ __forceinline__ void sp_decode(const SpDesc& d, uint32_t atile, const int32_t* wptr, int nwin,
                                          int rows_valid, int* uns) {
  const int P0 = wptr[0], P1 = wptr[nwin];
  int wl = -1, wend = P0;
  for (int base = P0 + (int)threadIdx.x; base < P1; base += kSpThreads * kSpUnroll) {
    int col[kSpUnroll], prev[kSpUnroll];
    uint16_t hv[kSpUnroll][V];
#pragma unroll
    for (int u = 0; u < kSpUnroll; ++u) {
      const int e = base + kSpThreads * u;
      col[u] = e < P1 ? __ldg(d.col_idx + e) : -1;
      prev[u] = (e < P1 && e > P0) ? __ldg(d.col_idx + e - 1) : -1;
      const uint16_t* src = d.vals + (int64_t)e * V;
      if (V == 8) {
        const uint4 t = e < P1 ? __ldg(reinterpret_cast<const uint4*>(src)) : make_uint4(0, 0, 0, 0);
        const uint32_t w[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
        for (int r = 0; r < V; ++r) hv[u][r] = (uint16_t)(w[r >> 1] >> (16 * (r & 1)));
      } else if (V == 4) {
        const uint2 t = e < P1 ? __ldg(reinterpret_cast<const uint2*>(src)) : make_uint2(0, 0);
        const uint32_t w[2] = {t.x, t.y};
#pragma unroll
        for (int r = 0; r < V; ++r) hv[u][r] = (uint16_t)(w[r >> 1] >> (16 * (r & 1)));
      } else if (V == 2) {
        const uint32_t t = e < P1 ? __ldg(reinterpret_cast<const unsigned int*>(src)) : 0u;
        hv[u][0] = (uint16_t)t;
        hv[u][1] = (uint16_t)(t >> 16);
      } else {
        hv[u][0] = e < P1 ? __ldg(src) : (uint16_t)0;
      }
    }
#pragma unroll
    for (int u = 0; u < kSpUnroll; ++u) {
      const int e = base + kSpThreads * u;
      if (e >= P1) continue;
      while (wend <= e) wend = wptr[++wl + 1];
      if (e > wptr[wl] && prev[u] >= col[u]) atomicOr(&uns[wl], 1);  // not strictly ascending
#pragma unroll
      for (int r = 0; r < V; ++r) {
        const int row = wl * V + r;
        if (row < rows_valid)
          asm volatile("st.shared.u16 [%0], %1;" ::"r"(atile + sp_adec(row, col[u])), "h"(hv[u][r]) : "memory");
      }
    }
  }
}

// Decode with 16-byte loads (col_idx and vals 16-byte aligned): thread t takes the four
// consecutive vectors [e0, e0 + 4) at e0 = 4t + 1024u (+ 4096 per round) of the 16-byte groups
// covering [P0, P1), kSpUnroll groups in flight: one int4 of col_idx and V/2 uint4 of vals per
// group.  The column before a group (ascending check) is the previous lane's last one (shuffle),
// or a load for lane 0.
template <int V>
__device__ __forceinline__ void sp_decode16(const SpDesc& d, uint32_t atile, const int32_t* wptr, int nwin,
                                            int rows_valid, int* uns) {
  const int P0 = wptr[0], P1 = wptr[nwin];
  const int Pa = P0 & ~3;
  const int lane = lane_id();
  int wl = -1, wend = P0;
  constexpr int NV = (4 * V * 2 + 15) / 16;  // uint4 of vals per group (V = 1: half of one)
  for (int base = Pa + 4 * (int)threadIdx.x; base - 4 * lane < P1; base += 4 * kSpThreads * kSpUnroll) {
    int4 cv[kSpUnroll];
    uint4 vv[kSpUnroll][NV];
    int pv[kSpUnroll];
#pragma unroll
    for (int u = 0; u < kSpUnroll; ++u) {
      const int e = base + 4 * kSpThreads * u;
      const bool full = e >= P0 && e + 3 < P1;
      if (full) {
        cv[u] = __ldg(reinterpret_cast<const int4*>(d.col_idx + e));
      } else {
        cv[u] = make_int4(e >= P0 && e < P1 ? __ldg(d.col_idx + e) : -1,
                          e + 1 >= P0 && e + 1 < P1 ? __ldg(d.col_idx + e + 1) : -1,
                          e + 2 >= P0 && e + 2 < P1 ? __ldg(d.col_idx + e + 2) : -1,
                          e + 3 >= P0 && e + 3 < P1 ? __ldg(d.col_idx + e + 3) : -1);
      }
      const uint16_t* src = d.vals + (int64_t)e * V;
      if (full) {
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          if (V == 1) {
            const uint2 t = __ldg(reinterpret_cast<const uint2*>(src));
            vv[u][q] = make_uint4(t.x, t.y, 0, 0);
          } else {
            vv[u][q] = __ldg(reinterpret_cast<const uint4*>(src) + q);
          }
        }
      } else {  // a partial group: per-entry loads (no read outside [P0, P1))
        uint32_t w[4 * NV] = {};
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
          for (int r = 0; r < V; ++r)
            if (e + j >= P0 && e + j < P1)
              w[(j * V + r) >> 1] |= (uint32_t)__ldg(src + j * V + r) << (16 * ((j * V + r) & 1));
#pragma unroll
        for (int q = 0; q < NV; ++q) vv[u][q] = make_uint4(w[4 * q], w[4 * q + 1], w[4 * q + 2], w[4 * q + 3]);
      }
      const int up = __shfl_up_sync(0xffffffffu, cv[u].w, 1);
      pv[u] = lane > 0 ? up : (e > P0 && e - 1 < P1 ? __ldg(d.col_idx + e - 1) : -1);
    }
#pragma unroll
    for (int u = 0; u < kSpUnroll; ++u) {
      const int c[4] = {cv[u].x, cv[u].y, cv[u].z, cv[u].w};
      uint32_t w[4 * NV];
#pragma unroll
      for (int q = 0; q < NV; ++q) {
        w[4 * q] = vv[u][q].x; w[4 * q + 1] = vv[u][q].y; w[4 * q + 2] = vv[u][q].z; w[4 * q + 3] = vv[u][q].w;
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int e = base + 4 * kSpThreads * u + j;
        if (e < P0 || e >= P1) continue;
        while (wend <= e) wend = wptr[++wl + 1];
        const int prev = j == 0 ? pv[u] : c[j - 1];
        if (e > wptr[wl] && prev >= c[j]) atomicOr(&uns[wl], 1);  // not strictly ascending
#pragma unroll
        for (int r = 0; r < V; ++r) {
          const int row = wl * V + r;
          const int hidx = j * V + r;  // half index within the group's vals
          const uint16_t hv = (uint16_t)(w[hidx >> 1] >> (16 * (hidx & 1)));
          if (row < rows_valid)
            asm volatile("st.shared.u16 [%0], %1;" ::"r"(atile + sp_adec(row, c[j])), "h"(hv) : "memory");
        }
      }
    }
  }
}

__global__ void __launch_bounds__(kSpThreads, 1) spmm_dense_kernel(const __grid_constant__ SpBatch b) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t full_bar[kSpStages], empty_bar[kSpStages], done_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ int32_t wptr[kSpU + 1];
  __shared__ int uns[kSpU];
  pdl_launch_dependents();  // the gather launch that follows may start at once (spmm.cu)
  const int64_t u = blockIdx.x;
  const int p = first_problem(b.first_unit, b.count, u);
  const SpDesc& d = b.d[p];
  const int rb = (int)(u - b.first_unit[p]);
  const int V = d.V;
  int64_t w0, w1;
  rb_windows(rb, V, d.W, w0, w1);
  const int nwin = (int)(w1 - w0);
  for (int i = threadIdx.x; i <= nwin; i += kSpThreads) wptr[i] = __ldg(d.row_ptr + w0 + i);
  if (threadIdx.x < kSpU) uns[threadIdx.x] = 0;
  const int warp = threadIdx.x >> 5, lane = lane_id();
  if (threadIdx.x == 0) {
    for (int s = 0; s < kSpStages; ++s) {
      tc::mbar_init(smem_u32(&full_bar[s]), 1);
      tc::mbar_init(smem_u32(&empty_bar[s]), 1);
    }
    tc::mbar_init(smem_u32(&done_bar), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int KB = (int)ceil_div64(d.K, 64);
  if ((int64_t)(wptr[nwin] - wptr[0]) * (int64_t)VS_SPMM_DENSE_CF <= (int64_t)kDenseRows * (KB * 64))
    return;  // CTA-uniform: a row block of the gather kernel (spmm_skip_window)

  const uint32_t smem = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t s_a = smem, s_ring = smem + (kSpKMax / 64) * kSpASlab;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(kSpNP));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  // zero the A tile (KB slabs), then decode the block's vectors into it
  for (int x = threadIdx.x; x < KB * kSpASlab / 16; x += kSpThreads)
    asm volatile("st.shared.v4.u32 [%0], {%1,%1,%1,%1};" ::"r"(s_a + x * 16), "r"(0) : "memory");
  __syncthreads();
  const int r0 = rb * kSpU;
  const int rows_valid = (int)(d.M - r0 < kSpU ? d.M - r0 : kSpU);
  if (d.in16) {
    switch (V) {
      case 1: sp_decode16<1>(d, s_a, wptr, nwin, rows_valid, uns); break;
      case 2: sp_decode16<2>(d, s_a, wptr, nwin, rows_valid, uns); break;
      case 4: sp_decode16<4>(d, s_a, wptr, nwin, rows_valid, uns); break;
      default: sp_decode16<8>(d, s_a, wptr, nwin, rows_valid, uns); break;
    }
  } else {
    switch (V) {
      case 1: sp_decode<1>(d, s_a, wptr, nwin, rows_valid, uns); break;
      case 2: sp_decode<2>(d, s_a, wptr, nwin, rows_valid, uns); break;
      case 4: sp_decode<4>(d, s_a, wptr, nwin, rows_valid, uns); break;
      default: sp_decode<8>(d, s_a, wptr, nwin, rows_valid, uns); break;
    }
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic stores -> tensor core reads
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = tmem_base_sh;
  const int row = 32 * (warp & 3) + lane;  // epilogue: this thread's row (TMEM lane)
  const bool row_ok = row < rows_valid && uns[row / V] == 0;
  const int h = warp >> 2;                 // epilogue: column half of the panel

  uint32_t it = 0;
  int panel = 0;
  for (int64_t n0 = 0; n0 < d.N; n0 += kSpNP, ++panel) {
    const int np = (int)(d.N - n0 < kSpNP ? ceil_div64(d.N - n0, 64) * 64 : kSpNP);  // MMA N (64-multiple)
    if (warp == 0) {
      if (lane == 0) {
        uint32_t j = it;
        for (int kb = 0; kb < KB; ++kb, ++j) {
          const uint32_t s = j % kSpStages, use = j / kSpStages;
          if (use > 0) tc::mbar_wait(smem_u32(&empty_bar[s]), (use - 1) & 1);
          const uint32_t st = s_ring + s * kSpBStage;
          tc::mbar_expect_tx(smem_u32(&full_bar[s]), (uint32_t)(np / 64) * kSpBBox);
          for (int q = 0; q < np / 64; ++q)
            tc::tma_load_2d(st + q * kSpBBox, &d.tmB, (int)n0 + 64 * q, kb * 64, smem_u32(&full_bar[s]));
        }
      }
      __syncwarp();
    } else if (warp == 1) {
      if (lane == 0) {
        const uint32_t idesc = tc::idesc_f16(128, np, 0, 1);
        uint32_t j = it;
        for (int kb = 0; kb < KB; ++kb, ++j) {
          const uint32_t s = j % kSpStages, use = j / kSpStages;
          tc::mbar_wait(smem_u32(&full_bar[s]), use & 1);
          tc::fence_after();
          const uint32_t st = s_ring + s * kSpBStage;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            tc::mma(tmem, tc::sdesc(s_a + kb * kSpASlab + 32 * k, 16, 1024), tc::sdesc(st + 2048 * k, kSpBBox, 1024),
                    idesc, (kb > 0 || k > 0) ? 1u : 0u);
          tc::commit(smem_u32(&empty_bar[s]));
        }
        tc::commit(smem_u32(&done_bar));
      }
      __syncwarp();
    }
    it += KB;
    // ---- epilogue of the panel
    tc::mbar_wait(smem_u32(&done_bar), panel & 1);
    tc::fence_after();
    for (int c0 = h * (np / 2); c0 < (h + 1) * (np / 2); c0 += 32) {
      uint32_t v[32];
      tc::ld32(tmem + ((uint32_t)(32 * (warp & 3)) << 16) + c0, v);
      tc::ld_wait();
      if (!row_ok) continue;
      uint32_t hh[16];
#pragma unroll
      for (int x = 0; x < 16; ++x) hh[x] = f2_to_h2(__uint_as_float(v[2 * x]), __uint_as_float(v[2 * x + 1]));
      for (int dd = 0; dd < d.nC; ++dd) {
        uint16_t* dst = d.C[dd] + (int64_t)(r0 + row) * d.ldc + n0 + c0;
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          if (n0 + c0 + 8 * g >= d.N) break;  // N % 8 == 0
          if (d.c16) {
            *reinterpret_cast<uint4*>(dst + 8 * g) = make_uint4(hh[4 * g], hh[4 * g + 1], hh[4 * g + 2], hh[4 * g + 3]);
          } else {
#pragma unroll
            for (int x = 0; x < 4; ++x) {
              dst[8 * g + 2 * x] = (uint16_t)hh[4 * g + x];
              dst[8 * g + 2 * x + 1] = (uint16_t)(hh[4 * g + x] >> 16);
            }
          }
        }
      }
    }
    tc::fence_before();
    __syncthreads();  // TMEM drained before the next panel's MMAs
    tc::fence_after();
  }
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kSpNP));
}

static cudaError_t launch_sp(const SpBatch& b, int num_sms, cudaStream_t s) {
  (void)num_sms;
  static std::once_flag once[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64)
    std::call_once(once[dev], [] {
      cudaFuncSetAttribute(spmm_dense_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSpSmem);
    });
  const int64_t units = b.first_unit[b.count];
  if (units > 0) spmm_dense_kernel<<<(unsigned)units, kSpThreads, kSpSmem, s>>>(b);
  return cudaGetLastError();
}

}  // namespace dt

// Problems the dense SpMM path can take at all (the per-row-block choice is made on the
// device): 0 < K <= 512 (the decoded A tile stays resident), N % 8 == 0 and 16-byte aligned B
// (TMA), vals aligned to 2V bytes (one load per vector).  Independent of N's size, so every
// N-panel shard of a problem decides alike.
bool spmm_dense_eligible(int64_t M, int64_t K, int64_t N, int V, const void* vals, const void* B) {
  return M > 0 && N > 0 && K > 0 && K <= dt::kSpKMax && V >= 2 && V <= 8 && N % 8 == 0 &&
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
    d.row_ptr = row_ptr[i];
    d.col_idx = col_idx[i];
    d.vals = static_cast<const uint16_t*>(vals[i]);
    bool c16 = (ldc[i] % 8) == 0;
    for (int k = 0; k < kMaxDst; ++k) {
      d.C[k] = k < nC[i] ? static_cast<uint16_t*>(C_dst[i][k]) : nullptr;
      if (k < nC[i]) c16 = c16 && ((reinterpret_cast<uintptr_t>(C_dst[i][k]) & 15) == 0);
    }
    d.nC = nC[i];
    d.ldc = ldc[i];
    d.c16 = c16 ? 1 : 0;
    d.in16 = ((reinterpret_cast<uintptr_t>(col_idx[i]) & 15) == 0 && (reinterpret_cast<uintptr_t>(vals[i]) & 15) == 0)
                 ? 1 : 0;
    batch.first_unit[batch.count + 1] = batch.first_unit[batch.count] + ceil_div64(M[i], kSpU);
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
