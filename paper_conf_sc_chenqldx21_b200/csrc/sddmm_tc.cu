// sddmm_tc.cu — SDDMM on the 5th-generation tensor cores (tcgen05.mma, accumulators in TMEM).
//
//   out_vals[p*V + r] = sum_k A[wV+r][k] * Bt[col_idx[p]][k]   (p in window w; §6)
//
// Same operation as sddmm.cu (the mma.sync path); this is the B200-native design:
//
// * Tile = (row window w, 128 consecutive stored vectors of w).  Tiles never straddle windows,
//   so one MMA operand pair serves the whole tile: D[128 x 16] += G[128 x 16] * A_w[16 x 16]^T
//   per K-step of 16, with G the gathered Bt rows (MMA M = vectors), A_w the V rows of the
//   window (MMA N = V padded to 16; the padding columns of D are never read) and MMA K = the
//   inner dimension (the operand switch of P:1059-1063).  Both operands are K-contiguous rows,
//   so they land in shared memory in the canonical K-major 128-byte-swizzle layout with plain
//   16-byte copies (chunk c of row r at c ^ (r & 7); tools/umma_probe.cu checks the layout).
//   No cross-octet reduction, no register fragments.
// * Persistent CTA per SM, warp-specialised:
//     warps 0-3  producers: per stage (tile, 64-wide K block) 128 gathered rows x 128 B + the
//                window's V rows, cp.async 16 B per lane (8 lanes per 128-byte line), stage
//                completion signalled by cp.async.mbarrier.arrive.noinc; column indices of
//                the next tile prefetched one tile ahead;
//     warp 8     MMA issuer: one elected lane waits for a full stage, issues 4 x
//                tcgen05.mma.kind::f16 (M=128, N=16, K=16), and tcgen05.commit frees the
//                stage; the last K block of a tile commits the TMEM accumulator;
//     warps 4-7  epilogue: tcgen05.ld of their 32-lane quarter of the accumulator (one vector
//                per lane, V fp32 columns), fp16 RN conversion, one 2V-byte store per vector
//                (a warp stores 32 consecutive vectors: contiguous), rows >= M written as 0.
//   A ring of kStages stages (18 KB each) and kAcc TMEM accumulators (16 columns each) keep
//   the gather, the MMAs and the epilogue of different tiles in flight at the same time.
// * Every role walks the same deterministic tile sequence: CTA c takes the global row
//   windows c, c + G, c + 2G, ... (G = grid size) of the concatenated problems, each window's
//   128-vector tiles in order.  row_ptr is read 32 windows at a time, one window per lane.
// * Rows of a tile past the window end are never copied (their D rows are not stored);
//   K-tail chunks are zero-filled in both operands.
#include <algorithm>
#include <cstdlib>
#include <vector>

#include "common.cuh"

#ifndef VS_WITH_SDDMM_TC
#define VS_WITH_SDDMM_TC 0
#endif
#if VS_WITH_SDDMM_TC  // opt-in build only (see sddmm.cu)
namespace vs {
namespace sddmm_tc {

// VS_TC_TRACE (debug builds only): CTA 0 records globaltimer stamps of its pipeline events.
#ifdef VS_TC_TRACE
__device__ unsigned long long g_trace[3][4096];
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define TC_TRACE(role, i) \
  do { if (blockIdx.x == 0 && lane_id() == 0 && (i) < 4096) g_trace[role][(i)] = gtime(); } while (0)
#else
#define TC_TRACE(role, i) do { } while (0)
#endif

#ifndef VS_TC_STAGES
#define VS_TC_STAGES 11
#endif
constexpr int kStages = VS_TC_STAGES;
#ifndef VS_TC_CTAS
#define VS_TC_CTAS 1
#endif
constexpr int kCtasPerSm = VS_TC_CTAS;  // resident CTAs per SM (ring sized to fit)
constexpr int kRowBytes = 128 * 128;  // 128 gathered rows x 64 fp16
constexpr int kWinBytes = 16 * 128;   // 16 window rows x 64 fp16 (V used)
constexpr int kStageBytes = kRowBytes + kWinBytes;
constexpr int kAcc = 4;               // TMEM accumulators
constexpr int kTmemCols = 64;         // kAcc x 16 columns
#ifndef VS_TC_PROD
#define VS_TC_PROD 8
#endif
constexpr int kProdWarps = VS_TC_PROD;  // producer warps (4, 8 or 16)
// stage completion: 0 = cp.async.mbarrier.arrive.noinc, 1 = commit/wait_group kLag behind
#ifndef VS_TC_ARRIVE
#define VS_TC_ARRIVE 1
#endif
constexpr int kLag = 4;
constexpr int kEpiWarp0 = kProdWarps;  // epilogue warps kEpiWarp0 .. +3 (warp % 4 = TMEM quarter)
constexpr int kMmaWarp = kProdWarps + 4;
constexpr int kThreads = (kProdWarps + 5) * 32;
constexpr int kMaxBatch = 128;
constexpr int kSmemBytes = kStages * kStageBytes + 1024;  // + alignment slack

struct Desc {
  int64_t M, K, W;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const uint16_t* A;
  const uint16_t* Bt;
  uint16_t* out;
};
struct Batch {
  int count;
  int64_t first_tile[kMaxBatch + 1];  // prefix of the virtual tiles W_p * ceil(N_p / 128)
  Desc d[kMaxBatch];
};

// ---- tcgen05 / mbarrier helpers -----------------------------------------------------------
__device__ __forceinline__ uint64_t smem_desc_sw128(uint32_t saddr) {
  // K-major, 128-byte swizzle: 8-row atoms of 1024 B (SBO), LBO unused for swizzled K-major
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
// kind::f16: fp16 A and B (K-major), fp32 D, M = 128, N = 16
constexpr uint32_t kIdesc = (1u << 4) | ((16u >> 3) << 17) | ((128u >> 4) << 24);

__device__ __forceinline__ void mbar_init_cnt(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
#ifndef VS_TC_WAIT
#define VS_TC_WAIT 1
#endif
#ifndef VS_TC_SLEEP
#define VS_TC_SLEEP 128
#endif
__device__ __forceinline__ void mbar_wait_parity(uint32_t bar, uint32_t parity) {
#if VS_TC_WAIT == 1
  // non-blocking probe first (a completed phase returns at once), then the blocking form
  uint32_t done;
  asm volatile(
      "{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(done)
      : "r"(bar), "r"(parity)
      : "memory");
  if (done) return;
#endif
  asm volatile(
      "{\n.reg .pred p;\nWAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
// polite wait (epilogue side): probe, then back off with nanosleep instead of spinning on the
// barrier unit that the producers' arrives and the MMA's commits also go through
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
#if VS_TC_SLEEP > 0
  while (true) {
    uint32_t done;
    asm volatile(
        "{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
    if (done) return;
    __nanosleep(VS_TC_SLEEP);
  }
#else
  mbar_wait_parity(bar, parity);
#endif
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void cp_async_arrive_noinc(uint32_t bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tc_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar)
               : "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t dt, uint64_t ad, uint64_t bd, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(dt),
      "l"(ad), "l"(bd), "r"(kIdesc), "r"(acc)
      : "memory");
}

// ---- deterministic tile walker (one per warp; every lane holds the same current tile) ------
// Virtual tiles: problem p has VT_p = ceil(N_p / 128) possible 128-vector tiles per window (a
// window stores at most N_p vectors), numbered tile-major (t * W_p + w), concatenated over
// the problems.  CTA c takes the virtual tiles c, c + G, c + 2G, ...; a virtual tile exists
// iff row_ptr[w] + 128 t < row_ptr[w + 1].  So every SM gets work even when a problem has
// fewer windows than SMs, and the empty virtual tiles of short windows sit in a contiguous
// tail.  row_ptr is read 32 virtual tiles at a time (one per lane), one table ahead.
struct Walker {
  int64_t total;  // virtual tiles over all problems
  int64_t k0;     // sequence index of the current table's entry 0 (g = blockIdx.x + k * gridDim.x)
  int j;          // current table entry
  int lp;         // lane's problem cursor (monotonic)
  int lpc, lpn;   // lane's entry (current / next table): problem
  int64_t lwc, lwn;  //   window
  int32_t lvc, lvn, lec, len;  //   tile start, window end (lvc >= lec: no tile)
  // current tile
  bool valid;
  int p;
  int64_t w;
  int32_t v0, pe;

  __device__ __forceinline__ void load_entry(const Batch& b, int64_t k, int& ep, int64_t& ew,
                                             int32_t& ev, int32_t& ee) {
    const int64_t g = (int64_t)blockIdx.x + (k + lane_id()) * (int64_t)gridDim.x;
    ev = 1;
    ee = 0;
    if (g < total) {
      while (b.first_tile[lp + 1] <= g) ++lp;
      const int64_t loc = g - b.first_tile[lp];
      const int64_t W = b.d[lp].W;
      const int64_t t = loc / W;
      ep = lp;
      ew = loc - t * W;
      ev = b.d[lp].row_ptr[ew] + 128 * (int32_t)t;
      ee = b.d[lp].row_ptr[ew + 1];
    }
  }
  __device__ __forceinline__ void init(const Batch& b) {
    total = b.first_tile[b.count];
    k0 = 0;
    j = -1;
    lp = 0;
    lpc = lpn = 0;
    lwc = lwn = 0;
    valid = false;
    load_entry(b, 0, lpc, lwc, lvc, lec);
    load_entry(b, 32, lpn, lwn, lvn, len);
    next(b);
  }
  __device__ __forceinline__ void next(const Batch& b) {
    while (true) {
      ++j;
      if (j == 32) {
        k0 += 32;
        j = 0;
        lpc = lpn; lwc = lwn; lvc = lvn; lec = len;
        load_entry(b, k0 + 32, lpn, lwn, lvn, len);
      }
      if ((int64_t)blockIdx.x + (k0 + j) * (int64_t)gridDim.x >= total) {
        valid = false;
        return;
      }
      const int32_t tv = __shfl_sync(0xffffffffu, lvc, j);
      const int32_t te = __shfl_sync(0xffffffffu, lec, j);
      if (tv < te) {
        p = __shfl_sync(0xffffffffu, lpc, j);
        w = __shfl_sync(0xffffffffu, lwc, j);
        v0 = tv;
        pe = te;
        valid = true;
        return;
      }
    }
  }
};

template <int V>
__global__ void __launch_bounds__(kThreads, kCtasPerSm) sddmm_tc_kernel(const __grid_constant__ Batch b) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t full_bar[kStages], empty_bar[kStages];
  __shared__ __align__(8) uint64_t tfull_bar[kAcc], tempty_bar[kAcc];
  __shared__ uint32_t tmem_base_sh;
  const uint32_t smem = (smem_u32(smem_raw) + 1023u) & ~1023u;  // 1024-B aligned ring
  const int warp = threadIdx.x >> 5, lane = lane_id();

  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      // ARRIVE 0: one noinc arrive per producer thread; 1: one arrive per producer warp
      mbar_init_cnt(smem_u32(&full_bar[s]), VS_TC_ARRIVE ? kProdWarps : kProdWarps * 32);
      mbar_init_cnt(smem_u32(&empty_bar[s]), 1);   // tcgen05.commit
    }
    for (int a = 0; a < kAcc; ++a) {
      mbar_init_cnt(smem_u32(&tfull_bar[a]), 1);   // tcgen05.commit
      mbar_init_cnt(smem_u32(&tempty_bar[a]), 4);  // one arrive per epilogue warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&tmem_base_sh)), "n"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;

  Walker wk;
  wk.init(b);
  uint32_t trace_i = 0;
  (void)trace_i;

  if (warp < kProdWarps) {
    // ============================ producers ============================
    // thread: chunk c (16 B of a 128-byte row piece), row slot rs; rows rs + kRowStep * i
    const int tid = threadIdx.x;
    const int c = tid & 7, rs = tid >> 3;
    constexpr int kRowStep = kProdWarps * 4;
    constexpr int kRowsPer = 128 / kRowStep;
    const uint32_t dst0 = rs * 128 + ((c ^ (rs & 7)) << 4);  // + i * kRowStep * 128
    uint32_t s = 0, ph = 0;
    int cur[kRowsPer], nxt[kRowsPer];
    auto load_idx = [&](const Walker& t, int (&ci)[kRowsPer]) {
      const int32_t* col = b.d[t.p].col_idx;
#pragma unroll
      for (int i = 0; i < kRowsPer; ++i) {
        const int32_t v = t.v0 + rs + kRowStep * i;
        ci[i] = (t.valid && v < t.pe) ? ldg32i(col + v) : -1;
      }
    };
    load_idx(wk, nxt);
    while (wk.valid) {
      const Walker t = wk;
#pragma unroll
      for (int i = 0; i < kRowsPer; ++i) cur[i] = nxt[i];
      wk.next(b);
      load_idx(wk, nxt);  // in flight while this tile's stages are issued
      const Desc& d = b.d[t.p];
      const int64_t K = d.K;
      const uint16_t* src[kRowsPer];
#pragma unroll
      for (int i = 0; i < kRowsPer; ++i) src[i] = cur[i] >= 0 ? d.Bt + (int64_t)cur[i] * K + 8 * c : nullptr;
      const bool arow_ok = rs < V && t.w * V + rs < d.M;
      const uint16_t* asrc = arow_ok ? d.A + (t.w * V + rs) * K + 8 * c : nullptr;
      for (int64_t kb = 0; kb < K; kb += 64) {
        mbar_wait_parity(smem_u32(&empty_bar[s]), ph ^ 1);
        const uint32_t st = smem + s * kStageBytes;
        const uint32_t sz = (kb + 8 * c < K) ? 16u : 0u;  // K tail: zero fill
#pragma unroll
        for (int i = 0; i < kRowsPer; ++i)
          if (src[i] != nullptr)
            cp_async_zfill<16>(st + dst0 + i * kRowStep * 128, sz ? (const void*)(src[i] + kb) : (const void*)d.Bt, sz);
        if (rs < V && (asrc != nullptr || sz == 0))
          cp_async_zfill<16>(st + kRowBytes + dst0, (asrc != nullptr && sz) ? (const void*)(asrc + kb) : (const void*)d.A,
                             asrc != nullptr ? sz : 0u);
#if VS_TC_ARRIVE == 0
        cp_async_arrive_noinc(smem_u32(&full_bar[s]));
#else
        // own completion tracking: commit group per stage; stage i - kLag is complete once
        // at most kLag groups are pending -> proxy fence -> plain arrive
        cp_async_commit();
        if (trace_i >= (uint32_t)kLag) {
          cp_async_wait<kLag>();
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          __syncwarp();
          if (lane == 0) mbar_arrive(smem_u32(&full_bar[(s + kStages - kLag) % kStages]));
        }
#endif
        if (tid == 0) TC_TRACE(0, trace_i);
        ++trace_i;
        if (++s == kStages) { s = 0; ph ^= 1; }
      }
    }
#if VS_TC_ARRIVE != 0
    // drain: the last min(kLag, stages) stages
    cp_async_wait<0>();
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    if (lane == 0)
      for (uint32_t i = trace_i > (uint32_t)kLag ? trace_i - kLag : 0; i < trace_i; ++i)
        mbar_arrive(smem_u32(&full_bar[i % kStages]));
#endif
    cp_async_wait_all();
  } else if (warp == kMmaWarp) {
    // ============================ MMA issuer ============================
    uint32_t it = 0, tile = 0;
    while (wk.valid) {
      const int64_t K = b.d[wk.p].K;
      const int a = tile % kAcc;
      mbar_wait_parity(smem_u32(&tempty_bar[a]), ((tile / kAcc) & 1) ^ 1);
      tc_fence_after();
      const uint32_t dt = tmem + a * 16;
      for (int64_t kb = 0; kb < K; kb += 64) {
        const int s = it % kStages;
        mbar_wait_parity(smem_u32(&full_bar[s]), (it / kStages) & 1);
        TC_TRACE(1, it);
        tc_fence_after();
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (lane == 0) {
          const uint32_t st = smem + s * kStageBytes;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            tc_mma(dt, smem_desc_sw128(st + 32 * k), smem_desc_sw128(st + kRowBytes + 32 * k),
                   (kb > 0 || k > 0) ? 1u : 0u);
          tc_commit(smem_u32(&empty_bar[s]));
        }
        __syncwarp();
        ++it;
      }
      if (lane == 0) tc_commit(smem_u32(&tfull_bar[a]));
      __syncwarp();
      ++tile;
      wk.next(b);
    }
  } else {
    // ============================ epilogue ============================
    const int q = warp & 3;  // TMEM lane quarter of this warp
    uint32_t tile = 0;
    while (wk.valid) {
      const int a = tile % kAcc;
      mbar_wait_sleep(smem_u32(&tfull_bar[a]), (tile / kAcc) & 1);
      if (q == 0) TC_TRACE(2, tile);
      tc_fence_after();
      uint32_t v[8];
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
          : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
            "=r"(v[7])
          : "r"(tmem + ((uint32_t)(32 * q) << 16) + a * 16));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(smem_u32(&tempty_bar[a]));
      const Desc& d = b.d[wk.p];
      const int64_t vec = (int64_t)wk.v0 + 32 * q + lane;
      if (vec < wk.pe) {
        float f[8];
#pragma unroll
        for (int r = 0; r < 8; ++r) f[r] = (r < V && wk.w * V + r < d.M) ? __uint_as_float(v[r]) : 0.f;
        uint16_t* dst = d.out + vec * V;
        if constexpr (V == 8) {
          *reinterpret_cast<uint4*>(dst) = make_uint4(f2_to_h2(f[0], f[1]), f2_to_h2(f[2], f[3]),
                                                      f2_to_h2(f[4], f[5]), f2_to_h2(f[6], f[7]));
        } else if constexpr (V == 4) {
          *reinterpret_cast<uint2*>(dst) = make_uint2(f2_to_h2(f[0], f[1]), f2_to_h2(f[2], f[3]));
        } else if constexpr (V == 2) {
          *reinterpret_cast<uint32_t*>(dst) = f2_to_h2(f[0], f[1]);
        } else {
          *dst = f_to_h(f[0]);
        }
      }
      ++tile;
      wk.next(b);
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == kMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kTmemCols));
  }
}

template <int V>
static void launch_v(const Batch& b, int num_sms, cudaStream_t s) {
  static bool attr_done[64] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(dev >= 0 && dev < 64 && attr_done[dev])) {
    cudaFuncSetAttribute(sddmm_tc_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
    if (dev >= 0 && dev < 64) attr_done[dev] = true;
  }
  const int64_t tiles = b.first_tile[b.count];
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * kCtasPerSm, tiles);
  if (grid > 0) sddmm_tc_kernel<V><<<grid, kThreads, kSmemBytes, s>>>(b);
}

}  // namespace sddmm_tc

#ifdef VS_TC_TRACE
extern "C" int vs_debug_tc_trace(unsigned long long* host_out) {
  return (int)cudaMemcpyFromSymbol(host_out, sddmm_tc::g_trace, sizeof(sddmm_tc::g_trace));
}
#endif

// Problems must satisfy sddmm_tc_eligible(); grouped by V, up to kMaxBatch per launch.
bool sddmm_tc_eligible(int64_t K, const void* A, const void* Bt, const void* out) {
  return K > 0 && K % 8 == 0 && (reinterpret_cast<uintptr_t>(A) & 15) == 0 &&
         (reinterpret_cast<uintptr_t>(Bt) & 15) == 0 && (reinterpret_cast<uintptr_t>(out) & 15) == 0;
}

cudaError_t launch_sddmm_tc_batched(int64_t count, const int64_t* M, const int64_t* N, const int64_t* K, const int* V,
                                    const int32_t* const* row_ptr, const int32_t* const* col_idx,
                                    const void* const* A, const void* const* Bt, void* const* out,
                                    int num_sms, cudaStream_t s) {
  using namespace sddmm_tc;
  for (int vv : {1, 2, 4, 8}) {
    Batch batch;
    batch.count = 0;
    batch.first_tile[0] = 0;
    auto flush = [&]() {
      if (batch.count == 0) return;
      switch (vv) {
        case 1: launch_v<1>(batch, num_sms, s); break;
        case 2: launch_v<2>(batch, num_sms, s); break;
        case 4: launch_v<4>(batch, num_sms, s); break;
        default: launch_v<8>(batch, num_sms, s); break;
      }
      batch.count = 0;
    };
    for (int64_t i = 0; i < count; ++i) {
      if (V[i] != vv) continue;
      Desc& d = batch.d[batch.count];
      const int64_t W = ceil_div64(M[i], vv);
      d = {M[i], K[i], W, row_ptr[i], col_idx[i], static_cast<const uint16_t*>(A[i]),
           static_cast<const uint16_t*>(Bt[i]), static_cast<uint16_t*>(out[i])};
      batch.first_tile[batch.count + 1] = batch.first_tile[batch.count] + W * ceil_div64(N[i], 128);
      ++batch.count;
      if (batch.count == kMaxBatch) {
        flush();
        batch.first_tile[0] = 0;
      }
    }
    flush();
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace vs
#endif  // VS_WITH_SDDMM_TC
