// spmm_tc.cu — SpMM on the 5th-generation tensor cores fed by the column-vector gather ring
// (build-time variant: -DVS_SPMM_TC=1; spmm.cu dispatches to it for V >= 2 and 16-byte aligned
// operands, the cases of the cp.async path).
//
//   C[i][n] = sum_p vals[p*V + i%V] * B[col_idx[p]][n]   (§5)
//
// Why: the mma.sync cp.async kernel sends every gathered byte through the L1TEX / shared-memory
// pipe twice (LDGSTS fill + ldmatrix read; ncu: the L1TEX data pipe is its bound).  tcgen05
// reads its operands from shared memory on its own path, so the gathered rows cross L1TEX once.
//
// Unit = (row window w, 128-column panel n0) -- the paper's V x TileN output tile
// with the operand switch of P:858-871: MMA M = the 128 panel columns (TMEM lanes), N = V rows
// padded to 16, K = 16 stored vectors per MMA (tcgen05.mma.kind::f16, fp32 accumulate in TMEM).
//   A operand = the 16 gathered B rows of a stage, [K = 16 vectors x M = 128 columns], MN-major
//     128-byte swizzle: 64-column half h at h * 2048, 8-vector group at + (k / 8) * 1024, vector
//     row at + (k % 8) * 128, 16-byte chunk c at c ^ (k % 8)  (LBO 2048, SBO 1024; checked by
//     tools/umma_probe.cu, profiles/r01b_tcgen05.md);
//   B operand = the stage's vals, [K = 16 x N = 16], MN-major without swizzle: core matrices of
//     8 vectors x 16 B (V fp16 + zero pad), LBO 128 between vector groups, SBO 256 between
//     8-row groups (rows >= V stay zero).
// Roles (one CTA = 9 warps, several CTAs per SM): warps 0-3 gather with cp.async (each thread
// two 16-byte pieces of the stage's rows; column indices one stage ahead in registers) and
// signal a stage full kLag stages later (commit groups + wait_group, proxy fence, one arrive
// per warp); warp 4 lane 0 issues one MMA per stage and tcgen05.commit frees the stage; warps 5-8
// drain their TMEM lane quarter (32 columns x V rows) and store fp16 (RN) rows of C, to every
// destination of vs_spmm_scatter.  Two TMEM accumulators: the drain of a unit overlaps the next
// unit's gathers and MMAs.  Units are dealt round-robin over persistent CTAs in panel-major
// order (concurrent CTAs share a B panel in L2).  Every stored vector adds into its row in
// storage order, 16 at a time: deterministic, and independent of the N-panel split.
#include <algorithm>
#include <mutex>
#include <vector>

#include "common.cuh"
#include "tc_common.cuh"

#ifndef VS_SPMM_TC
#define VS_SPMM_TC 0
#endif

#if VS_SPMM_TC
namespace vs {
namespace stc {

constexpr int kStages = 8;
constexpr int kLag = 3;                    // stages between a stage's issue and its full signal
constexpr int kRowBytes = 16 * 256;        // 16 vectors x 128 columns fp16
constexpr int kValBytes = 512;             // [16 x 16] fp16 B operand (no swizzle)
// rows tiles at s * kRowBytes (1024-byte aligned: the 128-byte swizzle atoms need it), vals
// tiles after all of them
constexpr int kThreads = 288;              // warps 0-3 producers, 4 MMA, 5-8 epilogue
constexpr int kCtas = 4;                   // resident CTAs per SM
constexpr int kSmem = kStages * (kRowBytes + kValBytes) + 1024;
constexpr uint32_t kIdesc = tc::idesc_f16(128, 16, 1, 1);
constexpr int kMaxBatch = 96;
constexpr int kMaxDst = 8;

struct Desc {
  int64_t M, N, W, n_panels;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const uint16_t* vals;
  const uint16_t* B;
  uint16_t* C[kMaxDst];
  int64_t ldc;
  int32_t nC, pad;
};
struct Batch {
  int count;
  int64_t first_unit[kMaxBatch + 1];
  Desc d[kMaxBatch];
};

// unit -> problem p, window w, panel pn (panel-major inside a problem)
struct UnitIt {
  int p;
  __device__ __forceinline__ void locate(const Batch& b, int64_t u, int64_t& w, int64_t& pn) {
    while (b.first_unit[p + 1] <= u) ++p;
    const int64_t loc = u - b.first_unit[p];
    pn = loc / b.d[p].W;
    w = loc - pn * b.d[p].W;
  }
};

template <int V>
__global__ void __launch_bounds__(kThreads, kCtas) spmm_tc_kernel(const __grid_constant__ Batch b) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t full_bar[kStages], empty_bar[kStages], tfull_bar[2], tempty_bar[2];
  __shared__ uint32_t tmem_base_sh;
  const uint32_t smem = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int64_t total = b.first_unit[b.count];

  // the vals tiles' padding (rows >= V, the second 8-row group) must read as zero
  for (int s = 0; s < kStages; ++s)
    for (int x = threadIdx.x; x < kValBytes / 16; x += kThreads)
      asm volatile("st.shared.v4.u32 [%0], {%1,%1,%1,%1};" ::"r"(smem + kStages * kRowBytes + s * kValBytes + x * 16),
                   "r"(0)
                   : "memory");
  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      tc::mbar_init(smem_u32(&full_bar[s]), 4);   // one arrive per producer warp
      tc::mbar_init(smem_u32(&empty_bar[s]), 1);  // tcgen05.commit
    }
    for (int a = 0; a < 2; ++a) {
      tc::mbar_init(smem_u32(&tfull_bar[a]), 1);
      tc::mbar_init(smem_u32(&tempty_bar[a]), 4);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 4) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(
        smem_u32(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = tmem_base_sh;
  UnitIt it{0};

  if (warp < 4) {
    // ================================ producers ================================
    const int tid = threadIdx.x;  // 0..127
    // this thread's two row pieces per stage: piece i in {tid, tid + 128}: vector slot i >> 4,
    // 16-byte chunk cc = i & 15 of the 256-byte panel row (half cc >> 3, chunk cc & 7)
    const int sl0 = tid >> 4, sl1 = sl0 + 8, cc = tid & 15;
    const uint32_t off0 = (cc >> 3) * 2048 + (sl0 >> 3) * 1024 + (sl0 & 7) * 128 + (((cc & 7) ^ (sl0 & 7)) << 4);
    const uint32_t off1 = (cc >> 3) * 2048 + (sl1 >> 3) * 1024 + (sl1 & 7) * 128 + (((cc & 7) ^ (sl1 & 7)) << 4);
    uint32_t s = 0, ph = 0, issued = 0;
    for (int64_t u = blockIdx.x; u < total; u += gridDim.x) {
      int64_t w, pn;
      it.locate(b, u, w, pn);
      const Desc& d = b.d[it.p];
      const int64_t pb = d.row_ptr[w], pe = d.row_ptr[w + 1];
      const int64_t n0 = pn * 128;
      const bool col_ok = n0 + 8 * cc < d.N;
      const uint16_t* Bp = d.B + n0 + 8 * cc;
      // column indices one stage ahead
      int c0 = (pb + sl0 < pe) ? ldg32i(d.col_idx + pb + sl0) : -1;
      int c1 = (pb + sl1 < pe) ? ldg32i(d.col_idx + pb + sl1) : -1;
      for (int64_t p0 = pb; p0 < pe; p0 += 16) {
        const int64_t q0 = p0 + 16;
        const int n0c = (q0 + sl0 < pe) ? ldg32i(d.col_idx + q0 + sl0) : -1;
        const int n1c = (q0 + sl1 < pe) ? ldg32i(d.col_idx + q0 + sl1) : -1;
        tc::mbar_wait(smem_u32(&empty_bar[s]), ph ^ 1);
        const uint32_t st = smem + s * kRowBytes;
        const uint32_t sv = smem + kStages * kRowBytes + s * kValBytes;
        const bool ok0 = c0 >= 0 && col_ok, ok1 = c1 >= 0 && col_ok;
        cp_async_zfill<16>(st + off0, ok0 ? (const void*)(Bp + (int64_t)c0 * d.N) : (const void*)d.B, ok0 ? 16u : 0u);
        cp_async_zfill<16>(st + off1, ok1 ? (const void*)(Bp + (int64_t)c1 * d.N) : (const void*)d.B, ok1 ? 16u : 0u);
        if (tid < 16) {
          const int64_t p = p0 + tid;
          const bool ok = p < pe;
          cp_async_zfill<2 * V>(sv + (tid >> 3) * 128 + (tid & 7) * 16,
                                ok ? (const void*)(d.vals + p * V) : (const void*)d.vals, ok ? (uint32_t)(2 * V) : 0u);
        }
        cp_async_commit();
        // stage issued kLag stages ago is complete -> make it visible to the tensor core
        if (issued >= (uint32_t)kLag) {
          cp_async_wait<kLag>();
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          __syncwarp();
          if (lane == 0) tc::mbar_arrive(smem_u32(&full_bar[(s + kStages - kLag) % kStages]));
        }
        ++issued;
        if (++s == kStages) { s = 0; ph ^= 1; }
        c0 = n0c;
        c1 = n1c;
      }
    }
    // drain: the last min(kLag, issued) stages
    cp_async_wait<0>();
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    if (lane == 0)
      for (uint32_t i = issued > (uint32_t)kLag ? issued - kLag : 0; i < issued; ++i)
        tc::mbar_arrive(smem_u32(&full_bar[i % kStages]));
  } else if (warp == 4) {
    // ================================ MMA issuer ================================
    uint32_t s = 0, ph = 0, tile = 0;
    for (int64_t u = blockIdx.x; u < total; u += gridDim.x) {
      int64_t w, pn;
      it.locate(b, u, w, pn);
      const Desc& d = b.d[it.p];
      const int64_t pb = d.row_ptr[w], pe = d.row_ptr[w + 1];
      if (pe <= pb) continue;  // empty window: the epilogue writes zeros
      const uint32_t acc = tile & 1;
      tc::mbar_wait(smem_u32(&tempty_bar[acc]), ((tile >> 1) & 1) ^ 1);
      tc::fence_after();
      for (int64_t p0 = pb; p0 < pe; p0 += 16) {
        tc::mbar_wait(smem_u32(&full_bar[s]), ph);
        tc::fence_after();
        if (lane == 0) {
          const uint32_t st = smem + s * kRowBytes;
          const uint32_t sv = smem + kStages * kRowBytes + s * kValBytes;
          tc::mma(tmem + acc * 16, tc::sdesc(st, 2048, 1024, 2), tc::sdesc(sv, 128, 256, 0), kIdesc,
                  p0 > pb ? 1u : 0u);
          tc::commit(smem_u32(&empty_bar[s]));
        }
        __syncwarp();
        if (++s == kStages) { s = 0; ph ^= 1; }
      }
      if (lane == 0) tc::commit(smem_u32(&tfull_bar[acc]));
      __syncwarp();
      ++tile;
    }
  } else {
    // ================================ epilogue ================================
    const int q = warp & 3;  // TMEM lane quarter: panel columns 32q .. 32q + 31
    uint32_t tile = 0;
    for (int64_t u = blockIdx.x; u < total; u += gridDim.x) {
      int64_t w, pn;
      it.locate(b, u, w, pn);
      const Desc& d = b.d[it.p];
      const int64_t pb = d.row_ptr[w], pe = d.row_ptr[w + 1];
      const int64_t n = pn * 128 + 32 * q + lane;
      float f[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
      if (pe > pb) {
        const uint32_t acc = tile & 1;
        tc::mbar_wait(smem_u32(&tfull_bar[acc]), (tile >> 1) & 1);
        tc::fence_after();
        uint32_t v[8];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
                       "=r"(v[7])
                     : "r"(tmem + ((uint32_t)(32 * q) << 16) + acc * 16));
        tc::ld_wait();
        tc::fence_before();
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(smem_u32(&tempty_bar[acc]));
#pragma unroll
        for (int r = 0; r < 8; ++r) f[r] = __uint_as_float(v[r]);
        ++tile;
      }
      if (n < d.N) {
#pragma unroll
        for (int r = 0; r < V; ++r) {
          const int64_t i = w * V + r;
          if (i >= d.M) break;
          const uint16_t h = f_to_h(f[r]);
          for (int dd = 0; dd < d.nC; ++dd) d.C[dd][i * d.ldc + n] = h;
        }
      }
    }
  }

  tc::fence_before();
  __syncthreads();
  if (warp == 4) {
    tc::fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tmem));
  }
}

template <int V>
static cudaError_t launch_v(const Batch& b, int num_sms, cudaStream_t s) {
  static std::once_flag once[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64)
    std::call_once(once[dev], [] {
      cudaFuncSetAttribute(spmm_tc_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem);
    });
  const int64_t units = b.first_unit[b.count];
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * kCtas, units);
  if (grid > 0) spmm_tc_kernel<V><<<grid, kThreads, kSmem, s>>>(b);
  return cudaGetLastError();
}

}  // namespace stc

// Problems the tcgen05 SpMM takes: V >= 2, N % 8 == 0, 16-byte aligned B and vals aligned to
// 2V bytes (the cp.async pieces), K > 0.
bool spmm_tc_eligible(int64_t K, int64_t N, int V, const void* vals, const void* B) {
  return K > 0 && V >= 2 && N % 8 == 0 && ((reinterpret_cast<uintptr_t>(B) & 15) == 0) &&
         ((reinterpret_cast<uintptr_t>(vals) & (uintptr_t)(2 * V - 1)) == 0);
}

// count problems (all eligible, M, N > 0); C_dst[i]: nC[i] destinations with leading dimension ldc[i]
cudaError_t launch_spmm_tc(int64_t count, const int64_t* M, const int64_t* N, const int* V,
                           const int32_t* const* row_ptr, const int32_t* const* col_idx,
                           const void* const* vals, const void* const* B, void* const* const* C_dst,
                           const int* nC, const int64_t* ldc, int num_sms, cudaStream_t s) {
  using namespace stc;
  for (int vv : {2, 4, 8}) {
    Batch batch;
    batch.count = 0;
    batch.first_unit[0] = 0;
    auto flush = [&]() -> cudaError_t {
      if (batch.count == 0) return cudaSuccess;
      const cudaError_t e = vv == 2 ? launch_v<2>(batch, num_sms, s)
                                    : vv == 4 ? launch_v<4>(batch, num_sms, s) : launch_v<8>(batch, num_sms, s);
      batch.count = 0;
      batch.first_unit[0] = 0;
      return e;
    };
    for (int64_t i = 0; i < count; ++i) {
      if (V[i] != vv) continue;
      Desc& d = batch.d[batch.count];
      d.M = M[i];
      d.N = N[i];
      d.W = ceil_div64(M[i], vv);
      d.n_panels = ceil_div64(N[i], 128);
      d.row_ptr = row_ptr[i];
      d.col_idx = col_idx[i];
      d.vals = static_cast<const uint16_t*>(vals[i]);
      d.B = static_cast<const uint16_t*>(B[i]);
      for (int k = 0; k < kMaxDst; ++k) d.C[k] = k < nC[i] ? static_cast<uint16_t*>(C_dst[i][k]) : nullptr;
      d.nC = nC[i];
      d.pad = 0;
      d.ldc = ldc[i];
      batch.first_unit[batch.count + 1] = batch.first_unit[batch.count] + d.W * d.n_panels;
      ++batch.count;
      if (batch.count == kMaxBatch) {
        const cudaError_t e = flush();
        if (e != cudaSuccess) return e;
      }
    }
    const cudaError_t e = flush();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace vs
#endif  // VS_SPMM_TC
