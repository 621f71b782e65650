// common.cuh — small device helpers shared by the libvs kernels (sm_100a).
// Not shared with oracle/ (the oracle is independent by construction).
#pragma once

#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>

namespace vs {

constexpr int kWarp = 32;

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// 16-byte read-only global load, cached in L1 (gathered rows are re-read by other warps
// of the same SM, so we want them to stay in L1).  VS_GATHER_HINT selects a cache-policy
// variant for experiments (0: default, 1: L1::evict_last, 2: L1::no_allocate).
#ifndef VS_GATHER_HINT
#define VS_GATHER_HINT 0
#endif
__device__ __forceinline__ uint4 ldg128(const void* p) {
  uint4 r;
#if VS_GATHER_HINT == 1
  asm volatile("ld.global.nc.L1::evict_last.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
#elif VS_GATHER_HINT == 2
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
#else
  asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
#endif
  return r;
}

// 16-byte streaming load that does not allocate in L1 (A / Bt rows of SDDMM that are
// consumed once per warp).
__device__ __forceinline__ uint4 ldg128_na(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ uint16_t ldg16(const void* p) {
  unsigned short r;
  asm volatile("ld.global.nc.u16 %0, [%1];" : "=h"(r) : "l"(p));
  return r;
}

__device__ __forceinline__ int ldg32i(const int32_t* p) {
  int r;
  asm volatile("ld.global.nc.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}

__device__ __forceinline__ void stg128(void* p, uint4 v) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}

// byte permute: result bytes picked from {b:a} by selector nibbles.
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
  return r;
}
// {lo(a), lo(b)} and {hi(a), hi(b)} for two f16x2 words.
__device__ __forceinline__ uint32_t pack_lo(uint32_t a, uint32_t b) { return prmt(a, b, 0x5410); }
__device__ __forceinline__ uint32_t pack_hi(uint32_t a, uint32_t b) { return prmt(a, b, 0x7632); }

__device__ __forceinline__ uint32_t pack_h2(uint16_t lo, uint16_t hi) {
  return (uint32_t)lo | ((uint32_t)hi << 16);
}

// fp32 pair -> f16x2 (round to nearest even), lo = a.
__device__ __forceinline__ uint32_t f2_to_h2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

__device__ __forceinline__ uint16_t f_to_h(float a) {
  __half h = __float2half_rn(a);
  return *reinterpret_cast<uint16_t*>(&h);
}

// D = A(16x16, row) * B(16x8, col) + D, fp16 inputs, fp32 accumulate.
__device__ __forceinline__ void mma_16816(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2,
                                          uint32_t a3, uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 "
      "{%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// ---- mbarrier + bulk async copy (global -> shared, completion counted in bytes) ----------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// bytes must be a multiple of 16; src and dst 16-byte aligned
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
// cp.async with zero fill: copies `src_size` (0 or SZ) bytes and fills the rest of the SZ-byte
// destination with zeros (src_size = 0 -> pure zero fill, src is not read).
template <int SZ>
__device__ __forceinline__ void cp_async_zfill(uint32_t dst, const void* src, uint32_t src_size) {
  if constexpr (SZ == 16) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src),
                 "r"(src_size)
                 : "memory");
  } else {
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2, %3;" ::"r"(dst), "l"(src),
                 "n"(SZ), "r"(src_size)
                 : "memory");
  }
}
// 16-byte cp.async that allocates in L1 (.ca): gathered rows re-read by other CTAs of the SM
__device__ __forceinline__ void cp_async_ca16_zfill(uint32_t dst, const void* src, uint32_t src_size) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_size)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
// Four 8x8 b16 matrices, transposed on the way: lane L supplies the address of row (L & 7)
// of matrix (L >> 3); thread 4g+t receives {m[2t][g], m[2t+1][g]} of each matrix.
__device__ __forceinline__ void ldsm_x4_trans(uint32_t addr, uint32_t& r0, uint32_t& r1,
                                              uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
// Inverse of ldsm_x4_trans: thread 4g+t holds {m[g][2t], m[g][2t+1]} of each matrix; the
// 16-byte row at the address of lane L receives column (L & 7) of matrix (L >> 3).
__device__ __forceinline__ void stsm_x4_trans(uint32_t addr, uint32_t r0, uint32_t r1, uint32_t r2,
                                              uint32_t r3) {
  asm volatile("stmatrix.sync.aligned.m8n8.x4.trans.shared.b16 [%0], {%1,%2,%3,%4};" ::"r"(addr),
               "r"(r0), "r"(r1), "r"(r2), "r"(r3)
               : "memory");
}
__device__ __forceinline__ uint16_t lds16(uint32_t addr) {
  unsigned short r;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(r) : "r"(addr));
  return r;
}
__device__ __forceinline__ uint4 lds128_u32(uint32_t addr) {
  uint4 r;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "r"(addr));
  return r;
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.wait_all;" ::: "memory");
}
__device__ __forceinline__ uint4 lds128(const void* p) {
  uint4 r;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "r"(smem_u32(p)));
  return r;
}

// Smallest i in [0, n] with a[i] >= target (a non-decreasing, a[n] treated as +inf).
// Warp-cooperative 32-ary search; every lane returns the result.
__device__ __forceinline__ int64_t warp_lower_bound(const int32_t* __restrict__ a, int64_t n,
                                                    int64_t target) {
  int64_t lo = 0, hi = n;  // answer in [lo, hi]
  const int lane = lane_id();
  while (lo < hi) {
    const int64_t span = hi - lo;
    const int64_t step = (span + 31) / 32;
    const int64_t probe = lo + (int64_t)lane * step;
    const bool less = (probe < hi) && (a[probe] < target);
    const unsigned ballot = __ballot_sync(0xffffffffu, less);
    if (ballot == 0) return lo;  // a[lo] >= target
    const int last = 31 - __clz(ballot);  // a[lo + last*step] < target
    lo = lo + (int64_t)last * step + 1;
    const int64_t nhi = lo - 1 + step;  // probe last+1 (if any) is >= target
    if (last < 31 && nhi < hi) hi = nhi;
  }
  return lo;
}

// Last index p in [0, count) with first[p] <= x (first[] non-decreasing, first[0] = 0).
__device__ __forceinline__ int first_problem(const int64_t* first, int count, int64_t x) {
  int lo = 0, hi = count - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (first[mid] <= x) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// Programmatic dependent launch (griddepcontrol): let the next kernel of the stream start while
// this one runs / wait until the previous kernel of the stream has completed and its writes are
// visible.  Both are no-ops in a kernel launched without the PDL attribute.
__device__ __forceinline__ void pdl_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void pdl_wait_prior() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

__host__ __device__ __forceinline__ int64_t ceil_div64(int64_t a, int64_t b) {
  return (a + b - 1) / b;
}

}  // namespace vs
