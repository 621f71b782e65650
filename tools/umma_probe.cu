// umma_probe.cu — checks the tcgen05 (UMMA) operand layouts the SDDMM/SpMM tcgen05 paths use,
// on one CTA, against a host fp64 product:
//   test 1 (SDDMM): A [128 x 64] and B [16 x 64], both K-major, 128-byte swizzle; 4 MMAs
//                   M=128 N=16 K=16; D = A * B^T (fp32 in TMEM, read back with tcgen05.ld).
//   test 2 (SpMM):  A [K=16 rows x M=128] MN-major, 128-byte swizzle (atoms of 8 K-rows x 64
//                   M at LBO = 2048 B between the two M halves, SBO = 1024 B between K groups);
//                   B [K=16 x N=16] MN-major, no swizzle (core matrices of 8 K-rows x 16 B,
//                   LBO = 128 B between K groups, SBO = 256 B between N groups).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/umma_probe tools/umma_probe.cu
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <math.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;  // version (sm_100)
  d |= (uint64_t)layout << 61;
  return d;
}
// kind::f16 instruction descriptor: fp16 A/B, fp32 D
__host__ __device__ constexpr uint32_t idesc_f16(int M, int N, int a_mn, int b_mn) {
  return (1u << 4) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) | ((uint32_t)(N >> 3) << 17) |
         ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_f16(uint32_t dt, uint64_t ad, uint64_t bd, uint32_t idesc, int acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(dt),
      "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
}

__device__ bool wait_bounded(uint64_t* bar, uint32_t parity) {
  for (long i = 0; i < (1L << 26); ++i) {
    uint32_t ok;
    asm volatile(
        "{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok)
        : "r"(su32(bar)), "r"(parity)
        : "memory");
    if (ok) return true;
  }
  return false;
}

// mode 0: SDDMM layouts; mode 1: SpMM layouts. out: 128 x 16 fp32
__global__ void probe(int mode, const __half* a, const __half* b, float* out, int* status, uint32_t aL,
                      uint32_t aS, uint32_t bL, uint32_t bS) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint8_t* sa = smem;            // 16 KB
  uint8_t* sb = smem + 16384;    // 4 KB
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t tbase;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (mode == 0) {
    // A [128][64] -> row r: 128 B, chunk c at c ^ (r & 7); 8-row atoms of 1024 B consecutive
    for (int i = tid; i < 128 * 8; i += blockDim.x) {
      const int r = i >> 3, c = i & 7;
      *(uint4*)(sa + r * 128 + ((c ^ (r & 7)) << 4)) = *(const uint4*)(a + r * 64 + c * 8);
    }
    for (int i = tid; i < 16 * 8; i += blockDim.x) {
      const int r = i >> 3, c = i & 7;
      *(uint4*)(sb + r * 128 + ((c ^ (r & 7)) << 4)) = *(const uint4*)(b + r * 64 + c * 8);
    }
  } else {
    // A logical [k][m] (16 x 128, m contiguous): k-row kk, m-half h: atom at h*2048 + (kk>>3)*1024,
    // row (kk & 7) at 128 B, chunk c at c ^ (kk & 7)
    for (int i = tid; i < 16 * 16; i += blockDim.x) {
      const int kk = i >> 4, cc = i & 15, h = cc >> 3, c = cc & 7;
      *(uint4*)(sa + h * 2048 + (kk >> 3) * 1024 + (kk & 7) * 128 + ((c ^ (kk & 7)) << 4)) =
          *(const uint4*)(a + kk * 128 + cc * 8);
    }
    // B logical [k][n] (16 x 16, n contiguous): core matrix (ng, kg) at ng*256 + kg*128,
    // K row (kk & 7) at 16 B
    for (int i = tid; i < 16 * 2; i += blockDim.x) {
      const int kk = i >> 1, ng = i & 1;
      *(uint4*)(sb + ng * 256 + (kk >> 3) * 128 + (kk & 7) * 16) = *(const uint4*)(b + kk * 16 + ng * 8);
    }
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(su32(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tbase;
  if (tid == 0) {
    if (mode == 0) {
      const uint32_t id = idesc_f16(128, 16, 0, 0);
      for (int k = 0; k < 4; ++k) {
        const uint64_t ad = sdesc(su32(sa) + 32 * k, 16, 1024, 2);
        const uint64_t bd = sdesc(su32(sb) + 32 * k, 16, 1024, 2);
        mma_f16(tmem, ad, bd, id, k > 0);
      }
    } else {
      const uint32_t id = idesc_f16(128, 16, 1, 1);
      const uint64_t ad = sdesc(su32(sa), aL, aS, 2);
      const uint64_t bd = sdesc(su32(sb), bL, bS, 0);
      mma_f16(tmem, ad, bd, id, 0);
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar))
                 : "memory");
  }
  __syncwarp();
  const bool ok = wait_bounded(&bar, 0);
  if (!ok && lane == 0) atomicExch(status, 1);
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (ok) {
    uint32_t v[16];
    const uint32_t taddr = tmem + ((uint32_t)(32 * warp) << 16);
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    const int m = 32 * warp + lane;
    for (int n = 0; n < 16; ++n) out[m * 16 + n] = __uint_as_float(v[n]);
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tmem));
}

static float h2f(__half h) { return __half2float(h); }

int main() {
  const int NA = 128 * 64, NB = 16 * 64;
  __half *ha = (__half*)malloc(NA * 2), *hb = (__half*)malloc(NB * 2);
  float* ho = (float*)malloc(128 * 16 * 4);
  srand(1);
  for (int i = 0; i < NA; ++i) ha[i] = __float2half((float)(rand() % 9 - 4));
  for (int i = 0; i < NB; ++i) hb[i] = __float2half((float)(rand() % 9 - 4));
  __half *da, *db;
  float* dout;
  int* dst;
  cudaMalloc(&da, NA * 2);
  cudaMalloc(&db, NB * 2);
  cudaMalloc(&dout, 128 * 16 * 4);
  cudaMalloc(&dst, 4);
  cudaMemcpy(da, ha, NA * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(db, hb, NB * 2, cudaMemcpyHostToDevice);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 24576);
  int fails = 0;
  const uint32_t var[5][4] = {{0, 0, 0, 0}, {2048, 1024, 128, 256}, {1024, 2048, 128, 256},
                              {2048, 1024, 256, 128}, {1024, 2048, 256, 128}};
  for (int vi = 0; vi < 5; ++vi) {
    const int mode = vi == 0 ? 0 : 1;
    cudaMemset(dout, 0xFF, 128 * 16 * 4);
    cudaMemset(dst, 0, 4);
    probe<<<1, 128, 24576>>>(mode, da, db, dout, dst, var[vi][0], var[vi][1], var[vi][2], var[vi][3]);
    cudaError_t e = cudaDeviceSynchronize();
    int st = 0;
    cudaMemcpy(&st, dst, 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(ho, dout, 128 * 16 * 4, cudaMemcpyDeviceToHost);
    int bad = 0;
    double maxerr = 0;
    for (int m = 0; m < 128; ++m)
      for (int n = 0; n < 16; ++n) {
        double ref = 0;
        if (mode == 0)
          for (int k = 0; k < 64; ++k) ref += (double)h2f(ha[m * 64 + k]) * h2f(hb[n * 64 + k]);
        else  // A[k][m] = ha[k*128 + m] (k < 16), B[k][n] = hb[k*16 + n]
          for (int k = 0; k < 16; ++k) ref += (double)h2f(ha[k * 128 + m]) * h2f(hb[k * 16 + n]);
        const double err = fabs(ref - ho[m * 16 + n]);
        if (err > maxerr) maxerr = err;
        if (err > 1e-3) {
          if (bad < 5) printf("  mode %d m %d n %d got %f want %f\n", mode, m, n, ho[m * 16 + n], ref);
          ++bad;
        }
      }
    printf("variant %d mode %d (%s) aLBO %u aSBO %u bLBO %u bSBO %u: cuda=%s status=%d mismatches=%d maxerr=%g\n", vi, mode,
           mode ? "spmm MN-major" : "sddmm K-major", var[vi][0], var[vi][1], var[vi][2], var[vi][3],
           cudaGetErrorString(e), st, bad, maxerr);
    if (vi <= 1) fails += (bad != 0) || (e != cudaSuccess) || st;
    if (e != cudaSuccess) break;
  }
  printf(fails ? "UMMA PROBE FAIL\n" : "UMMA PROBE OK\n");
  return fails ? 1 : 0;
}
