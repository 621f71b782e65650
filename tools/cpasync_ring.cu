// cpasync_ring.cu — per-SM throughput of a warp-specialised cp.async gather ring (the producer
// side of sddmm_tc.cu) in isolation: one CTA per SM, P producer warps fill 16 KB stages
// (128 random rows x 128 B, 8 lanes per 128-byte line) into an S-stage ring; optionally a
// consumer warp waits for each stage on an mbarrier and frees it (no MMA).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/cpasync_ring tools/cpasync_ring.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait_parity(uint32_t bar, uint32_t ph) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(bar),
               "r"(ph) : "memory");
}
__device__ __forceinline__ void arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

constexpr int S = 11, LAG = 4;

// MODE 0: producers only (wait_group LAG); 1: + full/empty mbarriers with a consumer warp
template <int P, int MODE>
__global__ void ring(const uint8_t* __restrict__ table, int nrows, int nstages, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t full[S], empty[S];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&full[s])), "r"(P));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&empty[s])));
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const long long t0 = clock64();
  if (warp < P) {
    const int tid = threadIdx.x, c = tid & 7, rs = tid >> 3;
    constexpr int STEP = P * 4, PER = 128 / STEP;
    uint32_t x = 0x9E3779B9u * (blockIdx.x * 1024 + tid / 8 + 1);
    int s = 0;
    uint32_t ph = 0;
    for (int i = 0; i < nstages; ++i) {
      if (MODE == 1) wait_parity(su32(&empty[s]), ph ^ 1);
      const uint32_t st = su32(smem) + s * 16384;
#pragma unroll
      for (int k = 0; k < PER; ++k) {
        x ^= x << 13; x ^= x >> 17; x ^= x << 5;
        const int r = rs + STEP * k;
        const uint8_t* src = table + (size_t)(x % (uint32_t)nrows) * 512 + (i & 3) * 128 + 16 * c;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(st + r * 128 + ((c ^ (r & 7)) << 4)), "l"(src)
                     : "memory");
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
      if (i >= LAG) {
        asm volatile("cp.async.wait_group %0;" ::"n"(LAG) : "memory");
        if (MODE == 1) {
          __syncwarp();
          if (lane == 0) arrive(su32(&full[(s + S - LAG) % S]));
        }
      }
      if (++s == S) { s = 0; ph ^= 1; }
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if (MODE == 1) {
      __syncwarp();
      if (lane == 0)
        for (int i = nstages > LAG ? nstages - LAG : 0; i < nstages; ++i) arrive(su32(&full[i % S]));
    }
  } else if (MODE == 1 && warp == P) {
    int s = 0;
    uint32_t ph = 0;
    for (int i = 0; i < nstages; ++i) {
      wait_parity(su32(&full[s]), ph);
      if (lane == 0) arrive(su32(&empty[s]));
      if (++s == S) { s = 0; ph ^= 1; }
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = clock64() - t0;
}

template <int P, int MODE>
void run(const uint8_t* table, int nrows, unsigned long long* d, int sms) {
  const int smem = S * 16384;
  cudaFuncSetAttribute(ring<P, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int nst = 512;
  for (int rep = 0; rep < 2; ++rep) {
    ring<P, MODE><<<sms, (P + 1) * 32, smem>>>(table, nrows, nst, d);
    cudaDeviceSynchronize();
  }
  unsigned long long h[256];
  cudaMemcpy(h, d, 8 * sms, cudaMemcpyDeviceToHost);
  double avg = 0;
  for (int i = 0; i < sms; ++i) avg += h[i];
  avg /= sms;
  printf("P=%2d mode=%d: %.1f clk/stage  %.1f B/clk/SM  (%s)\n", P, MODE, avg / nst, 16384.0 * nst / avg,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int nrows = 8192;  // 4 MB table (L2-resident)
  uint8_t* table;
  cudaMalloc(&table, (size_t)nrows * 512);
  cudaMemset(table, 1, (size_t)nrows * 512);
  unsigned long long* d;
  cudaMalloc(&d, 8 * 256);
  run<4, 0>(table, nrows, d, sms);
  run<8, 0>(table, nrows, d, sms);
  run<16, 0>(table, nrows, d, sms);
  run<4, 1>(table, nrows, d, sms);
  run<8, 1>(table, nrows, d, sms);
  run<16, 1>(table, nrows, d, sms);
  return 0;
}
