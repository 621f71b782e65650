// umma_rate.cu — issue rate of tcgen05.mma.kind::f16 (M=128, K=16) on B200 as a function of N
// and of how many independent TMEM accumulators the issuing thread rotates over.  One CTA per
// SM, operands resident in shared memory, one thread issues R MMAs then commits and waits.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/umma_rate tools/umma_rate.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

template <int N, int NACC>
__global__ void __launch_bounds__(128, 1) rate(int R, unsigned long long* cycles) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < (128 + 256) * 128 / 16; i += blockDim.x)
    reinterpret_cast<uint4*>(smem)[i] = make_uint4(0, 0, 0, 0);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tbase;
  constexpr uint32_t idesc = (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((128u >> 4) << 24);
  if (threadIdx.x == 0) {
    const uint64_t ad = sdesc(su32(smem)), bd = sdesc(su32(smem + 128 * 128));
    const long long t0 = clock64();
    for (int i = 0; i < R; ++i) {
      const uint32_t dt = tmem + (uint32_t)((i % NACC) * N);
      asm volatile(
          "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
          "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(dt),
          "l"(ad), "l"(bd), "r"(idesc), "r"(i >= NACC ? 1 : 0)
          : "memory");
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar))
                 : "memory");
    asm volatile(
        "{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(
            su32(&bar))
        : "memory");
    cycles[blockIdx.x] = clock64() - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}

template <int N, int NACC>
static void run(unsigned long long* d, int sms) {
  const int smem = (128 + 256) * 128;
  cudaFuncSetAttribute(rate<N, NACC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int R : {64, 1024}) {
    rate<N, NACC><<<sms, 128, smem>>>(R, d);
    cudaDeviceSynchronize();
    unsigned long long h[256];
    cudaMemcpy(h, d, sizeof(unsigned long long) * sms, cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < sms; ++i) avg += h[i];
    avg /= sms;
    const double flop = 2.0 * 128 * N * 16;
    printf("N=%3d acc=%d R=%4d: %7.1f clk/MMA  %6.1f flop/clk/SM  err=%s\n", N, NACC, R, avg / R,
           flop * R / avg, cudaGetErrorString(cudaGetLastError()));
  }
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* d;
  cudaMalloc(&d, 256 * sizeof(unsigned long long));
  run<16, 1>(d, sms);
  run<16, 4>(d, sms);
  run<16, 16>(d, sms);
  run<32, 1>(d, sms);
  run<32, 8>(d, sms);
  run<64, 1>(d, sms);
  run<64, 4>(d, sms);
  run<128, 1>(d, sms);
  run<128, 2>(d, sms);
  run<256, 1>(d, sms);
  run<256, 2>(d, sms);
  return 0;
}
