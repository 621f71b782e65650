// tma_bench.cu — throughput of TMA row gathers (cp.async.bulk.tensor.2d ... tile::gather4) and
// small 1-D bulk copies on B200: can TMA feed the SpMM gather (128-byte rows)?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/tma_bench tools/tma_bench.cu
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int STAGES>
__global__ void gather4_kernel(const __grid_constant__ CUtensorMap tmap, int rows, int iters,
                               int halves, unsigned long long* sink) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t full[STAGES];
  const int stage_bytes = 512 * halves;
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  uint32_t x = 0x9E3779B9u * (blockIdx.x + 1);
  for (int i = 0; i < iters; ++i) {
    const int s = i % STAGES;
    if (i >= STAGES) {  // wait for the previous use of this stage
      const uint32_t par = ((i / STAGES) - 1) & 1;
      asm volatile("{.reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W;}" ::"r"(
                       su32(&full[s])), "r"(par) : "memory");
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(stage_bytes)
                 : "memory");
    int r[4];
    for (int q = 0; q < 4; ++q) {
      x ^= x << 13; x ^= x >> 17; x ^= x << 5;
      r[q] = (int)(x % (uint32_t)rows);
    }
    for (int h = 0; h < halves; ++h) {
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
          " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(su32(smem + s * stage_bytes + h * 512)),
          "l"(&tmap), "r"(64 * h), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(su32(&full[s]))
          : "memory");
    }
  }
  for (int s = 0; s < STAGES; ++s) {
    const int last = iters - STAGES + s;
    if (last < 0) continue;
    const uint32_t par = (last / STAGES) & 1;
    asm volatile("{.reg .pred p; W2: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W2;}" ::"r"(
                     su32(&full[last % STAGES])), "r"(par) : "memory");
  }
  sink[blockIdx.x] = smem[5];
}

// 1-D bulk copies of `bytes` each from random row starts
template <int STAGES>
__global__ void bulk_kernel(const uint8_t* src, int rows, int row_bytes, int bytes, int iters,
                            unsigned long long* sink) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t full[STAGES];
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  uint32_t x = 0x9E3779B9u * (blockIdx.x + 7);
  for (int i = 0; i < iters; ++i) {
    const int s = i % STAGES;
    if (i >= STAGES) {
      const uint32_t par = ((i / STAGES) - 1) & 1;
      asm volatile("{.reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W;}" ::"r"(
                       su32(&full[s])), "r"(par) : "memory");
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(bytes)
                 : "memory");
    x ^= x << 13; x ^= x >> 17; x ^= x << 5;
    const uint8_t* g = src + (size_t)(x % (uint32_t)rows) * row_bytes;
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     su32(smem + s * bytes)), "l"(g), "r"(bytes), "r"(su32(&full[s]))
                 : "memory");
  }
  for (int s = 0; s < STAGES; ++s) {
    const int last = iters - STAGES + s;
    if (last < 0) continue;
    const uint32_t par = (last / STAGES) & 1;
    asm volatile("{.reg .pred p; W2: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W2;}" ::"r"(
                     su32(&full[last % STAGES])), "r"(par) : "memory");
  }
  sink[blockIdx.x] = smem[3];
}

int main() {
  const int K = 16384, N = 256;  // 8 MiB, L2-resident
  void* B;
  cudaMalloc(&B, (size_t)K * N * 2);
  cudaMemset(B, 0, (size_t)K * N * 2);
  unsigned long long* sink;
  cudaMalloc(&sink, 1 << 20);
  PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&encode, cudaEnableDefault, &q);
  CUtensorMap tmap;
  cuuint64_t gdim[2] = {(cuuint64_t)N, (cuuint64_t)K};
  cuuint64_t gstride[1] = {(cuuint64_t)N * 2};
  cuuint32_t box[2] = {64, 1};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = encode(&tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, B, gdim, gstride, box, estr,
                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                      CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("{\"encode\":%d}\n", (int)r);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  constexpr int S = 16;
  for (int halves = 1; halves <= 2; ++halves) {
    for (int ctas_per_sm = 1; ctas_per_sm <= 8; ctas_per_sm *= 2) {
      const int iters = 4000;
      const int smem = S * 512 * halves;
      cudaFuncSetAttribute(gather4_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      gather4_kernel<S><<<sms * ctas_per_sm, 32, smem>>>(tmap, K, 10, halves, sink);
      cudaEventRecord(a);
      gather4_kernel<S><<<sms * ctas_per_sm, 32, smem>>>(tmap, K, iters, halves, sink);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      double bytes = (double)sms * ctas_per_sm * iters * 512 * halves;
      printf("{\"test\":\"gather4\",\"halves\":%d,\"ctas_per_sm\":%d,\"GBps\":%.1f,\"err\":\"%s\"}\n", halves,
             ctas_per_sm, bytes / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
    }
  }
  for (int bytes = 128; bytes <= 2048; bytes *= 4) {
    for (int ctas_per_sm = 1; ctas_per_sm <= 8; ctas_per_sm *= 2) {
      const int iters = 4000;
      const int smem = S * bytes;
      cudaFuncSetAttribute(bulk_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      cudaEventRecord(a);
      bulk_kernel<S><<<sms * ctas_per_sm, 32, smem>>>((const uint8_t*)B, (K * N * 2) / bytes, bytes, bytes, iters, sink);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      double tot = (double)sms * ctas_per_sm * iters * bytes;
      printf("{\"test\":\"bulk1d\",\"bytes\":%d,\"ctas_per_sm\":%d,\"GBps\":%.1f,\"err\":\"%s\"}\n", bytes, ctas_per_sm,
             tot / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
