// tma_bench2.cu — can bulk (TMA) copies feed a row gather into shared memory on B200 when
// enough of them are in flight?  Round 1's tma_bench.cu had ONE thread per CTA issuing with 16
// ops in flight, and scaled linearly with CTAs/SM (latency-bound, never saturated).  Here
// every warp of a CTA owns a D-stage ring and R lanes of the warp issue one row copy each per
// stage, so a CTA keeps W*D*R row copies in flight (up to several hundred per SM).
//
//   bulk  : cp.async.bulk.shared::cluster.global (1-D, one row per op), rows of RB bytes
//   g4    : cp.async.bulk.tensor.2d ... tile::gather4 (4 rows x 128 B per op, 128B swizzle)
//   ldgsts: cp.async.cg 16 B per lane, 8 lanes per 128-B line (the SpMM ring of round 1)
// Source: 16 MiB fp16 matrix (L2-resident), uniformly random rows.  GB/s counts gathered bytes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/tma_bench2 tools/tma_bench2.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t par) {
  asm volatile("{.reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W;}" ::"r"(bar),
               "r"(par)
               : "memory");
}
__device__ __forceinline__ uint32_t xs(uint32_t x) {
  x ^= x << 13;
  x ^= x >> 17;
  x ^= x << 5;
  return x;
}

// MODE 0: bulk 1-D, MODE 1: gather4 (RB must be 128*h), MODE 2: ldgsts
template <int MODE, int D>
__global__ void ring_kernel(const __grid_constant__ CUtensorMap tmap, const uint8_t* __restrict__ src,
                            const int* __restrict__ idx, int nidx, int RB, int R, int iters,
                            unsigned long long* sink) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const int warps = blockDim.x / 32, wid = threadIdx.x / 32, lane = threadIdx.x & 31;
  const int stage_bytes = R * RB;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem);  // warps * D barriers
  uint8_t* ring = smem + 1024 + (size_t)wid * D * stage_bytes;
  if (threadIdx.x < warps * D) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bars[threadIdx.x])));
  }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  // row indices come from a precomputed random table (like col_idx), so no ALU work per op
  uint32_t cur = ((blockIdx.x * 64 + wid) * 977u) % (uint32_t)(nidx - 4096);
  // the row indices of stage i are loaded at iteration i - D (like col_idx riding D groups
  // ahead in the SpMM ring), so the index load latency is off the issue path
  int pre[D][4];
#pragma unroll
  for (int j = 0; j < D; ++j)
#pragma unroll
    for (int k = 0; k < 4; ++k) pre[j][k] = __ldg(idx + cur + j * R + 4 * (lane & 3) + k);
  unsigned acc = 0;
  // unrolled by D so that stage slot s and its index registers pre[s] are compile-time: no
  // register moves of in-flight loads (a MOV would wait for the load)
  for (int i0 = 0; i0 < iters + D; i0 += D)
#pragma unroll
  for (int s = 0; s < D; ++s) {
    const int i = i0 + s;
    if (i >= D) {  // consume stage s (issued D iterations ago)
      if (MODE == 2) {
        if (D == 2) asm volatile("cp.async.wait_group 1;" ::: "memory");
        else if (D == 4) asm volatile("cp.async.wait_group 3;" ::: "memory");
        else asm volatile("cp.async.wait_group 7;" ::: "memory");
      } else {
        mbar_wait(su32(&bars[wid * D + s]), ((i / D) - 1) & 1);
      }
      __syncwarp();
      acc += ring[s * stage_bytes + lane * 4];
    }
    if (i >= iters) continue;
    uint8_t* st = ring + s * stage_bytes;
    int rows4[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) rows4[k] = pre[s][k];
    // lane L's row for slot L (< 16): rows4 come from lane group (L & 3) -> shuffle
    int myrow = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int v = __shfl_sync(0xffffffffu, rows4[k], (lane >> 2) & 3);
      if ((lane & 3) == k) myrow = v;
    }
    int g4[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) g4[k] = __shfl_sync(0xffffffffu, rows4[k], (lane / (RB / 128)) & 3);
    if (MODE == 0) {
      if (lane == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bars[wid * D + s])),
                     "r"(stage_bytes)
                     : "memory");
      __syncwarp();
      if (lane < R) {
        const uint8_t* g = src + (size_t)myrow * RB;
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                su32(st + lane * RB)),
            "l"(g), "r"(RB), "r"(su32(&bars[wid * D + s]))
            : "memory");
      }
    } else if (MODE == 1) {
      if (lane == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bars[wid * D + s])),
                     "r"(stage_bytes)
                     : "memory");
      __syncwarp();
      const int halves = RB / 128;
      const int ops = (R / 4) * halves;  // each op: 4 rows x 128 B
      if (lane < ops) {
        const int q = lane / halves, h = lane % halves;
        int r[4];
        for (int k = 0; k < 4; ++k) r[k] = g4[k];
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
            " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(su32(st + (q * halves + h) * 512)),
            "l"(&tmap), "r"(64 * h), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(su32(&bars[wid * D + s]))
            : "memory");
      }
    } else {
      // 8 lanes per 128-B line: lane copies chunk (lane & 7) of rows (lane >> 3) + 4k
      const int lines = R * (RB / 128);
      for (int l = lane >> 3; l < lines; l += 4) {
        const int row = __shfl_sync(0xffffffffu, myrow, (l / (RB / 128)) & 15);
        const int seg = l % (RB / 128);
        const uint8_t* g = src + (size_t)row * RB + seg * 128 + (lane & 7) * 16;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(st + l * 128 + (lane & 7) * 16)),
                     "l"(g)
                     : "memory");
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    }
    cur = cur + (uint32_t)R < (uint32_t)(nidx - 64 - D * R) ? cur + R : 0;
    // indices of stage i + D into the slot just consumed (used D iterations from now)
#pragma unroll
    for (int k = 0; k < 4; ++k) pre[s][k] = __ldg(idx + cur + (D - 1) * R + 4 * (lane & 3) + k);
  }
  if (MODE == 2) asm volatile("cp.async.wait_all;" ::: "memory");
  sink[blockIdx.x * 64 + threadIdx.x % 64] = acc;
}

int main() {
  const int ROWS_BYTES = 16 << 20;
  uint8_t* B;
  cudaMalloc(&B, ROWS_BYTES);
  cudaMemset(B, 1, ROWS_BYTES);
  unsigned long long* sink;
  cudaMalloc(&sink, 1 << 22);
  const int NIDX = 1 << 22;
  int* idx;
  cudaMalloc(&idx, NIDX * 4);
  int* h = (int*)malloc(NIDX * 4);
  PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&encode, cudaEnableDefault, &q);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int RBs[3] = {128, 256, 512};
  for (int mode = 0; mode < 3; ++mode) {
    for (int ri = 0; ri < 3; ++ri) {
      const int RB = RBs[ri];
      CUtensorMap tmap;
      {
        const int cols = RB / 2, rows = ROWS_BYTES / RB;
        cuuint64_t gdim[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
        cuuint64_t gstride[1] = {(cuuint64_t)RB};
        cuuint32_t box[2] = {64, 1};
        cuuint32_t estr[2] = {1, 1};
        encode(&tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, B, gdim, gstride, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
               CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      }
      {
        uint32_t x = 12345u + RB;
        for (int i = 0; i < NIDX; ++i) {
          x ^= x << 13; x ^= x >> 17; x ^= x << 5;
          h[i] = (int)(x % (uint32_t)(ROWS_BYTES / RB));
        }
        cudaMemcpy(idx, h, NIDX * 4, cudaMemcpyHostToDevice);
      }
      const int R = 16;
      const int Ds[3] = {2, 4, 8};
      const int Ws[5] = {1, 2, 4, 8, 16};
      for (int di = 0; di < 3; ++di)
        for (int wi = 0; wi < 5; ++wi) {
          const int D = Ds[di], W = Ws[wi];
          const size_t smem = 1024 + (size_t)W * D * R * RB;
          if (smem > 227 * 1024) continue;
          auto pickk = [&](int m, int d) {
            if (d == 2) return m == 0 ? ring_kernel<0, 2> : m == 1 ? ring_kernel<1, 2> : ring_kernel<2, 2>;
            if (d == 4) return m == 0 ? ring_kernel<0, 4> : m == 1 ? ring_kernel<1, 4> : ring_kernel<2, 4>;
            return m == 0 ? ring_kernel<0, 8> : m == 1 ? ring_kernel<1, 8> : ring_kernel<2, 8>;
          };
          auto k = pickk(mode, D);
          cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
          const int iters = 2000;
          k<<<sms, W * 32, smem>>>(tmap, B, idx, NIDX, RB, R, 20, sink);
          cudaEventRecord(a);
          k<<<sms, W * 32, smem>>>(tmap, B, idx, NIDX, RB, R, iters, sink);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          const double bytes = (double)sms * W * iters * R * RB;
          printf("{\"mode\":\"%s\",\"row_bytes\":%d,\"stages\":%d,\"warps\":%d,\"rows_in_flight_per_sm\":%d,"
                 "\"GBps\":%.1f,\"err\":\"%s\"}\n",
                 mode == 0 ? "bulk" : mode == 1 ? "gather4" : "ldgsts", RB, D, W, W * D * R, bytes / ms / 1e6,
                 cudaGetErrorString(cudaGetLastError()));
          fflush(stdout);
        }
    }
  }
  return 0;
}
