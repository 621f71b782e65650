// gather_bench.cu — how fast can random 128-byte B rows reach the tensor-core operand
// registers on B200?  (SpMM design question; results in profiles/r02_*)
//   ldg_frag : LDG.128, mma.sync fragment lane mapping (lane 4g+t -> row t, chunk g)
//   ldg_line : LDG.128, 8 consecutive lanes per 128-byte row
//   ldgsts   : cp.async 16 B (8 lanes per row) into a D-stage per-warp ring + ldmatrix.x4.trans
//   ldg_sts  : LDG.128 (8 lanes per row) -> STS.128 -> ldmatrix.x4.trans (register staging)
// Each "group" = 16 random rows x 128 B = 2 KB; GB/s counts gathered bytes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/gather_bench tools/gather_bench.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t rnd(uint32_t& x) { x ^= x << 13; x ^= x >> 17; x ^= x << 5; return x; }

template <int MODE>
__global__ void ldg_kernel(const uint4* __restrict__ mat, int rows, int groups, uint4* sink) {
  const int lane = threadIdx.x & 31;
  const int rsel = MODE == 0 ? (lane & 3) : (lane >> 3);
  const int chunk = MODE == 0 ? (lane >> 2) : (lane & 7);
  uint32_t x = 0x9E3779B9u * (blockIdx.x * 64 + (threadIdx.x >> 5) * 4 + rsel + 1);
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (int it = 0; it < groups; ++it) {
    uint4 v[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int r = rnd(x) % rows;
      asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[k].x), "=r"(v[k].y), "=r"(v[k].z), "=r"(v[k].w) : "l"(mat + (int64_t)r * 8 + chunk));
    }
#pragma unroll
    for (int k = 0; k < 4; ++k) { acc.x ^= v[k].x; acc.y ^= v[k].y; acc.z ^= v[k].z; acc.w ^= v[k].w; }
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678) sink[threadIdx.x] = acc;
}

template <int D>
__global__ void ldgsts_kernel(const uint4* __restrict__ mat, int rows, int groups, uint4* sink) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint32_t base = smem_u32(smem + wid * D * 2048);
  const int cq = lane >> 3, cc = lane & 7;
  uint32_t x = 0x9E3779B9u * (blockIdx.x * 64 + wid * 4 + cq + 1);
  auto issue = [&](int j) {
    if (j < groups) {
      const uint32_t st = base + (j % D) * 2048;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int sl = cq + 4 * k;
        const int r = rnd(x) % rows;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(st + sl * 128 + ((cc ^ (sl & 7)) * 16)), "l"(mat + (int64_t)r * 8 + cc) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  for (int j = 0; j < D - 1; ++j) issue(j);
  uint32_t acc = 0;
  const int mi = lane >> 3, ri = lane & 7, slot = ri + 8 * (mi >> 1);
  for (int j = 0; j < groups; ++j) {
    issue(j + D - 1);
    asm volatile("cp.async.wait_group %0;" ::"n"(D - 1) : "memory");
    __syncwarp();
    const uint32_t rs = base + (j % D) * 2048 + slot * 128;
#pragma unroll
    for (int jj = 0; jj < 4; ++jj) {
      uint32_t a0, a1, a2, a3;
      const int chunk = 2 * jj + (mi & 1);
      asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];" : "=r"(a0), "=r"(a1), "=r"(a2), "=r"(a3) : "r"(rs + ((chunk ^ ri) * 16)));
      acc ^= a0 ^ a1 ^ a2 ^ a3;
    }
    __syncwarp();
  }
  if (acc == 0x12345678) sink[threadIdx.x] = make_uint4(acc, 0, 0, 0);
}

// register staging: LDG (8 lanes per row) of group j+1 in flight while group j is stored+read
__global__ void ldg_sts_kernel(const uint4* __restrict__ mat, int rows, int groups, uint4* sink) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint32_t base = smem_u32(smem + wid * 2048);
  const int cq = lane >> 3, cc = lane & 7;
  uint32_t x = 0x9E3779B9u * (blockIdx.x * 64 + wid * 4 + cq + 1);
  uint4 v[2][4];
  auto load = [&](uint4 (&r)[4]) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int row = rnd(x) % rows;
      asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r[k].x), "=r"(r[k].y), "=r"(r[k].z), "=r"(r[k].w) : "l"(mat + (int64_t)row * 8 + cc));
    }
  };
  uint32_t acc = 0;
  const int mi = lane >> 3, ri = lane & 7, slot = ri + 8 * (mi >> 1);
  auto consume = [&](const uint4 (&r)[4]) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int sl = cq + 4 * k;
      asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(base + sl * 128 + ((cc ^ (sl & 7)) * 16)), "r"(r[k].x), "r"(r[k].y), "r"(r[k].z), "r"(r[k].w) : "memory");
    }
    __syncwarp();
#pragma unroll
    for (int jj = 0; jj < 4; ++jj) {
      uint32_t a0, a1, a2, a3;
      const int chunk = 2 * jj + (mi & 1);
      asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];" : "=r"(a0), "=r"(a1), "=r"(a2), "=r"(a3) : "r"(base + slot * 128 + ((chunk ^ ri) * 16)));
      acc ^= a0 ^ a1 ^ a2 ^ a3;
    }
    __syncwarp();
  };
  load(v[0]);
  for (int j = 0; j < groups; j += 2) {
    load(v[1]);
    consume(v[0]);
    load(v[0]);
    consume(v[1]);
  }
  if (acc == 0x12345678) sink[threadIdx.x] = make_uint4(acc, 0, 0, 0);
}

template <typename F>
static float time_ms(F launch) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  launch();
  cudaDeviceSynchronize();
  float best = 1e30f;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(a);
    launch();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    if (ms < best) best = ms;
  }
  return best;
}

int main() {
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint4* buf; cudaMalloc(&buf, 64 << 20);
  cudaMemset(buf, 1, 64 << 20);
  uint4* sink; cudaMalloc(&sink, 1 << 20);
  const int groups = 512;
  for (int rowsMB : {16, 1}) {
    const int rows = (rowsMB << 20) / 128;
    for (int wps : {8, 16, 32, 64}) {  // warps per SM (4-warp CTAs)
      const int grid = sms * wps / 4;
      const double bytes = (double)grid * 4 * groups * 2048;
      float ms = time_ms([&] { ldg_kernel<0><<<grid, 128>>>(buf, rows, groups, sink); });
      printf("{\"test\":\"ldg_frag\",\"src_MB\":%d,\"warps_per_sm\":%d,\"GBps\":%.0f}\n", rowsMB, wps, bytes / ms / 1e6);
      ms = time_ms([&] { ldg_kernel<1><<<grid, 128>>>(buf, rows, groups, sink); });
      printf("{\"test\":\"ldg_line\",\"src_MB\":%d,\"warps_per_sm\":%d,\"GBps\":%.0f}\n", rowsMB, wps, bytes / ms / 1e6);
      if (wps <= 32) {
        cudaFuncSetAttribute(ldg_sts_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 2048);
        ms = time_ms([&] { ldg_sts_kernel<<<grid, 128, 4 * 2048>>>(buf, rows, groups, sink); });
        printf("{\"test\":\"ldg_sts_ldsm\",\"src_MB\":%d,\"warps_per_sm\":%d,\"GBps\":%.0f}\n", rowsMB, wps, bytes / ms / 1e6);
      }
      auto run_sts = [&](auto kern, int D) {
        const int smem = 4 * D * 2048;
        if ((int64_t)smem * (wps / 4) > 220 * 1024) return;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        float t = time_ms([&] { kern<<<grid, 128, smem>>>(buf, rows, groups, sink); });
        printf("{\"test\":\"ldgsts_ldsm\",\"D\":%d,\"src_MB\":%d,\"warps_per_sm\":%d,\"GBps\":%.0f}\n", D, rowsMB, wps, bytes / t / 1e6);
      };
      run_sts(ldgsts_kernel<2>, 2);
      run_sts(ldgsts_kernel<4>, 4);
      run_sts(ldgsts_kernel<8>, 8);
    }
  }
  return 0;
}
