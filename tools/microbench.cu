// microbench.cu — bandwidth ceilings that bound the gather (SURVEY §7 hard part 1):
//   HBM read   : LDG.128 streaming over 4 GiB
//   L2 read    : LDG.128 over a 48 MiB buffer (L2-resident), many passes, L1 bypassed
//   L1 read    : each CTA re-reads its own 32 KiB slice (L1-resident)
//   gather L2  : random 128-byte rows of a 16 MiB [rows x 64 fp16] matrix (the SpMM access)
//   mma.sync   : m16n8k16 f16->f32 issue rate, register operands
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/microbench tools/microbench.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__global__ void read_kernel(const uint4* __restrict__ p, int64_t n16, int passes, int64_t span16,
                            uint4* sink, int l1_bypass) {
  uint4 acc = make_uint4(0, 0, 0, 0);
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  for (int ps = 0; ps < passes; ++ps) {
    for (int64_t i = tid; i < n16; i += nth) {
      const uint4* q = p + (i % span16);
      uint4 v;
      if (l1_bypass)
        asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(q));
      else
        asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(q));
      acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
    }
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678) sink[tid] = acc;
}

// per-CTA private slice, re-read `passes` times (L1 hits after the first pass)
__global__ void l1_kernel(const uint4* __restrict__ p, int slice16, int passes, uint4* sink) {
  const uint4* base = p + (int64_t)blockIdx.x * slice16;
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (int ps = 0; ps < passes; ++ps)
    for (int i = threadIdx.x; i < slice16; i += blockDim.x) {
      uint4 v;
      asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(base + i));
      acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
    }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678) sink[threadIdx.x] = acc;
}

// gather: each group of 8 lanes reads one random 128-byte row (4 rows per LDG.128 instruction)
// mode 1: the mma.sync fragment mapping of the register-path SpMM (lane = 4g + t reads row t,
// chunk g): every quarter-warp phase touches 4 different rows instead of one.
__global__ void gather_kernel(const uint4* __restrict__ mat, int rows, int iters, uint4* sink,
                              int mode = 0) {
  const int lane = threadIdx.x & 31;
  const int rowsel = mode ? (lane & 3) : (lane >> 3);
  const int chunk = mode ? (lane >> 2) : (lane & 7);
  uint32_t x = 0x9E3779B9u * (blockIdx.x * blockDim.x / 8 + (threadIdx.x >> 5) * 4 + rowsel + 1);
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (int it = 0; it < iters; ++it) {
    x ^= x << 13; x ^= x >> 17; x ^= x << 5;
    const int r = x % rows;
    uint4 v;
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(mat + (int64_t)r * 8 + chunk));
    acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678) sink[threadIdx.x] = acc;
}

__global__ void mma_kernel(int iters, float* sink) {
  float d[4][4] = {};
  uint32_t a0 = threadIdx.x, a1 = a0 * 3, a2 = a0 * 5, a3 = a0 * 7, b0 = a0 * 11, b1 = a0 * 13;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k)
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                   : "+f"(d[k][0]), "+f"(d[k][1]), "+f"(d[k][2]), "+f"(d[k][3])
                   : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
  }
  float s = 0;
  for (int k = 0; k < 4; ++k) s += d[k][0] + d[k][1] + d[k][2] + d[k][3];
  if (s == 1.2345f) sink[threadIdx.x] = s;
}

static float time_ms(void (*launch)(void*), void* arg) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  launch(arg);
  cudaDeviceSynchronize();
  float best = 1e30f;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(a);
    launch(arg);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    if (ms < best) best = ms;
  }
  return best;
}

struct Args { const uint4* p; int64_t n16; int passes; int64_t span16; uint4* sink; int byp; int grid; int slice16; int rows; int iters; float* fs; };
static Args g;

int main() {
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk = 0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int64_t big = 4ll << 30;
  uint4* buf; cudaMalloc(&buf, big);
  cudaMemset(buf, 1, big);
  uint4* sink; cudaMalloc(&sink, 1 << 24);
  float* fs; cudaMalloc(&fs, 1 << 20);
  g = Args{buf, big / 16, 1, big / 16, sink, 1, sms * 8, 0, 0, 0, fs};
  // HBM
  float ms = time_ms([](void*) { read_kernel<<<g.grid, 512>>>(g.p, g.n16, 1, g.span16, g.sink, 1); }, nullptr);
  printf("{\"test\":\"hbm_read\",\"GBps\":%.1f}\n", big / ms / 1e6);
  // L2: 48 MiB span, 40 passes
  g.span16 = (48ll << 20) / 16; g.n16 = g.span16; g.passes = 40;
  ms = time_ms([](void*) { read_kernel<<<g.grid, 512>>>(g.p, g.n16, g.passes, g.span16, g.sink, 1); }, nullptr);
  printf("{\"test\":\"l2_read_cg\",\"GBps\":%.1f}\n", (double)g.span16 * 16 * g.passes / ms / 1e6);
  ms = time_ms([](void*) { read_kernel<<<g.grid, 512>>>(g.p, g.n16, g.passes, g.span16, g.sink, 0); }, nullptr);
  printf("{\"test\":\"l2_read_nc\",\"GBps\":%.1f}\n", (double)g.span16 * 16 * g.passes / ms / 1e6);
  // L1: 32 KiB per CTA, 1 CTA... sms*2 CTAs, 200 passes
  g.slice16 = 32 * 1024 / 16; g.passes = 200; g.grid = sms * 2;
  ms = time_ms([](void*) { l1_kernel<<<g.grid, 512>>>(g.p, g.slice16, g.passes, g.sink); }, nullptr);
  printf("{\"test\":\"l1_read\",\"GBps\":%.1f,\"B_per_clk_per_sm\":%.1f}\n",
         (double)g.grid * g.slice16 * 16 * g.passes / ms / 1e6,
         (double)g.grid * g.slice16 * 16 * g.passes / (ms * 1e-3) / (clk * 1e3) / sms);
  // gather of 128-byte rows from a 16 MiB matrix (L2-resident)
  g.rows = (16 << 20) / 128; g.iters = 2000; g.grid = sms * 16;
  ms = time_ms([](void*) { gather_kernel<<<g.grid, 256>>>(g.p, g.rows, g.iters, g.sink); }, nullptr);
  printf("{\"test\":\"gather128_l2\",\"GBps\":%.1f}\n", (double)g.grid * 256 * 16 * g.iters / ms / 1e6);
  // gather from a 64 KiB matrix (L1-resident rows)
  g.rows = (64 << 10) / 128;
  ms = time_ms([](void*) { gather_kernel<<<g.grid, 256>>>(g.p, g.rows, g.iters, g.sink); }, nullptr);
  printf("{\"test\":\"gather128_l1\",\"GBps\":%.1f}\n", (double)g.grid * 256 * 16 * g.iters / ms / 1e6);
  // the same gathers with the lane -> (row, chunk) mapping of the mma.sync A fragment
  g.rows = (16 << 20) / 128;
  ms = time_ms([](void*) { gather_kernel<<<g.grid, 256>>>(g.p, g.rows, g.iters, g.sink, 1); }, nullptr);
  printf("{\"test\":\"gather128_l2_fragmap\",\"GBps\":%.1f}\n", (double)g.grid * 256 * 16 * g.iters / ms / 1e6);
  g.rows = (64 << 10) / 128;
  ms = time_ms([](void*) { gather_kernel<<<g.grid, 256>>>(g.p, g.rows, g.iters, g.sink, 1); }, nullptr);
  printf("{\"test\":\"gather128_l1_fragmap\",\"GBps\":%.1f}\n", (double)g.grid * 256 * 16 * g.iters / ms / 1e6);
  // mma.sync m16n8k16 throughput
  g.iters = 4096; g.grid = sms * 4;
  ms = time_ms([](void*) { mma_kernel<<<g.grid, 512>>>(g.iters, g.fs); }, nullptr);
  double flops = (double)g.grid * 512 / 32 * g.iters * 4 * 2.0 * 16 * 8 * 16;
  printf("{\"test\":\"mma_sync_m16n8k16_f32acc\",\"TFLOPs\":%.1f}\n", flops / ms / 1e9);
  printf("{\"sms\":%d,\"clock_khz\":%d}\n", sms, clk);
  return 0;
}
