// Microbenchmark: tcgen05.ld (TMEM -> registers) throughput per SM with 4, 8 or 16 warps, and
// tcgen05.st. Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17
//   -I paper_conf_ppopp_liultj25_b200/csrc/kernels tools/tmem_bw.cu -o /tmp/tmem_bw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "sm100.cuh"
using namespace mario::sm100;

template <int NW, bool STORE>
__global__ void __launch_bounds__(NW * 32, 1) k(long long* cyc, uint32_t* sink, int iters) {
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32;
  if (warp == 0) tmem_alloc<512>(&slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t base = slot;
  const uint32_t lane_off = static_cast<uint32_t>((warp & 3) * 32) << 16;
  const uint32_t col0 = (warp / 4) * 32;   // warps beyond 4 read other column blocks
  uint32_t acc = 0;
  uint32_t r[32];
  for (int j = 0; j < 32; ++j) r[j] = j + threadIdx.x;
  __syncthreads();
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    const uint32_t a = base + lane_off + ((col0 + (i & 3) * 128) & 511);
    if (STORE) {
      tmem_st_32x32b_x32(a, r);
      tmem_st_wait();
    } else {
      tmem_ld_32x32b_x32(a, r);
      tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 32; ++j) acc += r[j];
    }
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc<512>(base);
}

template <int NW, bool STORE>
void run(const char* name) {
  const int iters = 4096, blocks = 148;
  long long* cyc;
  uint32_t* sink;
  cudaMalloc(&cyc, blocks * sizeof(long long));
  cudaMalloc(&sink, blocks * NW * 32 * 4);
  k<NW, STORE><<<blocks, NW * 32>>>(cyc, sink, iters);
  k<NW, STORE><<<blocks, NW * 32>>>(cyc, sink, iters);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double bytes = double(iters) * NW * 32 * 32 * 4;   // per CTA
  printf("%s warps=%d: %.1f B/clk per SM (%lld cycles, err=%s)\n", name, NW, bytes / h[0], h[0],
         cudaGetErrorString(e));
  cudaFree(cyc);
  cudaFree(sink);
}

int main() {
  run<1, false>("tcgen05.ld 32x32b.x32");
  run<4, false>("tcgen05.ld 32x32b.x32");
  run<8, false>("tcgen05.ld 32x32b.x32");
  run<16, false>("tcgen05.ld 32x32b.x32");
  run<4, true>("tcgen05.st 32x32b.x32");
  run<8, true>("tcgen05.st 32x32b.x32");
  return 0;
}
