// Microbenchmark: tcgen05.mma issue-to-completion rate per SM for the attention-backward shapes.
// One CTA per SM, one elected thread issues `iters` MMAs back to back (operands resident in shared
// memory / TMEM, contents irrelevant), commits, waits; clk per MMA = elapsed / iters.
//   SS N64  : M128 N64  K16, A and B K-major SW128 in smem        (S^T / dP^T of fa_bwd_dkdv_ts)
//   SS N128 : M128 N128 K16                                        (the N = 128 alternative)
//   SS N256 : M128 N256 K16                                        (GEMM-like)
//   TS N128 : M128 N128 K16, A from TMEM, B MN-major SW128 in smem (dV / dK += P^T dO, dS^T Q)
//   SS N64 x2: two accumulators alternating (S and dP interleaved as in the kernel)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//   -I paper_conf_ppopp_liultj25_b200/csrc/kernels tools/mma_rate.cu -o /tmp/mma_rate
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "sm100.cuh"
using namespace mario::sm100;

template <int MODE, bool BG = false>
__global__ void __launch_bounds__(128, 1) k(long long* cyc, int iters) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint32_t slot;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0x3c003c00u;
  __syncthreads();
  if (threadIdx.x == 0) reinterpret_cast<uint32_t*>(sm)[96 * 1024 / 4 - 1] = 0u;   // background stop flag
  if (warp == 0) tmem_alloc<512>(&slot);
  if (threadIdx.x == 32) { mbar_init(&bar, 1); fence_barrier_init(); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = slot;
  if (threadIdx.x == 0) {
    const uint32_t a = smem_u32(sm), b = smem_u32(sm + 32768);
    constexpr int N = MODE == 0 || MODE == 4 ? 64 : (MODE == 2 ? 256 : 128);
    constexpr uint32_t id_ss = umma_idesc_bf16(128, N, 0, 0);
    constexpr uint32_t id_ts = umma_idesc_bf16(128, 128, 0, 1);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const int kk = i & 7;
      const uint32_t ao = (kk >> 2) * (128 * 128) + (kk & 3) * 32, bo = (kk >> 2) * (N * 128) + (kk & 3) * 32;
      if (MODE == 3) {
        umma_bf16_ts(tm + 256, tm + (kk & 7) * 8, umma_desc_sw128(b + kk * 2048, 64 * 128, 1024), id_ts, 1);
      } else if (MODE == 4) {
        umma_bf16(tm + 256 + (i & 1) * 64, umma_desc_sw128(a + ao, 16, 1024), umma_desc_sw128(b + bo, 16, 1024), id_ss, 1);
      } else {
        umma_bf16(tm + 256 - (MODE == 2 ? 256 : 0), umma_desc_sw128(a + ao, 16, 1024), umma_desc_sw128(b + bo, 16, 1024),
                  id_ss, 1);
      }
    }
    umma_commit(&bar);
    mbar_wait(&bar, 0);
    long long t1 = clock64();
    cyc[blockIdx.x] = t1 - t0;
    if (BG) reinterpret_cast<volatile uint32_t*>(sm)[96 * 1024 / 4 - 1] = 1u;   // stop flag
  } else if (BG && threadIdx.x >= 32) {
    // background: warps 1-3 store 16 bytes per lane into a 16 KB region (no overlap with A / B) as
    // fast as they can, like softmax warps writing P tiles, until the MMA thread is done
    volatile uint32_t* stop = reinterpret_cast<volatile uint32_t*>(sm) + 96 * 1024 / 4 - 1;
    uint4* dst = reinterpret_cast<uint4*>(sm + 64 * 1024);
    uint4 v = make_uint4(threadIdx.x, 1, 2, 3);
    for (int i = 0; *stop == 0u; ++i) {
#pragma unroll
      for (int j = 0; j < 8; ++j) dst[((i * 8 + j) * 96 + threadIdx.x - 32) & 1023] = v;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc<512>(tm);
}

template <int MODE, bool BG = false>
void run(const char* name, int sms) {
  long long* d;
  cudaMalloc(&d, sms * sizeof(long long));
  const int smem = 100 * 1024;
  cudaFuncSetAttribute(k<MODE, BG>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int iters : {64, 4096}) {
    k<MODE, BG><<<sms, 128, smem>>>(d, iters);
    k<MODE, BG><<<sms, 128, smem>>>(d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    if (e) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
    long long h[1024];
    cudaMemcpy(h, d, sms * sizeof(long long), cudaMemcpyDeviceToHost);
    double s = 0;
    for (int i = 0; i < sms; ++i) s += h[i];
    printf("%-10s iters %5d: %.1f clk per MMA (mean over %d SMs)\n", name, iters, s / sms / iters, sms);
  }
  cudaFree(d);
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  run<0>("SS N64", sms);
  run<4>("SS N64x2", sms);
  run<1>("SS N128", sms);
  run<2>("SS N256", sms);
  run<3>("TS N128", sms);
  run<1, true>("SS N128+st", sms);
  run<3, true>("TS N128+st", sms);
  run<2, true>("SS N256+st", sms);
  return 0;
}
