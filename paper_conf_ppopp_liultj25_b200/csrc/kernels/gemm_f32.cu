// K4: true-fp32 SIMT GEMM for fp32 mode (tcgen05 kind::tf32 cannot meet the
// 1e-4 fp32 tolerance). Same operand contract as gemm_bf16: D = A . B^T with each operand
// K-major or MN-major, plus the same fused epilogue. 64x64 tiles, 16x16 threads, 4x4 per thread.
#include <cuda_runtime.h>
#include "kernels.h"
#include "kstats.h"

namespace mario {
namespace {

constexpr int T = 64, TK = 16;

__device__ __forceinline__ float gelu_f(float z) {
  const float c = 0.7978845608028654f;
  return 0.5f * z * (1.f + tanhf(c * (z + 0.044715f * z * z * z)));
}
__device__ __forceinline__ float gelu_grad_f(float z) {
  const float c = 0.7978845608028654f;
  float t = tanhf(c * (z + 0.044715f * z * z * z));
  return 0.5f * (1.f + t) + 0.5f * z * (1.f - t * t) * c * (1.f + 3.f * 0.044715f * z * z);
}

__global__ void __launch_bounds__(256) gemm_f32_kernel(GemmF32Args g) {
  __shared__ float As[TK][T + 1];
  __shared__ float Bs[TK][T + 1];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int m0 = blockIdx.y * T, n0 = blockIdx.x * T;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < g.K; k0 += TK) {
    for (int i = threadIdx.x; i < T * TK; i += 256) {
      int r, k;
      if (g.a_mn) { r = i % T; k = i / T; } else { k = i % TK; r = i / TK; }
      const int gm = m0 + r, gk = k0 + k;
      As[k][r] = (gm < g.M && gk < g.K) ? (g.a_mn ? g.A[(size_t)gk * g.lda + gm] : g.A[(size_t)gm * g.lda + gk]) : 0.f;
      if (g.b_mn) { r = i % T; k = i / T; } else { k = i % TK; r = i / TK; }
      const int gn = n0 + r, gk2 = k0 + k;
      Bs[k][r] = (gn < g.N && gk2 < g.K) ? (g.b_mn ? g.B[(size_t)gk2 * g.ldb + gn] : g.B[(size_t)gn * g.ldb + gk2]) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < TK; ++k) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { a[i] = As[k][ty + 16 * i]; b[i] = Bs[k][tx + 16 * i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int m = m0 + ty + 16 * i;
    if (m >= g.M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tx + 16 * j;
      if (n >= g.N) continue;
      float v = acc[i][j];
      if (g.bias) v += g.bias[n];
      if (g.aux) v *= gelu_grad_f(g.aux[(size_t)m * g.ld_aux + n]);
      if (g.residual) v += g.residual[(size_t)m * g.ld_res + n];
      float* d = g.D + (size_t)m * g.ldd + n;
      if (g.beta != 0.f) v += g.beta * *d;
      *d = v;
      if (g.D2) g.D2[(size_t)m * g.ldd + n] = (g.aux && g.d2_from_aux) ? gelu_f(g.aux[(size_t)m * g.ld_aux + n]) : gelu_f(v);
    }
  }
}

}  // namespace

cudaError_t gemm_f32(const GemmF32Args& g, cudaStream_t st) {
  if (g.M <= 0 || g.N <= 0) return cudaSuccess;
  dim3 grid((g.N + T - 1) / T, (g.M + T - 1) / T);
  const int tok = kstats_begin(K_GEMM, 2.0 * g.M * g.N * g.K, 0.0, st);
  gemm_f32_kernel<<<grid, 256, 0, st>>>(g);
  kstats_end(tok, st);
  note_launch();
  return cudaGetLastError();
}

}  // namespace mario
