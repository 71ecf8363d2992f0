// Internal launch interface of the per-layer kernels (K1-K15).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_bf16.h>

namespace mario {

int device_sm_count();          // SMs the launching thread may use (the device's, or its budget)
void set_sm_budget(int sms);     // 0 = the whole device
int device_sm_count_full();      // the device's SMs (reduction partitions that fix summation order)

// ------------------------------------------------------------------ GEMM (K1-K4)
struct GemmEpilogue {
  int out_f32 = 0;                        // 1: fp32 output (d_f32), 0: bf16 output (d_bf16)
  float* d_f32 = nullptr;
  __nv_bfloat16* d_bf16 = nullptr;
  __nv_bfloat16* d2_bf16 = nullptr;       // optional second output gelu(D) (GPT fc1)
  int ldd = 0;
  float beta = 0.f;                       // fp32 output: D = acc + beta * D
  const float* bias = nullptr;            // [N], added before activation / residual
  const __nv_bfloat16* residual = nullptr; int ld_res = 0;   // D += residual
  const __nv_bfloat16* aux = nullptr; int ld_aux = 0;        // D = acc * gelu'(aux)  (GeLU bwd)
  int d2_from_aux = 0;                    // with aux: D2 = gelu(aux) (recomputed MLP activation)
  // optional fused column sums of the bf16 output D (a bias gradient): colsum_part[M/32][N] fp32,
  // row block i = sum over rows [32 i, 32 i + 32) in row order. Requires bf16 output, M % 32 == 0,
  // N % 32 == 0 and 16-byte aligned pitches (gemm_bf16 returns cudaErrorInvalidValue otherwise).
  float* colsum_part = nullptr;
  // optional fused per-segment row dots of the bf16 output D with a bf16 input X (the attention
  // backward's D = rowsum(dO o O) per head, taken in the dO-producing GEMM): for every row r and
  // segment j of dot_seg columns, dot_out[j * dot_stride + r] = sum over the segment of bf16(D) * X.
  // Requires bf16 output without aux / residual, dot_seg % 32 == 0, N % dot_seg == 0, N % 32 == 0,
  // 16-byte aligned pitches (gemm_bf16 returns cudaErrorInvalidValue otherwise).
  const __nv_bfloat16* dot = nullptr; int ld_dot = 0;
  float* dot_out = nullptr; int dot_seg = 0; long dot_stride = 0;
};

struct GemmArgs {
  // D[M,N] = A[M,K] . B[N,K]^T ; a_mn / b_mn: operand stored MN-major ([K][rows]).
  const __nv_bfloat16* A = nullptr; int lda = 0; int a_mn = 0;
  const __nv_bfloat16* B = nullptr; int ldb = 0; int b_mn = 0;
  int M = 0, N = 0, K = 0;
  GemmEpilogue ep;
  int use_pair = -1;   // -1: auto, 0: never use the CTA-pair kernel, 1: always (if M, N >= 256)
  // 0: one CTA pair per tile instead of a persistent grid: when an independent GEMM runs on another
  // stream, its pairs are dispatched as the other kernel's last wave frees SMs (fills the wave tail)
  int persistent = 1;
};

cudaError_t gemm_bf16(const GemmArgs& g, cudaStream_t st);   // tcgen05 + TMA + TMEM

// fp32 SIMT GEMM (fp32 mode, K4): same contract with float operands.
struct GemmF32Args {
  const float* A = nullptr; int lda = 0; int a_mn = 0;
  const float* B = nullptr; int ldb = 0; int b_mn = 0;
  int M = 0, N = 0, K = 0;
  float* D = nullptr; int ldd = 0;
  float beta = 0.f;
  const float* bias = nullptr;
  const float* residual = nullptr; int ld_res = 0;
  float* D2 = nullptr;                  // gelu(D) second output
  const float* aux = nullptr; int ld_aux = 0;   // D = acc * gelu'(aux)
  int d2_from_aux = 0;                  // with aux: D2 = gelu(aux)
};
cudaError_t gemm_f32(const GemmF32Args& g, cudaStream_t st);

}  // namespace mario
