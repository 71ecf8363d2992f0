// C-ABI kernel-level entry points (include/mario_kernels.h): one call per kernel family,
// device pointers in, used by the GPU unit tests and the benchmark's per-kernel roofline.
#include <cuda_runtime.h>
#include "../kernels/kernels.h"
#include "../kernels/layers.h"
#include "../../../include/mario_kernels.h"

namespace mario { extern int g_gemm_variant; extern int g_attn_variant; extern int g_gemm_streamk; }
using namespace mario;

extern "C" int mario_k_gemm_set_variant(int variant) {
  if (variant < -1 || variant > 3) return 1;
  g_gemm_variant = variant;
  return 0;
}

extern "C" int mario_k_gemm_bf16(const void* A, int lda, int a_mn, const void* B, int ldb, int b_mn,
                                 int M, int N, int K, void* D, int ldd, int out_f32, float beta,
                                 const float* bias, const void* residual, int ld_res,
                                 void* D2, const void* aux, int ld_aux, void* stream) {
  GemmArgs g;
  g.A = static_cast<const __nv_bfloat16*>(A); g.lda = lda; g.a_mn = a_mn;
  g.B = static_cast<const __nv_bfloat16*>(B); g.ldb = ldb; g.b_mn = b_mn;
  g.M = M; g.N = N; g.K = K;
  g.ep.out_f32 = out_f32;
  if (out_f32) g.ep.d_f32 = static_cast<float*>(D); else g.ep.d_bf16 = static_cast<__nv_bfloat16*>(D);
  g.ep.ldd = ldd; g.ep.beta = beta; g.ep.bias = bias;
  g.ep.residual = static_cast<const __nv_bfloat16*>(residual); g.ep.ld_res = ld_res;
  g.ep.d2_bf16 = static_cast<__nv_bfloat16*>(D2);
  g.ep.aux = static_cast<const __nv_bfloat16*>(aux); g.ep.ld_aux = ld_aux;
  g.ep.d2_from_aux = (D2 && aux) ? 1 : 0;
  return static_cast<int>(gemm_bf16(g, static_cast<cudaStream_t>(stream)));
}

extern "C" int mario_k_gemm_set_streamk(int on) {
  if (on != 0 && on != 1) return 1;
  g_gemm_streamk = on;
  return 0;
}

extern "C" int mario_k_attn_set_variant(int variant) {
  if (variant < -1 || variant > 3) return 1;
  g_attn_variant = variant;
  return 0;
}

extern "C" int mario_k_gemm_f32(const float* A, int lda, int a_mn, const float* B, int ldb, int b_mn,
                                int M, int N, int K, float* D, int ldd, float beta, const float* bias,
                                const float* residual, int ld_res, float* D2, const float* aux, int ld_aux,
                                void* stream) {
  GemmF32Args g;
  g.A = A; g.lda = lda; g.a_mn = a_mn; g.B = B; g.ldb = ldb; g.b_mn = b_mn;
  g.M = M; g.N = N; g.K = K; g.D = D; g.ldd = ldd; g.beta = beta; g.bias = bias;
  g.residual = residual; g.ld_res = ld_res; g.D2 = D2; g.aux = aux; g.ld_aux = ld_aux;
  return static_cast<int>(gemm_f32(g, static_cast<cudaStream_t>(stream)));
}

extern "C" int mario_k_attn_fwd(const void* qkv, void* O, float* lse, int B, int s, int n_heads, int head_dim,
                                int bf16, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (bf16) {
    // a padded head dim (16 / 32 / 80) takes the tcgen05 kernels through a workspace of its own here
    void* pad = nullptr;
    const size_t pb = flash_attn_pad_bytes(head_dim, B, s, n_heads, 0);
    if (pb && cudaMalloc(&pad, pb) != cudaSuccess) return static_cast<int>(cudaErrorMemoryAllocation);
    attn_fwd<__nv_bfloat16>(static_cast<const __nv_bfloat16*>(qkv), static_cast<__nv_bfloat16*>(O), lse, B, s,
                            n_heads, head_dim, st, pad);
    if (pad) { cudaStreamSynchronize(st); cudaFree(pad); }
  }
  else attn_fwd<float>(static_cast<const float*>(qkv), static_cast<float*>(O), lse, B, s, n_heads, head_dim, st);
  return static_cast<int>(cudaGetLastError());
}

extern "C" int mario_k_attn_bwd(const void* qkv, const void* O, const void* dO, const float* lse, void* dqkv,
                                float* scratch, int B, int s, int n_heads, int head_dim, int bf16, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (bf16) {
    void* pad = nullptr;
    const size_t pb = flash_attn_pad_bytes(head_dim, B, s, n_heads, 1);
    if (pb && cudaMalloc(&pad, pb) != cudaSuccess) return static_cast<int>(cudaErrorMemoryAllocation);
    attn_bwd<__nv_bfloat16>(static_cast<const __nv_bfloat16*>(qkv), static_cast<const __nv_bfloat16*>(O),
                            static_cast<const __nv_bfloat16*>(dO), lse, static_cast<__nv_bfloat16*>(dqkv), scratch, B,
                            s, n_heads, head_dim, st, nullptr, 0, pad);
    if (pad) { cudaStreamSynchronize(st); cudaFree(pad); }
  }
  else attn_bwd<float>(static_cast<const float*>(qkv), static_cast<const float*>(O), static_cast<const float*>(dO), lse,
                       static_cast<float*>(dqkv), scratch, B, s, n_heads, head_dim, st);
  return static_cast<int>(cudaGetLastError());
}

extern "C" size_t mario_k_attn_bwd_ws_bytes(int B, int s, int n_heads, int head_dim) {
  return flash_attn_bwd_ds_bytes(head_dim, B, s, n_heads);
}

extern "C" int mario_k_attn_bwd_ws(const void* qkv, const void* O, const void* dO, const float* lse, void* dqkv,
                                   float* scratch, void* ds_ws, size_t ds_ws_bytes, int B, int s, int n_heads,
                                   int head_dim, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  attn_bwd<__nv_bfloat16>(static_cast<const __nv_bfloat16*>(qkv), static_cast<const __nv_bfloat16*>(O),
                          static_cast<const __nv_bfloat16*>(dO), lse, static_cast<__nv_bfloat16*>(dqkv), scratch, B, s,
                          n_heads, head_dim, st, ds_ws, ds_ws_bytes);
  return static_cast<int>(cudaGetLastError());
}

extern "C" int mario_k_norm_fwd(const void* x, const float* g, const float* b, void* y, float* stats, int rows, int n,
                                float eps, int rms, int bf16, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (bf16) {
    if (rms) rmsnorm_fwd<__nv_bfloat16>(static_cast<const __nv_bfloat16*>(x), g, static_cast<__nv_bfloat16*>(y), stats, rows, n, eps, st);
    else layernorm_fwd<__nv_bfloat16>(static_cast<const __nv_bfloat16*>(x), g, b, static_cast<__nv_bfloat16*>(y), stats, rows, n, eps, st);
  } else {
    if (rms) rmsnorm_fwd<float>(static_cast<const float*>(x), g, static_cast<float*>(y), stats, rows, n, eps, st);
    else layernorm_fwd<float>(static_cast<const float*>(x), g, b, static_cast<float*>(y), stats, rows, n, eps, st);
  }
  return static_cast<int>(cudaGetLastError());
}

extern "C" int mario_k_norm_bwd(const void* dy, const void* x, const float* stats, const float* g, const void* dres,
                                void* dx, float* dg, float* db, float* dsum, float* partial, long long partial_floats,
                                int rows, int n, int rms, int bf16, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (dg && !partial) return static_cast<int>(cudaErrorInvalidValue);
  const size_t pf = partial_floats > 0 ? static_cast<size_t>(partial_floats) : 0;
  if (bf16) {
    auto* X = static_cast<const __nv_bfloat16*>(x);
    auto* DY = static_cast<const __nv_bfloat16*>(dy);
    if (dg) norm_bwd<__nv_bfloat16>(DY, X, stats, g, static_cast<const __nv_bfloat16*>(dres),
                                    static_cast<__nv_bfloat16*>(dx), rows, n, rms, dg, db, dsum, partial, pf, st);
    else norm_bwd_dx<__nv_bfloat16>(DY, X, stats, g, static_cast<const __nv_bfloat16*>(dres),
                                    static_cast<__nv_bfloat16*>(dx), rows, n, rms, st);
  } else {
    auto* X = static_cast<const float*>(x);
    auto* DY = static_cast<const float*>(dy);
    if (dg) norm_bwd<float>(DY, X, stats, g, static_cast<const float*>(dres), static_cast<float*>(dx), rows, n, rms, dg,
                            db, dsum, partial, pf, st);
    else norm_bwd_dx<float>(DY, X, stats, g, static_cast<const float*>(dres), static_cast<float*>(dx), rows, n, rms, st);
  }
  return static_cast<int>(cudaGetLastError());
}

extern "C" int mario_k_norm_set_variant(int v) {
  if (v < 0 || v > 3) return static_cast<int>(cudaErrorInvalidValue);
  g_norm_tile = v;
  return 0;
}

extern "C" int mario_k_softmax_ce(const float* logits, const int* tokens, int ld_tok, int s, int rows, int V,
                                  float inv_ntok, void* dlogits, float* row_loss, int bf16, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (!logits || !tokens || !dlogits || !row_loss || s <= 0 || V <= 0 || ld_tok < s + 1)
    return static_cast<int>(cudaErrorInvalidValue);
  if (bf16) softmax_ce<__nv_bfloat16>(logits, tokens, ld_tok, s, rows, V, inv_ntok,
                                      static_cast<__nv_bfloat16*>(dlogits), row_loss, st);
  else softmax_ce<float>(logits, tokens, ld_tok, s, rows, V, inv_ntok, static_cast<float*>(dlogits), row_loss, st);
  return static_cast<int>(cudaGetLastError());
}
