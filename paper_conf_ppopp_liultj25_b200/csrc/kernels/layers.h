// Bandwidth-bound layer kernels, templated on the storage type
// T in {float, __nv_bfloat16}; all arithmetic in fp32. Every reduction is deterministic
// (fixed-order, no float atomics) so a Mario plan reproduces its base plan bit for bit.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_bf16.h>

namespace mario {

template <class T> void embed_fwd(const int32_t* tok, int ld_tok, int B, int s, const T* wte, const T* wpe,
                                  T* H, int h, cudaStream_t st);
// dwte[v] += sum_{tokens x=v} dH  (deterministic: per-micro-batch sort + segmented sum);
// dwpe[t] += sum_b dH[b,t] (if dwpe). scratch: >= 3*T int64 + 2*T int32 bytes.
template <class T> void embed_bwd(const int32_t* tok, int ld_tok, int B, int s, const T* dH, int h, float* dwte,
                                  float* dwpe, void* scratch, cudaStream_t st);

// LayerNorm / RMSNorm over rows of width n. stats = [rows][2] (mean, rstd) fp32.
template <class T> void layernorm_fwd(const T* x, const float* g, const float* b, T* y, float* stats, int rows,
                                      int n, float eps, cudaStream_t st);
template <class T> void rmsnorm_fwd(const T* x, const float* g, T* y, float* stats, int rows, int n, float eps,
                                    cudaStream_t st);
// y = norm(x) from stats the forward stored (b = NULL for RMSNorm): the backward's recompute of a
// norm output with the forward kernel's expression. Falls back to the full forward for fp32 / odd n.
template <class T> void norm_recompute(const T* x, const float* g, const float* b, T* y, float* stats, int rows,
                                       int n, float eps, int rms, cudaStream_t st);
// dx = LN'(dy) (+ dres); rms = 1 selects RMSNorm.
template <class T> void norm_bwd_dx(const T* dy, const T* x, const float* stats, const float* g, const T* dres,
                                    T* dx, int rows, int n, int rms, cudaStream_t st);
// Fused norm backward: dx as norm_bwd_dx, plus dg (+ db for LN) += the norm's column sums and, if
// dsum != NULL, dsum += column sums of the written dx (the bias gradient of the producing linear).
// partial: fp32 scratch of partial_floats (>= 3 * n * blocks used; falls back to separate passes).
template <class T> void norm_bwd(const T* dy, const T* x, const float* stats, const float* g, const T* dres, T* dx,
                                 int rows, int n, int rms, float* dg, float* db, float* dsum, float* partial,
                                 size_t partial_floats, cudaStream_t st);
// bf16 norm backward on the fp32 residual-gradient stream (reading A30): dx = norm'(dy) + residual,
// the residual taken from dres32 (fp32) if given, else dres (bf16), else none; dx is written as the
// bf16 operand of the following GEMMs and, if dx32 != NULL, in fp32 for the next residual add;
// dg / db / dsum as norm_bwd (dsum sums the fp32 dx when dx32 is given).
void norm_bwd_mixed(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                    const __nv_bfloat16* dres, const float* dres32, __nv_bfloat16* dx, float* dx32, int rows, int n,
                    int rms, float* dg, float* db, float* dsum, float* partial, size_t partial_floats, cudaStream_t st);
bool norm_bwd_pipe_mixed(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                         const __nv_bfloat16* dres, const float* dres32, __nv_bfloat16* dx, float* dx32, int rows,
                         int n, int rms, float* dg, float* db, float* dsum, float* partial, size_t partial_floats,
                         cudaStream_t st);
extern int g_norm_tile;
// Row-pipelined bf16 kernels (rowpipe.cu); false = shape not supported (caller falls back).
bool norm_pipe_supported(int n);
bool norm_fwd_warp(const __nv_bfloat16* x, const float* g, const float* b, __nv_bfloat16* y, float* stats, int rows,
                   int n, float eps, int rms, cudaStream_t st);
bool norm_fwd_pipe(const __nv_bfloat16* x, const float* g, const float* b, __nv_bfloat16* y, float* stats, int rows,
                   int n, float eps, int rms, cudaStream_t st);
bool norm_bwd_pipe(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                   const __nv_bfloat16* dres, __nv_bfloat16* dx, int rows, int n, int rms, float* dg, float* db,
                   float* dsum, float* partial, size_t partial_floats, cudaStream_t st);
bool softmax_ce_fast(const float* logits, const int32_t* tok, int ld_tok, int s, int rows, int V, float inv_ntok,
                     __nv_bfloat16* dlogits, float* row_loss, cudaStream_t st, long row0 = 0);
// Column reductions into fp32 grads (+=): mode 0: out0 += sum_r a[r,c]
// mode 1 (LN): out0 += sum dy*xhat, out1 += sum dy; mode 2 (RMS): out0 += sum dy*xhat.
// out[c] += sum_b partial[b][c] over nblk row blocks (fixed order): the second pass of column sums
// whose partials a GEMM epilogue produced (GemmEpilogue::colsum_part)
void colsum_finish(const float* partial, int nblk, int n, float* out, cudaStream_t st);
// out_k[c] += sum_b partial[k * nblk + b][c], k = 0..2 (null outputs skipped; no stream scope)
void colsum_reduce(const float* partial, int nblk, int n, float* out0, float* out1, float* out2, cudaStream_t st);
template <class T> void colsum(const T* a, const T* x, const float* stats, int rows, int n, int lda, int mode,
                               float* out0, float* out1, float* partial, cudaStream_t st);

// Causal attention over QKV [T, 3h] (q | k | v), heads of dh; O [T, h]; lse [nh][T] fp32.
template <class T> void attn_fwd(const T* qkv, T* O, float* lse, int B, int s, int nh, int dh, cudaStream_t st,
                                 void* pad_ws = nullptr);
// dqkv [T, 3h] from dO; Dscratch [nh][T] fp32.
// ds_ws (optional, >= flash_attn_bwd_ds_bytes): workspace for the dS image, which lets the bf16
// tcgen05 path compute dQ from the stored dS (fa_bwd_dq_img) instead of recomputing S and dP.
// bpart / bpart_done: see flash_attn_bwd_tc (bf16 only; *bpart_done = false otherwise)
template <class T> void attn_bwd(const T* qkv, const T* O, const T* dO, const float* lse, T* dqkv, float* Dscratch,
                                 int B, int s, int nh, int dh, cudaStream_t st, void* ds_ws = nullptr,
                                 size_t ds_ws_bytes = 0, void* pad_ws = nullptr, float* bpart = nullptr,
                                 bool* bpart_done = nullptr);
// bytes of that dS workspace for a shape (0 when the path does not apply)
size_t flash_attn_bwd_ds_bytes(int dh, int B, int s, int nh);

// RoPE (rotate-half) in place on the q and k parts of QKV; inverse = 1 rotates by -t*theta.
// tab (optional, bf16 path): the (cos, sin) table rope_table wrote for this (s, dh, base).
template <class T> void rope(T* qkv, int B, int s, int nh, int dh, float base, int inverse, cudaStream_t st,
                             const float2* tab = nullptr);
void rope_table(float2* tab, int s, int dh, float base, cudaStream_t st);   // [s][dh/2] (cos, sin)

// SwiGLU: M = silu(GU[:, :f]) * GU[:, f:];  backward dGU from dM.
template <class T> void swiglu_fwd(const T* GU, T* M, int rows, int f, cudaStream_t st);
template <class T> void swiglu_bwd(const T* GU, const T* dM, T* dGU, int rows, int f, cudaStream_t st);

// G = gelu_tanh(Z) elementwise (backward recompute of the MLP activation, GPT).
template <class T> void gelu_fwd(const T* Z, T* G, size_t n, cudaStream_t st);

// Softmax cross-entropy over fp32 logits [rows, V]: row_loss[r] = lse - z_y;
// dlogits (T) = (softmax - onehot) * inv_ntok. labels = tokens[:, 1:] of the micro-batch; local row r
// is the micro-batch's token row0 + r (a chunk of the fused head).
template <class T> void softmax_ce(const float* logits, const int32_t* tok, int ld_tok, int s, int rows, int V,
                                   float inv_ntok, T* dlogits, float* row_loss, cudaStream_t st, long row0 = 0);
// out[0] (double) = sum of row_loss[0..rows) in a fixed order.
void loss_reduce(const float* row_loss, int rows, double* out, cudaStream_t st);

// Tensor-core flash attention (bf16, mma.sync), used by attn_fwd/attn_bwd<bf16>.
bool flash_attn_supported(int dh);
// pad_ws (>= flash_attn_pad_bytes): a head dim the tcgen05 kernels do not tile (16, 32, 80) runs
// on them over zero-padded copies (attn_mma.cu); without it such head dims take mma.sync.
void flash_attn_fwd(const __nv_bfloat16* qkv, __nv_bfloat16* O, float* lse, int B, int s, int nh, int dh, cudaStream_t st,
                    void* pad_ws = nullptr);
// O == nullptr (head dims 16/32/64/128, no padding): Dd already holds D = rowsum(dO o O) per head
void flash_attn_bwd(const __nv_bfloat16* qkv, const __nv_bfloat16* O, const __nv_bfloat16* dO, const float* lse,
                    __nv_bfloat16* dqkv, float* Dd, int B, int s, int nh, int dh, cudaStream_t st,
                    void* ds_ws = nullptr, size_t ds_ws_bytes = 0, void* pad_ws = nullptr, float* bpart = nullptr,
                    bool* bpart_done = nullptr);
// bytes of the padded-head workspace (bwd = 0 forward, 1 backward incl. its dS image); 0: no padding
size_t flash_attn_pad_bytes(int dh, int B, int s, int nh, int bwd);
bool flash_attn_bwd_tc_supported(int dh, int B, int s, int nh);
// qk_scale: the softmax scale of q.k (<= 0: 1/sqrt(dh); the padded path passes 1/sqrt of the true dh)
bool flash_attn_fwd_tc(const __nv_bfloat16* qkv, __nv_bfloat16* O, float* lse, int B, int s, int nh, int dh,
                       cudaStream_t st, float qk_scale = 0.f);
// bpart (optional): fp32 [B*s/32][3*nh*dh] column partial sums of the written dQKV per 32-row block (the
// qkv-bias gradient's), filled only when the dK/dV kernel with the dS image and fa_bwd_dq_img run
// (*bpart_done = true); otherwise untouched and the caller sums dQKV itself.
bool flash_attn_bwd_tc(const __nv_bfloat16* qkv, const __nv_bfloat16* dO, const float* lse, const float* Dd,
                       __nv_bfloat16* dqkv, int B, int s, int nh, int dh, void* ds_ws, size_t ds_ws_bytes,
                       cudaStream_t st, float qk_scale = 0.f, float* bpart = nullptr, bool* bpart_done = nullptr);

void cast_f32_bf16(const float* x, __nv_bfloat16* y, size_t n, cudaStream_t st);
void add_f32(float* a, const float* b, size_t n, cudaStream_t st);       // a += b
void copy_f32(float* a, const float* b, size_t n, cudaStream_t st);
struct CopySrcs { const float* p[8]; int n; };                                 // n <= 8
void sum_copies_f32(float* dst, const CopySrcs& srcs, size_t n, cudaStream_t st);   // dst = sum in order

}  // namespace mario
