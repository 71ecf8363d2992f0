/* mario_kernels.h — kernel-level C-ABI of libmario.so.
 *
 * These are the per-layer kernels the executor (mario_run_iter) launches, exported one
 * call per kernel family so that unit tests and the benchmark's roofline leg can drive
 * them directly. All pointers are DEVICE pointers owned by the caller; `stream` is a
 * cudaStream_t (NULL = legacy default stream). Every call is asynchronous and returns a
 * cudaError_t value (0 = success) for launch/argument errors; no exception crosses the ABI.
 * Matrices are row-major; ld* are row pitches in ELEMENTS and must be multiples of 8 for
 * bf16 operands (16-byte TMA pitch), otherwise cudaErrorInvalidValue (1) is returned.
 */
#ifndef MARIO_KERNELS_H
#define MARIO_KERNELS_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* K1-K3: D[M,N] = A[M,K] . B[N,K]^T on tcgen05 tensor cores (bf16 in, fp32 accumulate).
 * The linear layers of SURVEY §8(c) c1 (H = A W^T + b) and their backward passes
 * (dX = dY W, dW = dY^T X) are the three operand-major combinations:
 *   a_mn = 0: A stored [M][lda] (K-major);   a_mn = 1: A stored [K][lda] (M-major)
 *   b_mn = 0: B stored [N][ldb] (K-major);   b_mn = 1: B stored [K][ldb] (N-major)
 * Epilogue, in order: + bias[N] (fp32, may be NULL); * gelu'(aux[M,N]) if aux != NULL
 * (GeLU-tanh backward, A1); + residual[M,N] (bf16) if != NULL; then
 *   out_f32 = 1: D (fp32) = v + beta * D      (wgrad accumulation, beta in {0,1})
 *   out_f32 = 0: D (bf16) = v, and D2 (bf16, same pitch) = gelu_tanh(v) if D2 != NULL -- or, when
 *   aux != NULL too, D2 = gelu_tanh(aux) (the backward's recompute of the MLP activation G = gelu(Z)
 *   fused into the fc2 dgrad that reads Z anyway). aux requires out_f32 = 0 and residual = NULL
 *   (cudaErrorInvalidValue otherwise). */
int mario_k_gemm_bf16(const void* A, int lda, int a_mn, const void* B, int ldb, int b_mn,
                      int M, int N, int K, void* D, int ldd, int out_f32, float beta,
                      const float* bias, const void* residual, int ld_res,
                      void* D2, const void* aux, int ld_aux, void* stream);

/* Kernel selection for K1-K3: -1 = auto (CTA-pair tiles when M, N >= 256 and the pair tiles fill
 * the GPU — 256x256, or 256x128 when that wastes less of the last wave — else single-CTA
 * 128x256/128x128), 0 = single-CTA only, 1 = CTA pair whenever M, N >= 256 (auto N),
 * 2 = CTA pair 256x128, 3 = CTA pair 256x256. Process-global; returns 0, or 1 if invalid. */
int mario_k_gemm_set_variant(int variant);
/* Stream-K for the 256x256 CTA-pair kernel (0 = off, default; 1 = on): when whole tiles would leave > 5% of
 * the last wave idle, every pair runs an equal contiguous share of the (tile, k-block) iterations;
 * a tile split between pairs is finished by the part holding k-block 0, which adds the other
 * parts' fp32 partials (library-owned per-device workspace, ~19 MB) in pair order — deterministic.
 * GEMMs using it must not run concurrently on two streams of one device. Measured on B200 at the cfg-2
 * layer shapes: no faster than whole tiles (the chip is power-capped, so idle SMs in the last wave
 * raise the clock of the busy ones; K = 2048 parts cost more in fix-up than they save). Returns 0, or 1. */
int mario_k_gemm_set_streamk(int on);

/* K4: the same contract in true fp32 on CUDA cores (fp32 mode, reading A6). */
int mario_k_gemm_f32(const float* A, int lda, int a_mn, const float* B, int ldb, int b_mn,
                     int M, int N, int K, float* D, int ldd, float beta, const float* bias,
                     const float* residual, int ld_res, float* D2, const float* aux, int ld_aux,
                     void* stream);

/* K5: causal attention forward (S = QK^T/sqrt(dh), S[t,u] = -inf for u > t,
 * P = softmax, O = PV) per (sample, head). qkv: [B*s][3*H] with H = n_heads*head_dim, columns
 * [0,H) = Q, [H,2H) = K, [2H,3H) = V, head j at j*head_dim; O: [B*s][H]; lse: fp32
 * [n_heads][B*s] row log-sum-exp (natural log). bf16 = 1: bf16 storage on tensor cores
 * (head_dim in {16,32,64,80,128}), else fp32. */
int mario_k_attn_fwd(const void* qkv, void* O, float* lse, int B, int s, int n_heads, int head_dim,
                     int bf16, void* stream);
/* Kernel selection for K5/K6 (bf16): -1 = auto (tcgen05 for head_dim 64/128: the two-Q-tile
 * forward when it fills the GPU, else the one-Q-tile forward; mma.sync otherwise), 0 = mma.sync
 * only, 2 / 3 = tcgen05 with the one- / two-Q-tile forward forced. Process-global; returns 0, or 1
 * for an invalid value. */
int mario_k_attn_set_variant(int variant);
/* K6: backward: dqkv [B*s][3*H] (dQ | dK | dV) from dO [B*s][H], with P recomputed from lse;
 * deterministic (no atomics). scratch: fp32 [n_heads][B*s]. */
int mario_k_attn_bwd(const void* qkv, const void* O, const void* dO, const float* lse, void* dqkv,
                     float* scratch, int B, int s, int n_heads, int head_dim, int bf16, void* stream);
/* K6 with a dS workspace (bf16 only; SURVEY §8(c) c1 attention backward: dS = P (dP - D), dQ =
 * dS K / sqrt(dh)): the tcgen05 dK/dV kernel also stores dS (bf16, the values its dK MMA uses) into
 * ds_ws as per-(sample, head, 128-query block) tiles over the causal key tiles, and dQ is then one
 * product per tile over that image (no S / dP recompute). ds_ws: device, caller-owned, at least
 * mario_k_attn_bwd_ws_bytes(B, s, n_heads, head_dim) bytes, contents undefined on return. When
 * that size is 0 (head_dim not 64/128, s not a multiple of 128) or ds_ws_bytes is smaller, this is
 * mario_k_attn_bwd. Deterministic. Returns the CUDA error code (0 = OK). */
size_t mario_k_attn_bwd_ws_bytes(int B, int s, int n_heads, int head_dim);
int mario_k_attn_bwd_ws(const void* qkv, const void* O, const void* dO, const float* lse, void* dqkv,
                        float* scratch, void* ds_ws, size_t ds_ws_bytes, int B, int s, int n_heads, int head_dim,
                        void* stream);

/* K7/K8: LayerNorm (rms = 0: y = (x - mean)/sqrt(var + eps) * g + b) or RMSNorm (rms = 1:
 * y = x / sqrt(mean(x^2) + eps) * g) over rows of width n; stats =
 * fp32 [rows][2] (mean, rstd; mean = 0 for RMS). x, y: [rows][n] bf16 (bf16 = 1) or fp32. */
int mario_k_norm_fwd(const void* x, const float* g, const float* b, void* y, float* stats, int rows, int n,
                     float eps, int rms, int bf16, void* stream);
/* Backward (A1/A2 derivative): dx = norm'(dy) (+ dres if non-NULL). If dg != NULL, also, fused:
 * dg += sum_rows dy * xhat, db += sum_rows dy (LN; ignored for RMS) and, if dsum != NULL,
 * dsum += sum_rows dx (column sums of the written dx: the bias gradient of the producing linear).
 * partial: fp32 device scratch of partial_floats (>= 3 * n * 148 * 4 uses the fused kernel; the
 * column sums are deterministic: fixed-order two-pass). Returns a cudaError_t value. */
int mario_k_norm_bwd(const void* dy, const void* x, const float* stats, const float* g, const void* dres,
                     void* dx, float* dg, float* db, float* dsum, float* partial, long long partial_floats,
                     int rows, int n, int rms, int bf16, void* stream);
/* Kernel variant for both directions (bf16): 3 (default): variant 2's backward with a persistent
 * warp-per-row forward for n <= 4096 (16-byte chunks per lane, all loads of a warp's rows in flight,
 * shifted one-pass row statistics, warp butterflies only); 2: row-pipelined persistent kernels — each CTA
 * streams its contiguous row range through a ring of shared-memory stages filled by cp.async.bulk,
 * column sums reduced per CTA and finished by a fixed-order pass; 1: block-per-row-tile backward
 * with fused column sums + warp-per-row forward; 0: warp-per-row kernels + separate column-sum
 * passes. Widths the selected variant does not tile fall back to the next one. */
int mario_k_norm_set_variant(int v);

/* K13: softmax cross-entropy of one micro-batch (readings A4/A21): logits fp32
 * [rows][V] (rows = B * s, device), tokens int32 [B][ld_tok] (device; labels y = tokens[b][t + 1]).
 * row_loss[r] = logsumexp(logits[r]) - logits[r][y] (fp32, device); dlogits [rows][V] =
 * (softmax(logits[r]) - onehot(y)) * inv_ntok, bf16 (bf16 = 1) or fp32. bf16 with V % 4 == 0 and
 * V <= 51200 uses the register-resident one-read kernel. Returns a cudaError_t value. */
int mario_k_softmax_ce(const float* logits, const int* tokens, int ld_tok, int s, int rows, int V, float inv_ntok,
                       void* dlogits, float* row_loss, int bf16, void* stream);

/* Instrumentation. mario_kernel_launches: number of kernels this library has launched since it
 * was loaded (every call above and every mario_run_iter kernel). mario_kstats_enable(mask) clears
 * the records and starts CUDA-event timing, on the launching stream, of every launch of the kinds
 * whose bit is set (bit k = kind k: 0 GEMM, 1 attention forward, 2 attention backward, 4 norms,
 * 5 column sums, 6 softmax-CE, 7 elementwise, 8 embedding; -1 = all; 0 = off). Each timed launch
 * costs two event records, so time only what you need inside a measured region.
 * mario_kstats_read sums durations (ms), algorithmic FLOPs and bytes and counts launches of one
 * kind (synchronizes on the recorded events). Launches captured into a CUDA graph (mario_set_graphs)
 * re-record their events on every replay: when such records exist only they are read, i.e. the
 * latest replay. Each mario_kstats_enable invalidates captured iterations (the next call
 * re-captures). Returns 0 / -1. */
long long mario_kernel_launches(void);
int mario_kstats_enable(int mask);
int mario_kstats_read(int kind, double* total_ms, double* flops, double* bytes, long long* launches);

#ifdef __cplusplus
}
#endif
#endif
