// Row-pipelined bandwidth kernels (SURVEY §2.2 K7/K8 norms, K13 softmax-CE, K14 column sums), bf16.
//
// Norms: a persistent grid (occupancy x SMs CTAs); CTA b owns the contiguous row range
// [rows*b/nblk, rows*(b+1)/nblk). Its rows stream through a ring of S shared-memory stages filled by
// 1-D bulk copies (cp.async.bulk, one mbarrier per stage), so S rows per CTA are in flight while
// the current one is reduced: the DRAM queue never drains between rows (the warp-per-row kernels
// load, reduce, store and only then start the next row: 1.5 TB/s measured). Thread t owns the
// 16-byte chunk t of a row (block = n/8 threads rounded up to a warp): row sums go warp -> shared
// memory -> every thread in a fixed order (deterministic), one __syncthreads per row, after which
// thread 0 refills the stage just consumed.
// Formulas: SURVEY §8(c) c1 (LN/RMS forward, readings A1/A2; backward dx = (g - mean g - xhat
// mean(g xhat)) / sigma, dgamma = sum dy xhat, dbeta = sum dy).
#include <cstdint>
#include <cstdlib>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "kstats.h"
#include "layers.h"
#include "sm100.cuh"

#include "kernels.h"

namespace mario {
namespace {
using bf16 = __nv_bfloat16;

// the device's full SM count, NOT the launching thread's budget: the row partition of the column
// reductions below follows it, so their fp32 partial sums (and the bits of the bias / gain
// gradients) do not depend on the SM partition a stage runs on (emulated pipeline, set_sm_budget)
int device_sms() { return device_sm_count_full(); }
using namespace sm100;

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ uint4 lds128(const void* p) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ float wsum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float wmax(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ void unpack8(const uint4& u, float (&f)[8]) {
  const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) { const float2 p = __bfloat1622float2(h[i]); f[2 * i] = p.x; f[2 * i + 1] = p.y; }
}
__device__ __forceinline__ uint4 pack8(const float (&f)[8]) {
  uint4 u;
  __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
  return u;
}
__device__ __forceinline__ void load8(const float* p, float (&f)[8]) {
  const float4 a = *reinterpret_cast<const float4*>(p), b = *reinterpret_cast<const float4*>(p + 4);
  f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
}

// packed fp32x2 arithmetic (sm_100 FADD2 / FMUL2 / FFMA2: two IEEE fp32 lanes per instruction,
// each lane rounded exactly like the scalar op). The norm kernels are issue-bound, not DRAM-bound
// (ncu: 40% of stall samples "selected / not selected", DRAM 18%), so halving the fp32 instruction
// count per element is what moves them.
__device__ __forceinline__ unsigned long long pk2(float2 a) {
  unsigned long long u;
  asm("mov.b64 %0, {%1, %2};" : "=l"(u) : "f"(a.x), "f"(a.y));
  return u;
}
__device__ __forceinline__ float2 upk2(unsigned long long u) {
  float2 a;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a.x), "=f"(a.y) : "l"(u));
  return a;
}
__device__ __forceinline__ float2 add2(float2 a, float2 b) {
  unsigned long long d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(pk2(a)), "l"(pk2(b)));
  return upk2(d);
}
__device__ __forceinline__ float2 mul2(float2 a, float2 b) {
  unsigned long long d;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(pk2(a)), "l"(pk2(b)));
  return upk2(d);
}
__device__ __forceinline__ float2 fma2(float2 a, float2 b, float2 c) {
  unsigned long long d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(pk2(a)), "l"(pk2(b)), "l"(pk2(c)));
  return upk2(d);
}
__device__ __forceinline__ float2 f2(float a, float b) { return make_float2(a, b); }
// y = (x - mean) * rstd * g + b for 8 values: the expression every norm-forward path uses
__device__ __forceinline__ void norm_out8(const float (&v)[8], float mean, float rstd, const float (&gg)[8],
                                          const float (&bb)[8], float (&o)[8]) {
#pragma unroll
  for (int j = 0; j < 8; j += 2) {
    const float2 t = mul2(add2(f2(v[j], v[j + 1]), f2(-mean, -mean)), f2(rstd, rstd));
    const float2 r = fma2(t, f2(gg[j], gg[j + 1]), f2(bb[j], bb[j + 1]));
    o[j] = r.x; o[j + 1] = r.y;
  }
}

// Totals of the per-warp row partials rp[(w * R + q) * 2 + c] over the nw warps, for every row q
// of the iteration and c = 0 / 1, broadcast to all lanes: lane l adds entries l, l + 32, ... (all
// with the same (q, c) = l mod 2R), a 3-step butterfly combines lanes of equal l mod 2R, a shuffle
// broadcasts. ~10 instructions per thread instead of 4 nw shared loads + adds. Fixed order.
template <int R>
__device__ __forceinline__ void cross_warp_sums(const float* rp, int nw, int lane, float (&A)[R], float (&Bv)[R]) {
  constexpr int PER = 2 * R;
  static_assert(32 % PER == 0, "partials per warp must divide the warp");
  float acc = 0.f;
  for (int l = lane; l < nw * PER; l += 32) acc += rp[l];
#pragma unroll
  for (int o = 16; o >= PER; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
#pragma unroll
  for (int q = 0; q < R; ++q) {
    A[q] = __shfl_sync(0xffffffffu, acc, 2 * q);
    Bv[q] = __shfl_sync(0xffffffffu, acc, 2 * q + 1);
  }
}

// shared memory: S slots of `stage_bytes` (16-byte multiples), S mbarriers, the reduction buffers
// rows per iteration of the norm kernels (R; their reductions interleave, one barrier per R rows):
// MARIO_NORM_FWD_R / MARIO_NORM_BWD_R select 2, 4 or 8
inline size_t pipe_smem_bytes(int S, int stage_bytes, int R) {
  return static_cast<size_t>(S) * stage_bytes + S * sizeof(uint64_t) + 2 * 32 * R * 2 * sizeof(float);
}
int norm_rows_per_iter(bool fwd) {
  static const int f = getenv("MARIO_NORM_FWD_R") ? atoi(getenv("MARIO_NORM_FWD_R")) : 4;   // A/B: 172 -> 162 ms of norm per step with the 2-D apply
  static const int b = getenv("MARIO_NORM_BWD_R") ? atoi(getenv("MARIO_NORM_BWD_R")) : 2;
  const int r = fwd ? f : b;
  return r == 8 ? 8 : (r == 4 ? 4 : 2);
}

// ------------------------------------------------------------------------- forward
// y = (x - mean) * rstd * g (+ b); stats[r] = (mean, rstd). R rows per iteration (their reductions
// interleave), one __syncthreads per iteration. LN sums are shifted by the row's first element K
// (one broadcast shared load): mean = K + S1/n, var = S2/n - (S1/n)^2 with S1 = sum(x - K),
// S2 = sum((x - K)^2), so the cancellation is relative to |mean - K| ~ one standard deviation, not
// |mean|. Warp sums -> shared memory [par][warp][R][2] -> every thread adds the warps in order.
template <bool RMS, int R>
__global__ void __launch_bounds__(R == 2 ? 1024 : 640) norm_fwd_pipe_k(const bf16* __restrict__ x, const float* __restrict__ g,
                                                        const float* __restrict__ b, bf16* __restrict__ y,
                                                        float* __restrict__ stats, int rows, int n, float eps, int S,
                                                        int nblk) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const int sb = n * 2;
  uint8_t* stage0 = smem_raw;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem_raw + static_cast<size_t>(S) * sb);
  float* red = reinterpret_cast<float*>(bar + S);     // [2][32][R][2]
  const int t = threadIdx.x, w = t / 32, lane = t % 32, nw = blockDim.x / 32;
  const bool act = t * 8 < n;
  const int rb = static_cast<int>(static_cast<long>(rows) * blockIdx.x / nblk);
  const int re = static_cast<int>(static_cast<long>(rows) * (blockIdx.x + 1) / nblk);
  if (t == 0) {
    for (int i = 0; i < S; ++i) mbar_init(&bar[i], 1);
    fence_barrier_init();
  }
  __syncthreads();
  if (t == 0) {
    for (int i = 0; i < S && rb + i < re; ++i) {
      mbar_arrive_expect_tx(&bar[i], sb);
      bulk_g2s(stage0 + static_cast<size_t>(i) * sb, x + static_cast<long>(rb + i) * n, sb, &bar[i]);
    }
  }
  float gg[8], bb[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) { gg[j] = 0.f; bb[j] = 0.f; }
  if (act) {
    load8(g + t * 8, gg);
    if (!RMS) load8(b + t * 8, bb);
  }
  const float inv_n = 1.f / n;
  for (int r0 = rb, it = 0; r0 < re; r0 += R, ++it) {
    float v[R][8], K[R], s1[R], s2[R];
    const int par = it & 1;
#pragma unroll
    for (int q = 0; q < R; ++q) {
      const int u = it * R + q, sl = u % S;
      s1[q] = 0.f; s2[q] = 0.f; K[q] = 0.f;
#pragma unroll
      for (int j = 0; j < 8; ++j) v[q][j] = 0.f;
      if (r0 + q < re) {
        const uint8_t* buf = stage0 + static_cast<size_t>(sl) * sb;
        mbar_wait(&bar[sl], (u / S) & 1);
        if (act) unpack8(lds128(buf + t * 16), v[q]);
        if (!RMS) K[q] = __bfloat162float(*reinterpret_cast<const bf16*>(buf));
      }
      if (act) {
        float2 a1 = f2(0.f, 0.f), a2 = f2(0.f, 0.f);
#pragma unroll
        for (int j = 0; j < 8; j += 2) {
          const float2 d = add2(f2(v[q][j], v[q][j + 1]), f2(-K[q], -K[q]));
          a1 = add2(a1, d);
          a2 = fma2(d, d, a2);
        }
        s1[q] = a1.x + a1.y;
        s2[q] = a2.x + a2.y;
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
      for (int q = 0; q < R; ++q) {
        if (!RMS) s1[q] += __shfl_xor_sync(0xffffffffu, s1[q], o);
        s2[q] += __shfl_xor_sync(0xffffffffu, s2[q], o);
      }
    }
    float* rp = red + par * (32 * R * 2);
    if (lane == 0) {
#pragma unroll
      for (int q = 0; q < R; ++q) { rp[(w * R + q) * 2] = s1[q]; rp[(w * R + q) * 2 + 1] = s2[q]; }
    }
    __syncthreads();
    // every thread holds its chunks in registers: refill the slots just consumed
    if (t == 0) {
#pragma unroll
      for (int q = 0; q < R; ++q) {
        const int u = it * R + q, rn = rb + u + S;
        if (rn < re) {
          const int sl = u % S;
          mbar_arrive_expect_tx(&bar[sl], sb);
          bulk_g2s(stage0 + static_cast<size_t>(sl) * sb, x + static_cast<long>(rn) * n, sb, &bar[sl]);
        }
      }
    }
    float S1[R], S2[R];
    cross_warp_sums<R>(rp, nw, lane, S1, S2);
#pragma unroll
    for (int q = 0; q < R; ++q) {
      const int r = r0 + q;
      if (r >= re) break;
      float mean = 0.f, var;
      if (RMS) {
        var = S2[q] * inv_n;
      } else {
        const float m1 = S1[q] * inv_n;
        mean = K[q] + m1;
        var = fmaxf(S2[q] * inv_n - m1 * m1, 0.f);
      }
      const float rstd = rsqrtf(var + eps);
      if (act) {
        float o[8];
        norm_out8(v[q], mean, rstd, gg, bb, o);
        *reinterpret_cast<uint4*>(y + static_cast<long>(r) * n + t * 8) = pack8(o);
      }
      if (t == 0) *reinterpret_cast<float2*>(stats + 2 * static_cast<long>(r)) = make_float2(mean, rstd);
    }
  }
}

// ------------------------------------------------------------------------ backward
// dx = (dy g - mean(dy g) - xhat mean(dy g xhat)) rstd (+ dres); the CTA's column partial sums
// partial[0][blk] = sum dy xhat, [1] = sum dy (LN), [2] = sum of the written dx (when sum_out).
// Slot = [dy row | x row | dres row]; R rows per iteration. Phase 1 reads dy, x from shared
// memory (row sums), phase 2 (after the barrier) re-reads dy, x, dres and writes dx, so nothing
// but the column accumulators stays in registers; a slot is refilled at the NEXT iteration's
// barrier, when every thread is past its phase 2. Stats of the CTA's range are staged in smem.
// RES: residual input dres none (0) / bf16 (1) / fp32 (2); OUT32: also write dx in fp32 (dx32).
// With the fp32 residual-gradient stream (reading A30) the layer-to-layer dH chain stays fp32 and
// the bf16 dx is only the operand copy of the following GEMMs; the column sums of dx (a bias
// gradient) are then taken over the fp32 values.
template <int R, int V, int RES, bool OUT32>   // V: 16-byte chunks per thread (t, t + nt, ...)
__global__ void __launch_bounds__(640) norm_bwd_pipe_k(const bf16* __restrict__ dy, const bf16* __restrict__ x,
                                                       const float* __restrict__ stats, const float* __restrict__ g,
                                                       const void* __restrict__ dres, bf16* __restrict__ dx,
                                                       float* __restrict__ dx32, int rows,
                                                       int n, int rms, float* __restrict__ partial, int nblk,
                                                       int sum_out, int S, int max_range) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const int row_bytes = n * 2, res_bytes = RES == 2 ? n * 4 : (RES == 1 ? n * 2 : 0);
  const int sb = 2 * row_bytes + res_bytes;
  uint8_t* stage0 = smem_raw;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem_raw + static_cast<size_t>(S) * sb);
  float* red = reinterpret_cast<float*>(bar + S);            // [2][32][R][2]
  float2* sstat = reinterpret_cast<float2*>(red + 2 * 32 * R * 2);
  const int t = threadIdx.x, w = t / 32, lane = t % 32, nw = blockDim.x / 32, nt = blockDim.x;
  bool act[V];
#pragma unroll
  for (int k = 0; k < V; ++k) act[k] = (t + k * nt) * 8 < n;
  const int rb = static_cast<int>(static_cast<long>(rows) * blockIdx.x / nblk);
  const int re = static_cast<int>(static_cast<long>(rows) * (blockIdx.x + 1) / nblk);
  auto issue = [&](int sl, int r) {
    uint8_t* buf = stage0 + static_cast<size_t>(sl) * sb;
    mbar_arrive_expect_tx(&bar[sl], sb);
    bulk_g2s(buf, dy + static_cast<long>(r) * n, row_bytes, &bar[sl]);
    bulk_g2s(buf + row_bytes, x + static_cast<long>(r) * n, row_bytes, &bar[sl]);
    if (RES) bulk_g2s(buf + 2 * row_bytes, static_cast<const uint8_t*>(dres) + static_cast<long>(r) * res_bytes,
                      res_bytes, &bar[sl]);
  };
  if (t == 0) {
    for (int i = 0; i < S; ++i) mbar_init(&bar[i], 1);
    fence_barrier_init();
  }
  __syncthreads();
  if (t == 0)
    for (int i = 0; i < S && rb + i < re; ++i) issue(i, rb + i);
  for (int i = t; i < re - rb && i < max_range; i += blockDim.x)
    sstat[i] = *reinterpret_cast<const float2*>(stats + 2 * static_cast<long>(rb + i));
  float gg[V][8], ag[V][8], ab[V][8], ao[V][8];
#pragma unroll
  for (int k = 0; k < V; ++k) {
#pragma unroll
    for (int j = 0; j < 8; ++j) { gg[k][j] = 0.f; ag[k][j] = 0.f; ab[k][j] = 0.f; ao[k][j] = 0.f; }
    if (act[k]) load8(g + (t + k * nt) * 8, gg[k]);
  }
  __syncthreads();
  const float inv_n = 1.f / n;
  for (int r0 = rb, it = 0; r0 < re; r0 += R, ++it) {
    const int par = it & 1;
    float sg[R], sgx[R];
#pragma unroll
    for (int q = 0; q < R; ++q) {
      const int u = it * R + q, sl = u % S;
      sg[q] = 0.f; sgx[q] = 0.f;
      if (r0 + q >= re) continue;
      const uint8_t* buf = stage0 + static_cast<size_t>(sl) * sb;
      const float2 ms = sstat[u];
      mbar_wait(&bar[sl], (u / S) & 1);
      float2 a_sg = f2(0.f, 0.f), a_sgx = f2(0.f, 0.f);
#pragma unroll
      for (int k = 0; k < V; ++k) {
        if (!act[k]) continue;
        const int off = (t + k * nt) * 16;
        float d[8], xh[8];
        unpack8(lds128(buf + off), d);
        unpack8(lds128(buf + row_bytes + off), xh);
#pragma unroll
        for (int j = 0; j < 8; j += 2) {
          const float2 dd = f2(d[j], d[j + 1]);
          const float2 xx = mul2(add2(f2(xh[j], xh[j + 1]), f2(-ms.x, -ms.x)), f2(ms.y, ms.y));
          const float2 gp = mul2(dd, f2(gg[k][j], gg[k][j + 1]));
          a_sg = add2(a_sg, gp);
          a_sgx = fma2(gp, xx, a_sgx);
          const float2 na = fma2(dd, xx, f2(ag[k][j], ag[k][j + 1]));
          const float2 nb = add2(f2(ab[k][j], ab[k][j + 1]), dd);
          ag[k][j] = na.x; ag[k][j + 1] = na.y; ab[k][j] = nb.x; ab[k][j + 1] = nb.y;
        }
      }
      sg[q] = a_sg.x + a_sg.y;
      sgx[q] = a_sgx.x + a_sgx.y;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
      for (int q = 0; q < R; ++q) {
        sg[q] += __shfl_xor_sync(0xffffffffu, sg[q], o);
        sgx[q] += __shfl_xor_sync(0xffffffffu, sgx[q], o);
      }
    }
    float* rp = red + par * (32 * R * 2);
    if (lane == 0) {
#pragma unroll
      for (int q = 0; q < R; ++q) { rp[(w * R + q) * 2] = sg[q]; rp[(w * R + q) * 2 + 1] = sgx[q]; }
    }
    __syncthreads();
    // every thread is past phase 2 of the previous iteration: refill its slots
    if (t == 0 && it > 0) {
#pragma unroll
      for (int q = 0; q < R; ++q) {
        const int u = (it - 1) * R + q, rn = rb + u + S;
        if (rn < re) issue(u % S, rn);
      }
    }
    float tg[R], tgx[R];
    cross_warp_sums<R>(rp, nw, lane, tg, tgx);
#pragma unroll
    for (int q = 0; q < R; ++q) {
      const int r = r0 + q;
      if (r >= re) break;
      const int u = it * R + q;
      const uint8_t* buf = stage0 + static_cast<size_t>(u % S) * sb;
      const float2 ms = sstat[u];
      const float mg = rms ? 0.f : tg[q] * inv_n, mgx = tgx[q] * inv_n;
#pragma unroll
      for (int k = 0; k < V; ++k) {
        if (!act[k]) continue;
        const int cidx = t + k * nt, off = cidx * 16;
        float d[8], xh[8], rr[8];
        unpack8(lds128(buf + off), d);
        unpack8(lds128(buf + row_bytes + off), xh);
        if (RES == 1) {
          unpack8(lds128(buf + 2 * row_bytes + off), rr);
        } else if (RES == 2) {
          const float4 r0 = *reinterpret_cast<const float4*>(buf + 2 * row_bytes + 2 * off);
          const float4 r1 = *reinterpret_cast<const float4*>(buf + 2 * row_bytes + 2 * off + 16);
          rr[0] = r0.x; rr[1] = r0.y; rr[2] = r0.z; rr[3] = r0.w;
          rr[4] = r1.x; rr[5] = r1.y; rr[6] = r1.z; rr[7] = r1.w;
        } else {
#pragma unroll
          for (int j = 0; j < 8; ++j) rr[j] = 0.f;
        }
        float o[8];
#pragma unroll
        for (int j = 0; j < 8; j += 2) {
          const float2 xhat = mul2(add2(f2(xh[j], xh[j + 1]), f2(-ms.x, -ms.x)), f2(ms.y, ms.y));
          const float2 uu = add2(mul2(f2(d[j], d[j + 1]), f2(gg[k][j], gg[k][j + 1])), f2(-mg, -mg));
          const float2 ww = fma2(xhat, f2(-mgx, -mgx), uu);
          const float2 res = fma2(ww, f2(ms.y, ms.y), f2(rr[j], rr[j + 1]));
          o[j] = res.x; o[j + 1] = res.y;
        }
        const uint4 pk = pack8(o);
        *reinterpret_cast<uint4*>(dx + static_cast<long>(r) * n + cidx * 8) = pk;
        if (OUT32) {
          float* d32 = dx32 + static_cast<long>(r) * n + cidx * 8;
          *reinterpret_cast<float4*>(d32) = make_float4(o[0], o[1], o[2], o[3]);
          *reinterpret_cast<float4*>(d32 + 4) = make_float4(o[4], o[5], o[6], o[7]);
        }
        if (sum_out) {
          float qv[8];
          if (OUT32) {
#pragma unroll
            for (int j = 0; j < 8; ++j) qv[j] = o[j];
          } else {
            unpack8(pk, qv);
          }
#pragma unroll
          for (int j = 0; j < 8; j += 2) {
            const float2 a = add2(f2(ao[k][j], ao[k][j + 1]), f2(qv[j], qv[j + 1]));
            ao[k][j] = a.x; ao[k][j + 1] = a.y;
          }
        }
      }
    }
  }
  if (!partial) return;
#pragma unroll
  for (int k = 0; k < V; ++k) {
    if (!act[k]) continue;
    const int c = (t + k * nt) * 8;
    float* p0 = partial + static_cast<long>(blockIdx.x) * n + c;
    *reinterpret_cast<float4*>(p0) = make_float4(ag[k][0], ag[k][1], ag[k][2], ag[k][3]);
    *reinterpret_cast<float4*>(p0 + 4) = make_float4(ag[k][4], ag[k][5], ag[k][6], ag[k][7]);
    if (!rms) {
      float* p1 = partial + static_cast<long>(nblk + blockIdx.x) * n + c;
      *reinterpret_cast<float4*>(p1) = make_float4(ab[k][0], ab[k][1], ab[k][2], ab[k][3]);
      *reinterpret_cast<float4*>(p1 + 4) = make_float4(ab[k][4], ab[k][5], ab[k][6], ab[k][7]);
    }
    if (sum_out) {
      float* p2 = partial + static_cast<long>(2 * nblk + blockIdx.x) * n + c;
      *reinterpret_cast<float4*>(p2) = make_float4(ao[k][0], ao[k][1], ao[k][2], ao[k][3]);
      *reinterpret_cast<float4*>(p2 + 4) = make_float4(ao[k][4], ao[k][5], ao[k][6], ao[k][7]);
    }
  }
}

// ---------------------------------------------------------------- softmax-CE
// One CTA (512 threads) per row; the whole fp32 row is held in registers (thread t: float4 chunks
// t, t + 512, ...), so the logits are read from HBM exactly once: block max, then p = 2^((z-M)log2e)
// kept in place, block sum, dlogits = (p / sum - [c == y]) / Ntok written as bf16, row_loss =
// log(sum) + M - z_y.
template <int NV>
__global__ void __launch_bounds__(512, 1) softmax_ce_reg_k(const float* __restrict__ logits,
                                                           const int32_t* __restrict__ tok, int ld_tok, int s, int V,
                                                           float inv_ntok, bf16* __restrict__ dlogits,
                                                           float* __restrict__ row_loss, long row0) {
  __shared__ float red[2][16];
  constexpr float LOG2E = 1.4426950408889634f;
  const long r = blockIdx.x;
  const int t = threadIdx.x, w = t / 32, lane = t % 32;
  const int nv4 = V / 4;
  const float4* z = reinterpret_cast<const float4*>(logits + r * V);
  const int bi = static_cast<int>((row0 + r) / s), ti = static_cast<int>((row0 + r) % s);
  const int y = tok[static_cast<long>(bi) * ld_tok + ti + 1];
  float zy = 0.f;
  if (t == 0) zy = logits[r * V + y];
  float4 v[NV];
  float m = -INFINITY;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = t + i * 512;
    v[i] = c < nv4 ? z[c] : make_float4(-INFINITY, -INFINITY, -INFINITY, -INFINITY);
    m = fmaxf(m, fmaxf(fmaxf(v[i].x, v[i].y), fmaxf(v[i].z, v[i].w)));
  }
  m = wmax(m);
  if (lane == 0) red[0][w] = m;
  __syncthreads();
  float M = red[0][0];
#pragma unroll
  for (int i = 1; i < 16; ++i) M = fmaxf(M, red[0][i]);
  const float ml = M * LOG2E;
  float l = 0.f;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    v[i].x = exp2f(fmaf(v[i].x, LOG2E, -ml));
    v[i].y = exp2f(fmaf(v[i].y, LOG2E, -ml));
    v[i].z = exp2f(fmaf(v[i].z, LOG2E, -ml));
    v[i].w = exp2f(fmaf(v[i].w, LOG2E, -ml));
    l += (v[i].x + v[i].y) + (v[i].z + v[i].w);
  }
  l = wsum(l);
  if (lane == 0) red[1][w] = l;
  __syncthreads();
  float L = 0.f;
#pragma unroll
  for (int i = 0; i < 16; ++i) L += red[1][i];
  const float sc = inv_ntok / L;
  uint2* out = reinterpret_cast<uint2*>(dlogits + r * V);
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = t + i * 512;
    if (c < nv4) {
      const int c0 = 4 * c;
      const float a = v[i].x * sc - (c0 == y ? inv_ntok : 0.f);
      const float b = v[i].y * sc - (c0 + 1 == y ? inv_ntok : 0.f);
      const float cc = v[i].z * sc - (c0 + 2 == y ? inv_ntok : 0.f);
      const float d = v[i].w * sc - (c0 + 3 == y ? inv_ntok : 0.f);
      uint2 u;
      *reinterpret_cast<__nv_bfloat162*>(&u.x) = __floats2bfloat162_rn(a, b);
      *reinterpret_cast<__nv_bfloat162*>(&u.y) = __floats2bfloat162_rn(cc, d);
      out[c] = u;
    }
  }
  if (t == 0) row_loss[r] = (M + logf(L)) - zy;
}

template <class K>
int occ_grid(K kernel, int threads, size_t smem) {
  int occ = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, smem);
  return device_sms() * (occ < 1 ? 1 : occ);
}
inline int threads_for(int n) { return ((n / 8 + 31) / 32) * 32; }
inline int cdivl(long a, long b) { return static_cast<int>((a + b - 1) / b); }
}  // namespace

// Backward recompute of a norm output from the forward's stored row statistics (the lean activation
// set keeps x and (mean, rstd), not y): y = (x - mean) * rstd * g + b, the forward kernel's exact
// expression, as one streaming pass without row reductions. Thread i owns 16-byte vectors i and
// i + nthreads (both loads issued before any math).
__global__ void __launch_bounds__(256) norm_apply_k(const bf16* __restrict__ x, const float* __restrict__ g,
                                                    const float* __restrict__ b, const float* __restrict__ stats,
                                                    bf16* __restrict__ y, long nvec, int nv_row) {
  const long stride = static_cast<long>(gridDim.x) * blockDim.x;
  const long i0 = static_cast<long>(blockIdx.x) * blockDim.x + threadIdx.x;
  uint4 u[2];
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const long i = i0 + k * stride;
    if (i < nvec) u[k] = __ldg(reinterpret_cast<const uint4*>(x) + i);
  }
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const long i = i0 + k * stride;
    if (i >= nvec) break;
    const long r = i / nv_row;
    const int c = static_cast<int>(i - r * nv_row) * 8;
    const float2 ms = __ldg(reinterpret_cast<const float2*>(stats) + r);
    float v[8], gg[8], bb[8], o[8];
    unpack8(u[k], v);
    load8(g + c, gg);
    if (b) load8(b + c, bb);
    else {
#pragma unroll
      for (int j = 0; j < 8; ++j) bb[j] = 0.f;
    }
    norm_out8(v, ms.x, ms.y, gg, bb, o);
    reinterpret_cast<uint4*>(y)[i] = pack8(o);
  }
}

// The same recompute with the column chunk fixed per thread (a 2-D grid: x over 16-byte column
// vectors, y over groups of RPT rows): g / b are loaded once, the RPT rows' x vectors are all in
// flight before any math, and no per-vector row division (the 1-D kernel's 64-bit i / nv_row per
// vector kept it issue-bound: ncu SM 29%, DRAM 23%). Same expression, bitwise the same output.
template <int RPT>
__global__ void __launch_bounds__(256) norm_apply2_k(const bf16* __restrict__ x, const float* __restrict__ g,
                                                     const float* __restrict__ b, const float* __restrict__ stats,
                                                     bf16* __restrict__ y, int rows, int nv_row) {
  const int cv = blockIdx.x * blockDim.x + threadIdx.x;
  if (cv >= nv_row) return;
  const int r0 = blockIdx.y * RPT;
  uint4 u[RPT];
#pragma unroll
  for (int k = 0; k < RPT; ++k)
    if (r0 + k < rows) u[k] = __ldg(reinterpret_cast<const uint4*>(x) + static_cast<long>(r0 + k) * nv_row + cv);
  float gg[8], bb[8];
  load8(g + cv * 8, gg);
  if (b) load8(b + cv * 8, bb);
  else {
#pragma unroll
    for (int j = 0; j < 8; ++j) bb[j] = 0.f;
  }
#pragma unroll
  for (int k = 0; k < RPT; ++k) {
    const int r = r0 + k;
    if (r >= rows) break;
    const float2 ms = __ldg(reinterpret_cast<const float2*>(stats) + r);
    float v[8], o[8];
    unpack8(u[k], v);
    norm_out8(v, ms.x, ms.y, gg, bb, o);
    reinterpret_cast<uint4*>(y)[static_cast<long>(r) * nv_row + cv] = pack8(o);
  }
}

bool norm_apply(const bf16* x, const float* g, const float* b, const float* stats, bf16* y, int rows, int n,
                cudaStream_t st) {
  if (n % 8 != 0 || (reinterpret_cast<uintptr_t>(x) & 15) || (reinterpret_cast<uintptr_t>(y) & 15)) return false;
  const long nvec = static_cast<long>(rows) * (n / 8);
  if (nvec <= 0) return true;
  static const int v2 = getenv("MARIO_NORM_APPLY") ? atoi(getenv("MARIO_NORM_APPLY")) : 2;
  if (v2 == 2 && (rows + 3) / 4 <= 65535) {
    constexpr int RPT = 4;
    const int nv_row = n / 8, bx = nv_row < 256 ? ((nv_row + 31) / 32) * 32 : 256;
    dim3 grid(cdivl(nv_row, bx), cdivl(rows, RPT));
    norm_apply2_k<RPT><<<grid, bx, 0, st>>>(x, g, b, stats, y, rows, nv_row);
    note_launch();
    return true;
  }
  const long thr = (nvec + 1) / 2;
  norm_apply_k<<<cdivl(thr, 256), 256, 0, st>>>(x, g, b, stats, y, nvec, n / 8);
  note_launch();
  return true;
}

bool norm_pipe_supported(int n) { return n % 8 == 0 && n >= 8 && n <= 8192; }

// ------------------------------------------------------------ forward, warp per row (v2)
// norm_fwd_warp_k: a persistent grid of 8-warp CTAs; warp w takes RPW rows at a time (rows
// RPW*w, RPW*(w + nwarps), ...). Lane l owns the 16-byte chunks l, l + 32, ... of a row (NC per
// row, coalesced 512-byte warp accesses), all loads of the RPW rows are issued before any math
// (ld.global.nc, no L1 allocation: L1 keeps g / b, which the RPW rows of a chunk share). Row
// statistics are shifted one-pass sums from registers (below; RMS: var = sum(x^2)/n), warp
// butterflies only: no shared memory, no block barrier, no mbarrier
// polling (the row-pipelined kernel above spent ~1700 warp instructions per 2048-wide row on
// those; this one ~330). Output = norm_out8, the expression norm_apply recomputes with.
__device__ __forceinline__ uint4 ldg_nc_na(const void* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ float2 bf2f2(uint32_t u) {
  return make_float2(__uint_as_float(u << 16), __uint_as_float(u & 0xffff0000u));
}
__device__ __forceinline__ float wsum_bfly(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
template <bool RMS, int NC, int RPW>
__global__ void __launch_bounds__(256, (NC * RPW <= 16 ? 2 : 1)) norm_fwd_warp_k(const bf16* __restrict__ x, const float* __restrict__ g,
                                                       const float* __restrict__ b, bf16* __restrict__ y,
                                                       float* __restrict__ stats, int rows, int n, float eps) {
  const int lane = threadIdx.x & 31;
  const int nwarps = gridDim.x * (blockDim.x >> 5);
  const float inv_n = 1.f / n;
  for (int r0 = (blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * RPW; r0 < rows; r0 += nwarps * RPW) {
    uint4 v[RPW][NC];
#pragma unroll
    for (int q = 0; q < RPW; ++q) {
      const bf16* xr = x + static_cast<long>(r0 + q) * n;
#pragma unroll
      for (int i = 0; i < NC; ++i) {
        const int c = (i * 32 + lane) * 8;
        v[q][i] = (r0 + q < rows && c < n) ? ldg_nc_na(xr + c) : make_uint4(0u, 0u, 0u, 0u);
      }
    }
    // one pass, shifted by the row's first element K (as the row-pipelined kernel): S1 = sum(x - K),
    // S2 = sum((x - K)^2), mean = K + S1/n, var = S2/n - (S1/n)^2 -- the cancellation is relative to
    // |mean - K|, about one standard deviation; each packed value is converted once (a two-pass form
    // keeps NC*8 floats per row live: 138 registers, 1 CTA per SM). Padding chunks are skipped.
    float mean[RPW], rstd[RPW];
#pragma unroll
    for (int q = 0; q < RPW; ++q) {
      const float K = RMS ? 0.f : __uint_as_float(__shfl_sync(0xffffffffu, v[q][0].x, 0) << 16);
      float2 a1 = f2(0.f, 0.f), a2 = f2(0.f, 0.f);
#pragma unroll
      for (int i = 0; i < NC; ++i) {
        if ((i * 32 + lane) * 8 >= n) continue;
        const uint32_t w4[4] = {v[q][i].x, v[q][i].y, v[q][i].z, v[q][i].w};
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const float2 d = RMS ? bf2f2(w4[k]) : add2(bf2f2(w4[k]), f2(-K, -K));
          if (!RMS) a1 = add2(a1, d);
          a2 = fma2(d, d, a2);
        }
      }
      const float S2 = wsum_bfly(a2.x + a2.y) * inv_n;
      if (RMS) {
        mean[q] = 0.f;
        rstd[q] = rsqrtf(S2 + eps);
      } else {
        const float m1 = wsum_bfly(a1.x + a1.y) * inv_n;
        mean[q] = K + m1;
        rstd[q] = rsqrtf(fmaxf(S2 - m1 * m1, 0.f) + eps);
      }
    }
#pragma unroll
    for (int i = 0; i < NC; ++i) {
      const int c = (i * 32 + lane) * 8;
      if (c >= n) continue;
      float gg[8], bb[8];
      load8(g + c, gg);
      if (!RMS) load8(b + c, bb);
      else {
#pragma unroll
        for (int j = 0; j < 8; ++j) bb[j] = 0.f;
      }
#pragma unroll
      for (int q = 0; q < RPW; ++q) {
        if (r0 + q >= rows) break;
        float vv[8], o[8];
        unpack8(v[q][i], vv);
        norm_out8(vv, mean[q], rstd[q], gg, bb, o);
        *reinterpret_cast<uint4*>(y + static_cast<long>(r0 + q) * n + c) = pack8(o);
      }
    }
    if (lane == 0) {
#pragma unroll
      for (int q = 0; q < RPW; ++q)
        if (r0 + q < rows) *reinterpret_cast<float2*>(stats + 2 * static_cast<long>(r0 + q)) = make_float2(mean[q], rstd[q]);
    }
  }
}

template <bool RMS, int NC, int RPW>
void norm_fwd_warp_launch(const bf16* x, const float* g, const float* b, bf16* y, float* stats, int rows, int n,
                          float eps, cudaStream_t st) {
  const int need = cdivl(rows, 8 * RPW);
  int grid = occ_grid(norm_fwd_warp_k<RMS, NC, RPW>, 256, 0);
  grid = grid < need ? grid : need;
  norm_fwd_warp_k<RMS, NC, RPW><<<grid, 256, 0, st>>>(x, g, b, y, stats, rows, n, eps);
  note_launch();
}


template <int kPipeR>
bool norm_fwd_pipe_r(const bf16* x, const float* g, const float* b, bf16* y, float* stats, int rows, int n, float eps,
                     int rms, cudaStream_t st) {
  const int nt = threads_for(n), sb = n * 2;
  // ring bytes / max stages per CTA (MARIO_NORM_FWD_RING, MARIO_NORM_FWD_SMAX: tuning experiments)
  static const int ring = getenv("MARIO_NORM_FWD_RING") ? atoi(getenv("MARIO_NORM_FWD_RING")) : 24576;
  static const int smax = getenv("MARIO_NORM_FWD_SMAX") ? atoi(getenv("MARIO_NORM_FWD_SMAX")) : 8;
  int S = ring / sb;
  S = S < 2 * kPipeR ? 2 * kPipeR : (S > smax ? smax : S);
  S -= S % kPipeR;
  const size_t smem = pipe_smem_bytes(S, sb, kPipeR);
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(norm_fwd_pipe_k<false, kPipeR>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(norm_fwd_pipe_k<true, kPipeR>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    attr = true;
  }
  int nblk = rms ? occ_grid(norm_fwd_pipe_k<true, kPipeR>, nt, smem) : occ_grid(norm_fwd_pipe_k<false, kPipeR>, nt, smem);
  nblk = nblk < rows ? nblk : rows;
  if (rms) norm_fwd_pipe_k<true, kPipeR><<<nblk, nt, smem, st>>>(x, g, b, y, stats, rows, n, eps, S, nblk);
  else norm_fwd_pipe_k<false, kPipeR><<<nblk, nt, smem, st>>>(x, g, b, y, stats, rows, n, eps, S, nblk);
  note_launch();
  return true;
}

bool norm_fwd_pipe(const bf16* x, const float* g, const float* b, bf16* y, float* stats, int rows, int n, float eps,
                   int rms, cudaStream_t st) {
  if (!norm_pipe_supported(n)) return false;
  if (rows <= 0) return true;
  if (n > 5120) return norm_fwd_pipe_r<2>(x, g, b, y, stats, rows, n, eps, rms, st);   // R 4 / 8: <= 640 threads
  switch (norm_rows_per_iter(true)) {
    case 8: return norm_fwd_pipe_r<8>(x, g, b, y, stats, rows, n, eps, rms, st);
    case 4: return norm_fwd_pipe_r<4>(x, g, b, y, stats, rows, n, eps, rms, st);
    default: return norm_fwd_pipe_r<2>(x, g, b, y, stats, rows, n, eps, rms, st);
  }
}

bool norm_fwd_warp(const bf16* x, const float* g, const float* b, bf16* y, float* stats, int rows, int n, float eps,
                   int rms, cudaStream_t st) {
  if (n % 8 != 0 || n > 8192 || (reinterpret_cast<uintptr_t>(x) & 15) || (reinterpret_cast<uintptr_t>(y) & 15))
    return false;
  if (rows <= 0) return true;
  const int nc = cdivl(n, 256);
#define NFW_CASE(NC, RPW)                                                                   \
  if (nc <= NC) {                                                                           \
    if (rms) norm_fwd_warp_launch<true, NC, RPW>(x, g, b, y, stats, rows, n, eps, st);      \
    else norm_fwd_warp_launch<false, NC, RPW>(x, g, b, y, stats, rows, n, eps, st);         \
    return true;                                                                            \
  }
  NFW_CASE(1, 2)
  NFW_CASE(2, 2)
  NFW_CASE(4, 2)
  NFW_CASE(8, 2)
  NFW_CASE(16, 1)
  NFW_CASE(20, 1)
  NFW_CASE(32, 1)
#undef NFW_CASE
  return false;
}

template <int V, int RES, bool OUT32, int kPipeR>
bool norm_bwd_pipe_vr(const bf16* dy, const bf16* x, const float* stats, const float* g, const void* dres, bf16* dx,
                     float* dx32, int rows, int n, int rms, float* dg, float* db, float* dsum, float* partial,
                     size_t partial_floats, cudaStream_t st) {
  const int nt = ((n / (8 * V) + 31) / 32) * 32, sb = 4 * n + (RES == 2 ? 4 * n : (RES == 1 ? 2 * n : 0));
  if (nt > 640) return false;
  static const int ring = getenv("MARIO_NORM_BWD_RING") ? atoi(getenv("MARIO_NORM_BWD_RING")) : 49152;
  static const int smax = getenv("MARIO_NORM_BWD_SMAX") ? atoi(getenv("MARIO_NORM_BWD_SMAX")) : 6;
  int S = ring / sb;
  S = S < 2 * kPipeR ? 2 * kPipeR : (S > smax ? smax : S);
  S -= S % kPipeR;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(norm_bwd_pipe_k<kPipeR, V, RES, OUT32>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         220 * 1024);
    attr = true;
  }
  // the stats of a CTA's range are staged in shared memory: size for the smallest grid we may use
  const size_t base = pipe_smem_bytes(S, sb, kPipeR);
  int nblk = occ_grid(norm_bwd_pipe_k<kPipeR, V, RES, OUT32>, nt,
                      base + 8 * static_cast<size_t>(cdivl(rows, device_sms())));
  // CTAs per SM cap (MARIO_NORM_BWD_CPS, A/B: fewer CTAs = fewer column-sum partials to reduce)
  static const int cps = getenv("MARIO_NORM_BWD_CPS") ? atoi(getenv("MARIO_NORM_BWD_CPS")) : 0;
  if (cps > 0 && nblk > cps * device_sms()) nblk = cps * device_sms();
  if (dg) {
    const long cap = static_cast<long>(partial_floats / (3 * static_cast<size_t>(n)));
    if (cap < 1) return false;
    nblk = nblk < cap ? nblk : static_cast<int>(cap);
  }
  nblk = nblk < rows ? nblk : rows;
  const int max_range = cdivl(rows, nblk) + 1;
  const size_t smem = base + 8 * static_cast<size_t>(max_range);
  if (smem > 220 * 1024) return false;
  norm_bwd_pipe_k<kPipeR, V, RES, OUT32><<<nblk, nt, smem, st>>>(dy, x, stats, g, dres, dx, dx32, rows, n, rms,
                                                                 dg ? partial : nullptr, nblk, dsum ? 1 : 0, S,
                                                                 max_range);
  note_launch();
  if (dg) {
    colsum_reduce(partial, nblk, n, dg, rms ? nullptr : db, dsum, st);
  }
  return true;
}

template <int V, int RES, bool OUT32>
bool norm_bwd_pipe_v(const bf16* dy, const bf16* x, const float* stats, const float* g, const void* dres, bf16* dx,
                     float* dx32, int rows, int n, int rms, float* dg, float* db, float* dsum, float* partial,
                     size_t partial_floats, cudaStream_t st) {
  if (norm_rows_per_iter(false) == 4)
    return norm_bwd_pipe_vr<V, RES, OUT32, 4>(dy, x, stats, g, dres, dx, dx32, rows, n, rms, dg, db, dsum, partial,
                                              partial_floats, st);
  return norm_bwd_pipe_vr<V, RES, OUT32, 2>(dy, x, stats, g, dres, dx, dx32, rows, n, rms, dg, db, dsum, partial,
                                            partial_floats, st);
}

bool norm_bwd_pipe(const bf16* dy, const bf16* x, const float* stats, const float* g, const bf16* dres, bf16* dx,
                   int rows, int n, int rms, float* dg, float* db, float* dsum, float* partial, size_t partial_floats,
                   cudaStream_t st) {
  if (!norm_pipe_supported(n)) return false;
  if (rows <= 0) return true;
  // 16-byte chunks per thread (MARIO_NORM_BWD_V)
  static const int vsel = getenv("MARIO_NORM_BWD_V") ? atoi(getenv("MARIO_NORM_BWD_V")) : 2;
  if (vsel == 2 && n % 2048 == 0)   // measured: h 4096 73.8 -> 63.9 us, h 2048 equal, h 5120 slower
    return dres ? norm_bwd_pipe_v<2, 1, false>(dy, x, stats, g, dres, dx, nullptr, rows, n, rms, dg, db, dsum, partial,
                                                partial_floats, st)
                : norm_bwd_pipe_v<2, 0, false>(dy, x, stats, g, nullptr, dx, nullptr, rows, n, rms, dg, db, dsum,
                                                partial, partial_floats, st);
  return dres ? norm_bwd_pipe_v<1, 1, false>(dy, x, stats, g, dres, dx, nullptr, rows, n, rms, dg, db, dsum, partial,
                                              partial_floats, st)
              : norm_bwd_pipe_v<1, 0, false>(dy, x, stats, g, nullptr, dx, nullptr, rows, n, rms, dg, db, dsum, partial,
                                              partial_floats, st);
}

bool norm_bwd_pipe_mixed(const bf16* dy, const bf16* x, const float* stats, const float* g, const bf16* dres,
                         const float* dres32, bf16* dx, float* dx32, int rows, int n, int rms, float* dg, float* db,
                         float* dsum, float* partial, size_t partial_floats, cudaStream_t st) {
  if (!norm_pipe_supported(n)) return false;
  if (rows <= 0) return true;
  static const int vsel = getenv("MARIO_NORM_BWD_V") ? atoi(getenv("MARIO_NORM_BWD_V")) : 2;
  const bool v2 = vsel == 2 && n % 2048 == 0;
#define NB_CASE(VV, RR, OO, DR)                                                                                  \
  return norm_bwd_pipe_v<VV, RR, OO>(dy, x, stats, g, DR, dx, dx32, rows, n, rms, dg, db, dsum, partial,        \
                                     partial_floats, st)
  if (v2) {
    if (dres32) { if (dx32) NB_CASE(2, 2, true, dres32); NB_CASE(2, 2, false, dres32); }
    if (dres) { if (dx32) NB_CASE(2, 1, true, dres); NB_CASE(2, 1, false, dres); }
    if (dx32) NB_CASE(2, 0, true, nullptr);
    NB_CASE(2, 0, false, nullptr);
  }
  if (dres32) { if (dx32) NB_CASE(1, 2, true, dres32); NB_CASE(1, 2, false, dres32); }
  if (dres) { if (dx32) NB_CASE(1, 1, true, dres); NB_CASE(1, 1, false, dres); }
  if (dx32) NB_CASE(1, 0, true, nullptr);
  NB_CASE(1, 0, false, nullptr);
#undef NB_CASE
}

bool softmax_ce_fast(const float* logits, const int32_t* tok, int ld_tok, int s, int rows, int V, float inv_ntok,
                     bf16* dlogits, float* row_loss, cudaStream_t st, long row0) {
  if (V % 4 || V < 4) return false;
  const int need = cdivl(V / 4, 512);
  if (rows <= 0) return true;
#define CE_CASE(NV)                                                                                            \
  if (need <= NV) {                                                                                            \
    softmax_ce_reg_k<NV><<<rows, 512, 0, st>>>(logits, tok, ld_tok, s, V, inv_ntok, dlogits, row_loss, row0);  \
    note_launch();                                                                                             \
    return true;                                                                                               \
  }
  CE_CASE(1)
  CE_CASE(2)
  CE_CASE(4)
  CE_CASE(8)
  CE_CASE(16)
  CE_CASE(25)
#undef CE_CASE
  return false;
}

}  // namespace mario
