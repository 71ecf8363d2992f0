// K5/K6: causal flash attention forward/backward for bf16 on tensor cores
// (mma.sync m16n8k16, fp32 accumulate; P kept in registers). Definition: SURVEY §8(c) c1
// (S = QK^T/sqrt(dh), causal mask, softmax, O = PV; dS = P*(dP - rowsum(dO*O))).
// Deterministic backward: dK/dV by key tiles and dQ by query tiles in separate passes (no
// atomics), so recomputation and rescheduling reproduce every bit.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "layers.h"
#include "kstats.h"

namespace mario {

int g_attn_variant = -1;   // mario_k_attn_set_variant: -1 auto (tcgen05 where supported), 0 mma.sync only

namespace {

using bf16 = __nv_bfloat16;
constexpr int BR = 64;       // rows (queries or keys) per CTA, 16 per warp
constexpr int BC = 64;       // columns per inner tile (forward)
constexpr int BCB = 32;      // columns per inner tile (backward: keeps dK/dV/dQ in registers)
constexpr float LOG2E = 1.4426950408889634f;

__device__ __forceinline__ uint32_t smem_addr(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

__device__ __forceinline__ void ldsm_x4(uint32_t (&r)[4], const bf16* p) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(smem_addr(p)));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t (&r)[4], const bf16* p) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(smem_addr(p)));
}
__device__ __forceinline__ void mma16816(float (&c)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
               : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
               : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t pack_bf16(float lo, float hi) {
  __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&v);
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" :: "r"(smem_addr(dst)), "l"(src), "r"(valid ? 16 : 0));
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
}

// Load rows [r0, r0+64) (clamped to s) of a [s][ld] bf16 matrix slice of width D into smem
// with row pitch D+8 elements; rows >= s are zero-filled.
template <int D, int ROWS = 64>
__device__ __forceinline__ void load_tile(bf16* sm, const bf16* g, int r0, int s, int ld) {
  constexpr int LDS = D + 8, CH = D / 8;   // 16-byte chunks per row
  for (int i = threadIdx.x; i < ROWS * CH; i += blockDim.x) {
    const int r = i / CH, c = i % CH;
    const bool ok = r0 + r < s;
    const bf16* src = g + static_cast<long>(ok ? r0 + r : 0) * ld + c * 8;
    cp_async16(sm + r * LDS + c * 8, src, ok);
  }
}

// lane -> (row offset, column offset) of ldmatrix.x4 source rows
__device__ __forceinline__ int a_row(int lane) { return lane & 15; }
__device__ __forceinline__ int a_col(int lane) { return (lane >> 4) * 8; }
__device__ __forceinline__ int b_row(int lane) { return (lane & 7) + ((lane >> 4) << 3); }
__device__ __forceinline__ int b_col(int lane) { return ((lane >> 3) & 1) * 8; }

// ------------------------------------------------------------------------ forward
template <int D>
__global__ void __launch_bounds__(128) fa_fwd_k(const bf16* qkv, bf16* O, float* lse, int B, int s, int nh) {
  constexpr int LDS = D + 8;
  extern __shared__ __align__(16) uint8_t smraw[];
  bf16* sQ = reinterpret_cast<bf16*>(smraw);
  bf16* sK = sQ + BR * LDS;
  bf16* sV = sK + BC * LDS;
  const int qt = blockIdx.x, b = blockIdx.y / nh, head = blockIdx.y % nh;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32, g = lane >> 2, t4 = lane & 3;
  const int h = nh * D, ld = 3 * h;
  const long Ttok = static_cast<long>(B) * s;
  const bf16* q = qkv + static_cast<long>(b) * s * ld + head * D;
  const bf16* k = q + h;
  const bf16* v = q + 2 * h;
  const float sl2 = rsqrtf(static_cast<float>(D)) * LOG2E;

  load_tile<D>(sQ, q, qt * BR, s, ld);
  cp_async_wait_all();
  __syncthreads();
  uint32_t qf[D / 16][4];
#pragma unroll
  for (int kk = 0; kk < D / 16; ++kk) ldsm_x4(qf[kk], sQ + (warp * 16 + a_row(lane)) * LDS + kk * 16 + a_col(lane));

  float o[D / 8][4];
#pragma unroll
  for (int i = 0; i < D / 8; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;
  float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
  const int row0 = qt * BR + warp * 16 + g;   // rows row0 and row0 + 8

  for (int j = 0; j <= qt; ++j) {
    __syncthreads();
    load_tile<D>(sK, k, j * BC, s, ld);
    load_tile<D>(sV, v, j * BC, s, ld);
    cp_async_wait_all();
    __syncthreads();
    float sc[8][4];
#pragma unroll
    for (int i = 0; i < 8; ++i) sc[i][0] = sc[i][1] = sc[i][2] = sc[i][3] = 0.f;
#pragma unroll
    for (int kk = 0; kk < D / 16; ++kk) {
#pragma unroll
      for (int nb2 = 0; nb2 < 4; ++nb2) {
        uint32_t bf[4];
        ldsm_x4(bf, sK + (nb2 * 16 + b_row(lane)) * LDS + kk * 16 + b_col(lane));
        mma16816(sc[2 * nb2], qf[kk], bf[0], bf[1]);
        mma16816(sc[2 * nb2 + 1], qf[kk], bf[2], bf[3]);
      }
    }
    float mx[2] = {-INFINITY, -INFINITY};
#pragma unroll
    for (int nb = 0; nb < 8; ++nb)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int col = j * BC + nb * 8 + 2 * t4 + (e & 1);
        const int row = row0 + (e >> 1) * 8;
        float x = sc[nb][e] * sl2;
        if (col > row) x = -INFINITY;
        sc[nb][e] = x;
        mx[e >> 1] = fmaxf(mx[e >> 1], x);
      }
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 1));
      mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 2));
    }
    float mn[2], corr[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      mn[r] = fmaxf(m[r], mx[r]);
      corr[r] = exp2f(m[r] - mn[r]);
      l[r] *= corr[r];
      m[r] = mn[r];
    }
#pragma unroll
    for (int i = 0; i < D / 8; ++i) { o[i][0] *= corr[0]; o[i][1] *= corr[0]; o[i][2] *= corr[1]; o[i][3] *= corr[1]; }
#pragma unroll
    for (int nb = 0; nb < 8; ++nb)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float p = exp2f(sc[nb][e] - mn[e >> 1]);
        sc[nb][e] = p;
        l[e >> 1] += p;
      }
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      uint32_t a[4] = {pack_bf16(sc[2 * kk][0], sc[2 * kk][1]), pack_bf16(sc[2 * kk][2], sc[2 * kk][3]),
                       pack_bf16(sc[2 * kk + 1][0], sc[2 * kk + 1][1]), pack_bf16(sc[2 * kk + 1][2], sc[2 * kk + 1][3])};
#pragma unroll
      for (int db = 0; db < D / 16; ++db) {
        uint32_t bv[4];
        ldsm_x4_t(bv, sV + (kk * 16 + a_row(lane)) * LDS + db * 16 + a_col(lane));
        mma16816(o[2 * db], a, bv[0], bv[1]);
        mma16816(o[2 * db + 1], a, bv[2], bv[3]);
      }
    }
  }
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    l[r] += __shfl_xor_sync(0xffffffffu, l[r], 1);
    l[r] += __shfl_xor_sync(0xffffffffu, l[r], 2);
  }
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int row = row0 + r * 8;
    if (row >= s) continue;
    const float inv = 1.f / l[r];
    bf16* orow = O + (static_cast<long>(b) * s + row) * h + head * D;
#pragma unroll
    for (int db = 0; db < D / 8; ++db)
      *reinterpret_cast<__nv_bfloat162*>(orow + db * 8 + 2 * t4) =
          __floats2bfloat162_rn(o[db][2 * r] * inv, o[db][2 * r + 1] * inv);
    if (t4 == 0) lse[static_cast<long>(head) * Ttok + static_cast<long>(b) * s + row] = (m[r] + log2f(l[r])) / LOG2E;
  }
}

// ------------------------------------------------------- backward preprocessing
__global__ void fa_bwd_dot_k(const bf16* O, const bf16* dO, float* Dd, long Ttok, int nh, int dh) {
  const long gw = (static_cast<long>(blockIdx.x) * blockDim.x + threadIdx.x) / 32;
  const int lane = threadIdx.x % 32;
  if (gw >= Ttok * nh) return;
  const int head = static_cast<int>(gw % nh);
  const long r = gw / nh;
  const int h = nh * dh;
  float acc = 0.f;
  for (int d = lane; d < dh; d += 32)
    acc += __bfloat162float(O[r * h + head * dh + d]) * __bfloat162float(dO[r * h + head * dh + d]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (lane == 0) Dd[static_cast<long>(head) * Ttok + r] = acc;
}

// D = rowsum(dO * O) with 16-byte loads: G = dh / 8 lanes per (token, head) (G a power of two)
template <int G>
__global__ void fa_bwd_dot_v8_k(const bf16* O, const bf16* dO, float* Dd, long Ttok, int nh) {
  const long gi = static_cast<long>(blockIdx.x) * blockDim.x + threadIdx.x;
  const long pair = gi / G;                 // (token, head), head fastest
  const int sub = static_cast<int>(gi % G);
  const bool ok = pair < Ttok * nh;
  const int head = static_cast<int>(pair % nh);
  const long r = pair / nh;
  const int dh = G * 8, h = nh * dh;
  float acc = 0.f;
  if (ok) {
    const long off = r * h + head * dh + sub * 8;
    const uint4 a = *reinterpret_cast<const uint4*>(O + off), b = *reinterpret_cast<const uint4*>(dO + off);
    const __nv_bfloat162* ha = reinterpret_cast<const __nv_bfloat162*>(&a);
    const __nv_bfloat162* hb = reinterpret_cast<const __nv_bfloat162*>(&b);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 x = __bfloat1622float2(ha[i]), y = __bfloat1622float2(hb[i]);
      acc += x.x * y.x + x.y * y.y;
    }
  }
#pragma unroll
  for (int o = G / 2; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (ok && sub == 0) Dd[static_cast<long>(head) * Ttok + r] = acc;
}

// ---------------------------------------------------- backward: dK, dV per key tile
template <int D>
__global__ void __launch_bounds__(128) fa_bwd_dkdv_k(const bf16* qkv, const bf16* dO, const float* lse, const float* Dd,
                                                     bf16* dqkv, int B, int s, int nh) {
  constexpr int LDS = D + 8;
  extern __shared__ __align__(16) uint8_t smraw[];
  bf16* sK = reinterpret_cast<bf16*>(smraw);
  bf16* sV = sK + BR * LDS;
  bf16* sQ = sV + BR * LDS;
  bf16* sG = sQ + BCB * LDS;
  float* sL = reinterpret_cast<float*>(sG + BCB * LDS);
  float* sD = sL + BCB;
  const int kt = blockIdx.x, b = blockIdx.y / nh, head = blockIdx.y % nh;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32, g = lane >> 2, t4 = lane & 3;
  const int h = nh * D, ld = 3 * h;
  const long Ttok = static_cast<long>(B) * s;
  const bf16* q = qkv + static_cast<long>(b) * s * ld + head * D;
  const bf16* k = q + h;
  const bf16* v = q + 2 * h;
  const bf16* go = dO + static_cast<long>(b) * s * h + head * D;
  const float scale = rsqrtf(static_cast<float>(D));
  const float sl2 = scale * LOG2E;

  load_tile<D>(sK, k, kt * BR, s, ld);
  load_tile<D>(sV, v, kt * BR, s, ld);
  cp_async_wait_all();
  __syncthreads();
  float dk[D / 8][4], dv[D / 8][4];
#pragma unroll
  for (int i = 0; i < D / 8; ++i)
#pragma unroll
    for (int e = 0; e < 4; ++e) dk[i][e] = dv[i][e] = 0.f;
  const int key0 = kt * BR + warp * 16 + g;
  const int nq = (s + BCB - 1) / BCB;
  for (int i = kt * (BR / BCB); i < nq; ++i) {
    __syncthreads();
    load_tile<D, BCB>(sQ, q, i * BCB, s, ld);
    load_tile<D, BCB>(sG, go, i * BCB, s, h);
    for (int c = threadIdx.x; c < BCB; c += blockDim.x) {
      const int qq = i * BCB + c;
      const long r = static_cast<long>(b) * s + qq;
      sL[c] = qq < s ? lse[static_cast<long>(head) * Ttok + r] * LOG2E : 0.f;
      sD[c] = qq < s ? Dd[static_cast<long>(head) * Ttok + r] : 0.f;
    }
    cp_async_wait_all();
    __syncthreads();
    float sc[BCB / 8][4], dp[BCB / 8][4];
#pragma unroll
    for (int n = 0; n < BCB / 8; ++n)
#pragma unroll
      for (int e = 0; e < 4; ++e) sc[n][e] = dp[n][e] = 0.f;
#pragma unroll
    for (int kk = 0; kk < D / 16; ++kk) {
      uint32_t kf[4], vf[4];
      ldsm_x4(kf, sK + (warp * 16 + a_row(lane)) * LDS + kk * 16 + a_col(lane));
      ldsm_x4(vf, sV + (warp * 16 + a_row(lane)) * LDS + kk * 16 + a_col(lane));
#pragma unroll
      for (int nb2 = 0; nb2 < BCB / 16; ++nb2) {
        uint32_t bq[4], bg[4];
        ldsm_x4(bq, sQ + (nb2 * 16 + b_row(lane)) * LDS + kk * 16 + b_col(lane));
        ldsm_x4(bg, sG + (nb2 * 16 + b_row(lane)) * LDS + kk * 16 + b_col(lane));
        mma16816(sc[2 * nb2], kf, bq[0], bq[1]);
        mma16816(sc[2 * nb2 + 1], kf, bq[2], bq[3]);
        mma16816(dp[2 * nb2], vf, bg[0], bg[1]);
        mma16816(dp[2 * nb2 + 1], vf, bg[2], bg[3]);
      }
    }
    // P^T[key][query], dS^T = P^T (dP^T - D_query)
#pragma unroll
    for (int nb = 0; nb < BCB / 8; ++nb)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int c = nb * 8 + 2 * t4 + (e & 1);
        const int qq = i * BCB + c;
        const int key = key0 + (e >> 1) * 8;
        float p = exp2f(sc[nb][e] * sl2 - sL[c]);
        if (qq < key || qq >= s) p = 0.f;
        sc[nb][e] = p;
        dp[nb][e] = p * (dp[nb][e] - sD[c]);
      }
#pragma unroll
    for (int kk = 0; kk < BCB / 16; ++kk) {
      uint32_t ap[4] = {pack_bf16(sc[2 * kk][0], sc[2 * kk][1]), pack_bf16(sc[2 * kk][2], sc[2 * kk][3]),
                        pack_bf16(sc[2 * kk + 1][0], sc[2 * kk + 1][1]), pack_bf16(sc[2 * kk + 1][2], sc[2 * kk + 1][3])};
      uint32_t as[4] = {pack_bf16(dp[2 * kk][0], dp[2 * kk][1]), pack_bf16(dp[2 * kk][2], dp[2 * kk][3]),
                        pack_bf16(dp[2 * kk + 1][0], dp[2 * kk + 1][1]), pack_bf16(dp[2 * kk + 1][2], dp[2 * kk + 1][3])};
#pragma unroll
      for (int db = 0; db < D / 16; ++db) {
        uint32_t bg[4], bq[4];
        ldsm_x4_t(bg, sG + (kk * 16 + a_row(lane)) * LDS + db * 16 + a_col(lane));
        ldsm_x4_t(bq, sQ + (kk * 16 + a_row(lane)) * LDS + db * 16 + a_col(lane));
        mma16816(dv[2 * db], ap, bg[0], bg[1]);
        mma16816(dv[2 * db + 1], ap, bg[2], bg[3]);
        mma16816(dk[2 * db], as, bq[0], bq[1]);
        mma16816(dk[2 * db + 1], as, bq[2], bq[3]);
      }
    }
  }
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int key = key0 + r * 8;
    if (key >= s) continue;
    bf16* krow = dqkv + (static_cast<long>(b) * s + key) * ld + h + head * D;
    bf16* vrow = krow + h;
#pragma unroll
    for (int db = 0; db < D / 8; ++db) {
      *reinterpret_cast<__nv_bfloat162*>(krow + db * 8 + 2 * t4) =
          __floats2bfloat162_rn(dk[db][2 * r] * scale, dk[db][2 * r + 1] * scale);
      *reinterpret_cast<__nv_bfloat162*>(vrow + db * 8 + 2 * t4) = __floats2bfloat162_rn(dv[db][2 * r], dv[db][2 * r + 1]);
    }
  }
}

// ---------------------------------------------------------- backward: dQ per query tile
template <int D>
__global__ void __launch_bounds__(128) fa_bwd_dq_k(const bf16* qkv, const bf16* dO, const float* lse, const float* Dd,
                                                   bf16* dqkv, int B, int s, int nh) {
  constexpr int LDS = D + 8;
  extern __shared__ __align__(16) uint8_t smraw[];
  bf16* sQ = reinterpret_cast<bf16*>(smraw);
  bf16* sG = sQ + BR * LDS;
  bf16* sK = sG + BR * LDS;
  bf16* sV = sK + BCB * LDS;
  const int qt = blockIdx.x, b = blockIdx.y / nh, head = blockIdx.y % nh;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32, g = lane >> 2, t4 = lane & 3;
  const int h = nh * D, ld = 3 * h;
  const long Ttok = static_cast<long>(B) * s;
  const bf16* q = qkv + static_cast<long>(b) * s * ld + head * D;
  const bf16* k = q + h;
  const bf16* v = q + 2 * h;
  const bf16* go = dO + static_cast<long>(b) * s * h + head * D;
  const float scale = rsqrtf(static_cast<float>(D));
  const float sl2 = scale * LOG2E;
  load_tile<D>(sQ, q, qt * BR, s, ld);
  load_tile<D>(sG, go, qt * BR, s, h);
  cp_async_wait_all();
  __syncthreads();
  uint32_t qf[D / 16][4], gf[D / 16][4];
#pragma unroll
  for (int kk = 0; kk < D / 16; ++kk) {
    ldsm_x4(qf[kk], sQ + (warp * 16 + a_row(lane)) * LDS + kk * 16 + a_col(lane));
    ldsm_x4(gf[kk], sG + (warp * 16 + a_row(lane)) * LDS + kk * 16 + a_col(lane));
  }
  const int row0 = qt * BR + warp * 16 + g;
  float Lr[2], Dr[2];
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int row = row0 + r * 8;
    const long gr = static_cast<long>(b) * s + (row < s ? row : 0);
    Lr[r] = lse[static_cast<long>(head) * Ttok + gr] * LOG2E;
    Dr[r] = Dd[static_cast<long>(head) * Ttok + gr];
  }
  float dq[D / 8][4];
#pragma unroll
  for (int i = 0; i < D / 8; ++i) dq[i][0] = dq[i][1] = dq[i][2] = dq[i][3] = 0.f;
  const int jmax = min((qt * BR + BR - 1) / BCB, (s - 1) / BCB);
  for (int j = 0; j <= jmax; ++j) {
    __syncthreads();
    load_tile<D, BCB>(sK, k, j * BCB, s, ld);
    load_tile<D, BCB>(sV, v, j * BCB, s, ld);
    cp_async_wait_all();
    __syncthreads();
    float sc[BCB / 8][4], dp[BCB / 8][4];
#pragma unroll
    for (int n = 0; n < BCB / 8; ++n)
#pragma unroll
      for (int e = 0; e < 4; ++e) sc[n][e] = dp[n][e] = 0.f;
#pragma unroll
    for (int kk = 0; kk < D / 16; ++kk) {
#pragma unroll
      for (int nb2 = 0; nb2 < BCB / 16; ++nb2) {
        uint32_t bk[4], bv[4];
        ldsm_x4(bk, sK + (nb2 * 16 + b_row(lane)) * LDS + kk * 16 + b_col(lane));
        ldsm_x4(bv, sV + (nb2 * 16 + b_row(lane)) * LDS + kk * 16 + b_col(lane));
        mma16816(sc[2 * nb2], qf[kk], bk[0], bk[1]);
        mma16816(sc[2 * nb2 + 1], qf[kk], bk[2], bk[3]);
        mma16816(dp[2 * nb2], gf[kk], bv[0], bv[1]);
        mma16816(dp[2 * nb2 + 1], gf[kk], bv[2], bv[3]);
      }
    }
#pragma unroll
    for (int nb = 0; nb < BCB / 8; ++nb)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int col = j * BCB + nb * 8 + 2 * t4 + (e & 1);
        const int row = row0 + (e >> 1) * 8;
        float p = exp2f(sc[nb][e] * sl2 - Lr[e >> 1]);
        if (col > row) p = 0.f;
        dp[nb][e] = p * (dp[nb][e] - Dr[e >> 1]);
      }
#pragma unroll
    for (int kk = 0; kk < BCB / 16; ++kk) {
      uint32_t as[4] = {pack_bf16(dp[2 * kk][0], dp[2 * kk][1]), pack_bf16(dp[2 * kk][2], dp[2 * kk][3]),
                        pack_bf16(dp[2 * kk + 1][0], dp[2 * kk + 1][1]), pack_bf16(dp[2 * kk + 1][2], dp[2 * kk + 1][3])};
#pragma unroll
      for (int db = 0; db < D / 16; ++db) {
        uint32_t bk[4];
        ldsm_x4_t(bk, sK + (kk * 16 + a_row(lane)) * LDS + db * 16 + a_col(lane));
        mma16816(dq[2 * db], as, bk[0], bk[1]);
        mma16816(dq[2 * db + 1], as, bk[2], bk[3]);
      }
    }
  }
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int row = row0 + r * 8;
    if (row >= s) continue;
    bf16* qrow = dqkv + (static_cast<long>(b) * s + row) * ld + head * D;
#pragma unroll
    for (int db = 0; db < D / 8; ++db)
      *reinterpret_cast<__nv_bfloat162*>(qrow + db * 8 + 2 * t4) =
          __floats2bfloat162_rn(dq[db][2 * r] * scale, dq[db][2 * r + 1] * scale);
  }
}

template <int D>
void launch_fwd(const bf16* qkv, bf16* O, float* lse, int B, int s, int nh, cudaStream_t st) {
  constexpr size_t smem = 3 * 64 * (D + 8) * sizeof(bf16);
  static bool set = false;
  if (!set) { cudaFuncSetAttribute(fa_fwd_k<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); set = true; }
  dim3 grid((s + BR - 1) / BR, B * nh);
  // causal algorithmic FLOPs: QK^T and PV over the lower triangle
  const double fl = 4.0 * B * nh * D * (static_cast<double>(s) * (s + 1) / 2);
  const int tok = kstats_begin(K_ATTN_FWD, fl, 0.0, st);
  if (g_attn_variant != 0 && flash_attn_fwd_tc(qkv, O, lse, B, s, nh, D, st)) {
    kstats_end(tok, st);
    return;
  }
  fa_fwd_k<D><<<grid, 128, smem, st>>>(qkv, O, lse, B, s, nh);
  kstats_end(tok, st);
  note_launch();
}
template <int D>
void launch_bwd(const bf16* qkv, const bf16* O, const bf16* dO, const float* lse, bf16* dqkv, float* Dd, int B, int s,
                int nh, cudaStream_t st, void* ds_ws, size_t ds_ws_bytes, float* bpart = nullptr,
                bool* bpart_done = nullptr) {
  const long Ttok = static_cast<long>(B) * s;
  if (O) {   // O == nullptr: the caller already wrote D = rowsum(dO o O) into Dd
    const long thr = Ttok * nh * (D / 8);
    const int grid = static_cast<int>((thr + 255) / 256);
    if (D == 128) fa_bwd_dot_v8_k<16><<<grid, 256, 0, st>>>(O, dO, Dd, Ttok, nh);
    else if (D == 64) fa_bwd_dot_v8_k<8><<<grid, 256, 0, st>>>(O, dO, Dd, Ttok, nh);
    else if (D == 32) fa_bwd_dot_v8_k<4><<<grid, 256, 0, st>>>(O, dO, Dd, Ttok, nh);
    else if (D == 16) fa_bwd_dot_v8_k<2><<<grid, 256, 0, st>>>(O, dO, Dd, Ttok, nh);
    else fa_bwd_dot_k<<<static_cast<int>((Ttok * nh * 32 + 255) / 256), 256, 0, st>>>(O, dO, Dd, Ttok, nh, D);
  }
  if (g_attn_variant != 0) {   // tcgen05 backward (attn_tc.cu) when supported
    const double fl = 8.0 * B * nh * D * (static_cast<double>(s) * (s + 1) / 2);
    const int tok = kstats_begin(K_ATTN_BWD, fl, 0.0, st);
    const bool ok = flash_attn_bwd_tc(qkv, dO, lse, Dd, dqkv, B, s, nh, D, ds_ws, ds_ws_bytes, st, 0.f, bpart,
                                      bpart_done);
    kstats_end(tok, st);
    if (ok) { note_launch(); return; }
  }
  constexpr size_t smem_kv = (2 * BR + 2 * BCB) * (D + 8) * sizeof(bf16) + 2 * BCB * sizeof(float);
  constexpr size_t smem_q = (2 * BR + 2 * BCB) * (D + 8) * sizeof(bf16);
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(fa_bwd_dkdv_k<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_kv);
    cudaFuncSetAttribute(fa_bwd_dq_k<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_q);
    set = true;
  }
  dim3 grid((s + BR - 1) / BR, B * nh);
  // algorithmic backward FLOPs (dV, dP, dQ, dK: 4 causal products; the S recompute excluded)
  const double fl = 8.0 * B * nh * D * (static_cast<double>(s) * (s + 1) / 2);
  const int tok = kstats_begin(K_ATTN_BWD, fl, 0.0, st);
  fa_bwd_dkdv_k<D><<<grid, 128, smem_kv, st>>>(qkv, dO, lse, Dd, dqkv, B, s, nh);
  fa_bwd_dq_k<D><<<grid, 128, smem_q, st>>>(qkv, dO, lse, Dd, dqkv, B, s, nh);
  kstats_end(tok, st);
  note_launch(3);
}

}  // namespace

bool flash_attn_supported(int dh) { return dh == 16 || dh == 32 || dh == 64 || dh == 80 || dh == 128; }

// ------------------------------------------------------------------ padded head dims on tcgen05
// Head dims the tcgen05 kernels do not tile (16, 32, 80: GPT-3 2.7B's dh 80 in cfg 4) run on the
// dh_p = 64 / 128 kernels over zero-padded copies: QKV [T][3][nh][dh] -> [T][3][nh][dh_p], the
// kernels told the true softmax scale 1/sqrt(dh); the zero columns add nothing to q.k, and the
// O / dQ / dK / dV padding columns are zero and dropped. Row sums D = rowsum(dO O) come from the
// unpadded tensors. Same values as an unpadded kernel: only zeros are added to each dot product.
namespace {
int padded_dh(int dh) { return dh < 64 ? 64 : 128; }
bool needs_pad(int dh) { return dh != 64 && dh != 128 && dh % 8 == 0 && dh < 128; }

// out[t][p][h][0..Dp) = in[t][p][h][0..dh) (x scale for p == 0), zero-padded; 16-byte chunks
__global__ void attn_pad_k(const bf16* __restrict__ in, bf16* __restrict__ out, long T, int parts, int nh, int dh,
                           int Dp, float scale0) {
  const int cpr = Dp / 8;
  const long total = T * parts * nh * cpr;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < total;
       i += static_cast<long>(gridDim.x) * blockDim.x) {
    const int j = static_cast<int>(i % cpr);
    long r = i / cpr;
    const int hh = static_cast<int>(r % nh);
    r /= nh;
    const int p = static_cast<int>(r % parts);
    const long t = r / parts;
    uint4 v = make_uint4(0, 0, 0, 0);
    if (j * 8 < dh) {
      v = *reinterpret_cast<const uint4*>(in + (t * parts + p) * nh * static_cast<long>(dh) + hh * dh + j * 8);
      if (p == 0 && scale0 != 1.f) {
        __nv_bfloat162* h2 = reinterpret_cast<__nv_bfloat162*>(&v);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float2 f = __bfloat1622float2(h2[e]);
          h2[e] = __floats2bfloat162_rn(f.x * scale0, f.y * scale0);
        }
      }
    }
    *reinterpret_cast<uint4*>(out + (t * parts + p) * nh * static_cast<long>(Dp) + hh * Dp + j * 8) = v;
  }
}
// out[t][p][h][0..dh) = in[t][p][h][0..dh) of the padded layout (x scale for p == 0)
__global__ void attn_unpad_k(const bf16* __restrict__ in, bf16* __restrict__ out, long T, int parts, int nh, int dh,
                             int Dp, float scale0) {
  const int cpr = dh / 8;
  const long total = T * parts * nh * cpr;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < total;
       i += static_cast<long>(gridDim.x) * blockDim.x) {
    const int j = static_cast<int>(i % cpr);
    long r = i / cpr;
    const int hh = static_cast<int>(r % nh);
    r /= nh;
    const int p = static_cast<int>(r % parts);
    const long t = r / parts;
    uint4 v = *reinterpret_cast<const uint4*>(in + (t * parts + p) * nh * static_cast<long>(Dp) + hh * Dp + j * 8);
    if (p == 0 && scale0 != 1.f) {
      __nv_bfloat162* h2 = reinterpret_cast<__nv_bfloat162*>(&v);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 f = __bfloat1622float2(h2[e]);
        h2[e] = __floats2bfloat162_rn(f.x * scale0, f.y * scale0);
      }
    }
    *reinterpret_cast<uint4*>(out + (t * parts + p) * nh * static_cast<long>(dh) + hh * dh + j * 8) = v;
  }
}
void pad(const bf16* in, bf16* out, long T, int parts, int nh, int dh, int Dp, float sc, cudaStream_t st) {
  const long total = T * parts * nh * (Dp / 8);
  const long g = (total + 255) / 256;
  attn_pad_k<<<static_cast<int>(g < 148 * 16 ? g : 148 * 16), 256, 0, st>>>(in, out, T, parts, nh, dh, Dp, sc);
  note_launch();
}
void unpad(const bf16* in, bf16* out, long T, int parts, int nh, int dh, int Dp, float sc, cudaStream_t st) {
  const long total = T * parts * nh * (dh / 8);
  const long g = (total + 255) / 256;
  attn_unpad_k<<<static_cast<int>(g < 148 * 16 ? g : 148 * 16), 256, 0, st>>>(in, out, T, parts, nh, dh, Dp, sc);
  note_launch();
}
}  // namespace

size_t flash_attn_pad_bytes(int dh, int B, int s, int nh, int bwd) {
  if (!needs_pad(dh)) return 0;
  const int Dp = padded_dh(dh);
  if (!flash_attn_bwd_tc_supported(Dp, B, s, nh)) return 0;
  const size_t T = static_cast<size_t>(B) * s, row = static_cast<size_t>(nh) * Dp * 2;
  const size_t al = 256;
  auto up = [&](size_t x) { return (x + al - 1) / al * al; };
  // fwd: qkv' [T, 3 nh Dp], O' [T, nh Dp]; bwd: qkv', dO', dqkv' (+ the dS image for dh_p)
  if (!bwd) return up(T * 3 * row) + up(T * row);
  return up(T * 3 * row) + up(T * row) + up(T * 3 * row) + up(flash_attn_bwd_ds_bytes(Dp, B, s, nh));
}

void flash_attn_fwd(const bf16* qkv, bf16* O, float* lse, int B, int s, int nh, int dh, cudaStream_t st,
                    void* pad_ws) {
  if (pad_ws && needs_pad(dh) && g_attn_variant != 0 && flash_attn_pad_bytes(dh, B, s, nh, 0)) {
    const int Dp = padded_dh(dh);
    const long T = static_cast<long>(B) * s;
    bf16* qkvp = static_cast<bf16*>(pad_ws);
    bf16* Op = qkvp + ((T * 3 * nh * Dp * 2 + 255) / 256 * 256) / 2;
    const double fl = 4.0 * B * nh * dh * (static_cast<double>(s) * (s + 1) / 2);
    const int tok = kstats_begin(K_ATTN_FWD, fl, 0.0, st);
    pad(qkv, qkvp, T, 3, nh, dh, Dp, 1.f, st);
    const bool ok = flash_attn_fwd_tc(qkvp, Op, lse, B, s, nh, Dp, st, rsqrtf(static_cast<float>(dh)));
    if (ok) unpad(Op, O, T, 1, nh, dh, Dp, 1.f, st);
    kstats_end(tok, st);
    if (ok) return;
  }
  switch (dh) {
    case 16: launch_fwd<16>(qkv, O, lse, B, s, nh, st); break;
    case 32: launch_fwd<32>(qkv, O, lse, B, s, nh, st); break;
    case 64: launch_fwd<64>(qkv, O, lse, B, s, nh, st); break;
    case 80: launch_fwd<80>(qkv, O, lse, B, s, nh, st); break;
    default: launch_fwd<128>(qkv, O, lse, B, s, nh, st); break;
  }
}

void flash_attn_bwd(const bf16* qkv, const bf16* O, const bf16* dO, const float* lse, bf16* dqkv, float* Dd, int B,
                    int s, int nh, int dh, cudaStream_t st, void* ds_ws, size_t ds_ws_bytes, void* pad_ws, float* bpart,
                    bool* bpart_done) {
  (void)ds_ws; (void)ds_ws_bytes;
  if (bpart_done) *bpart_done = false;
  if (pad_ws && needs_pad(dh) && g_attn_variant != 0 && flash_attn_pad_bytes(dh, B, s, nh, 1)) {
    const int Dp = padded_dh(dh);
    const long T = static_cast<long>(B) * s;
    auto up = [](long x) { return (x + 255) / 256 * 256; };
    uint8_t* w = static_cast<uint8_t*>(pad_ws);
    bf16* qkvp = reinterpret_cast<bf16*>(w);
    bf16* dOp = reinterpret_cast<bf16*>(w + up(T * 3 * nh * Dp * 2));
    bf16* dqkvp = reinterpret_cast<bf16*>(w + up(T * 3 * nh * Dp * 2) + up(T * nh * Dp * 2));
    uint8_t* img = w + up(T * 3 * nh * Dp * 2) + up(T * nh * Dp * 2) + up(T * 3 * nh * Dp * 2);
    const size_t img_bytes = flash_attn_bwd_ds_bytes(Dp, B, s, nh);
    {   // D = rowsum(dO * O) of the unpadded head (padding columns are zero)
      const long thr = T * nh * 32;
      fa_bwd_dot_k<<<static_cast<int>((thr + 255) / 256), 256, 0, st>>>(O, dO, Dd, T, nh, dh);
      note_launch();
    }
    const double fl = 8.0 * B * nh * dh * (static_cast<double>(s) * (s + 1) / 2);
    const int tok = kstats_begin(K_ATTN_BWD, fl, 0.0, st);
    pad(qkv, qkvp, T, 3, nh, dh, Dp, 1.f, st);
    pad(dO, dOp, T, 1, nh, dh, Dp, 1.f, st);
    const bool ok = flash_attn_bwd_tc(qkvp, dOp, lse, Dd, dqkvp, B, s, nh, Dp, img_bytes ? img : nullptr, img_bytes,
                                      st, rsqrtf(static_cast<float>(dh)));
    if (ok) unpad(dqkvp, dqkv, T, 3, nh, dh, Dp, 1.f, st);
    kstats_end(tok, st);
    if (ok) { note_launch(); return; }
  }
  switch (dh) {
    case 16: launch_bwd<16>(qkv, O, dO, lse, dqkv, Dd, B, s, nh, st, ds_ws, ds_ws_bytes); break;
    case 32: launch_bwd<32>(qkv, O, dO, lse, dqkv, Dd, B, s, nh, st, ds_ws, ds_ws_bytes); break;
    case 64: launch_bwd<64>(qkv, O, dO, lse, dqkv, Dd, B, s, nh, st, ds_ws, ds_ws_bytes, bpart, bpart_done); break;
    case 80: launch_bwd<80>(qkv, O, dO, lse, dqkv, Dd, B, s, nh, st, ds_ws, ds_ws_bytes); break;
    default: launch_bwd<128>(qkv, O, dO, lse, dqkv, Dd, B, s, nh, st, ds_ws, ds_ws_bytes, bpart, bpart_done); break;
  }
}

}  // namespace mario
