// K6 on tcgen05: causal flash-attention backward for bf16, head_dim 64 / 128.
// Same math as attn_mma.cu / SURVEY §8(c) c1:  P = exp(S - lse), dS = P (dP - D),
//   dV = P^T dO,  dK = dS^T Q / sqrt(dh),  dQ = dS K / sqrt(dh),   D = rowsum(dO * O).
//
// dK/dV kernel: one CTA per 128 keys (= 128 TMEM lanes) of one (sample, head); loop over
// 64-query tiles q >= first key:
//   warp 0      TMA: K, V once; Q_i / dO_i into a 2-stage ring (128B swizzle)
//   warp 1      single-thread tcgen05.mma:  S^T = K Q_i^T, dP^T = V dO_i^T  (M128 N64, into a
//               double-buffered TMEM pair), then dV += P^T dO_i, dK += dS^T Q_i (M128 N=dh,
//               accumulated in TMEM across the whole loop). The Q_i / dO_i tiles are read as
//               K-major B for the first products and as MN-major B for the second.
//   warps 2..5  one key row per thread: tcgen05.ld S^T, dP^T rows -> P^T, dS^T (bf16) into
//               swizzled smem for the next MMAs; epilogue tcgen05.ld dK, dV -> global.
// dQ kernel: the mirror image (128 queries per CTA, loop over 64-key tiles, dQ += dS K).
// No atomics: deterministic.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "kernels.h"
#include "kstats.h"
#include "layers.h"
#include "sm100.cuh"

namespace mario {

extern int g_attn_variant;   // attn_mma.cu
bool make_tmap_bf16_2d(CUtensorMap* map, const void* base, uint64_t inner, uint64_t outer, uint64_t ld,
                       uint32_t box_inner, uint32_t box_outer);   // gemm_tc.cu

size_t flash_attn_bwd_ds_bytes(int dh, int B, int s, int nh);   // below

namespace {
using namespace sm100;
using bf16 = __nv_bfloat16;
constexpr float LOG2E = 1.4426950408889634f;
constexpr int kRows = 128;   // rows per CTA (TMEM lanes)
constexpr int kCols = 64;    // inner tile
constexpr int kThreads = 192;

// 2^x on the SFU: one MUFU.EX2 (flush-to-zero; P underflowing to 0 instead of a subnormal is
// harmless) instead of exp2f's range fix-up (FSETP/FSEL/FMUL around the MUFU)
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// 2^x on the FMA pipe (for a share of the softmax exponentials, so the SFU -- 16 ex2 per clock per SM,
// exactly the tensor core's pace at this tile shape -- is not the bottleneck): round x to an integer
// j with the 1.5 * 2^23 magic add, 2^(x - j) by the degree-3 Taylor polynomial on [-1/2, 1/2]
// (relative error <= 8e-4 measured over [-126, 8], below the bf16 rounding P gets), and j added into the exponent field.
// x <= 8 here (lazy max), clamped below at -127 so masked -inf scores give 0.
__device__ __forceinline__ float ex2_poly(float x) {
  x = fmaxf(x, -127.f);
  const float t = x + 12582912.f;
  const float j = t - 12582912.f;
  const float f = x - j;
  float p = fmaf(f, 0.0555041087f, 0.240226507f);
  p = fmaf(f, p, 0.693147181f);
  p = fmaf(f, p, 1.f);
  return __int_as_float(__float_as_int(p) + (__float_as_int(t) << 23));
}
__device__ __forceinline__ void st_shared_f32(const void* p, float v) {
  asm volatile("st.shared.f32 [%0], %1;" :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(p))), "f"(v) : "memory");
}
__device__ __forceinline__ float4 ld_shared_f4(const void* p) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"(static_cast<uint32_t>(__cvta_generic_to_shared(p))) : "memory");
  return v;
}
__device__ __forceinline__ float ld_shared_f32(const void* p) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(static_cast<uint32_t>(__cvta_generic_to_shared(p))) : "memory");
  return v;
}

// L2 eviction priorities (MARIO_ATTN_L2HINT, default off): the tiles many CTAs re-read (K/V in the
// forward and the dQ pass, Q/dO/lse/D in the dK/dV pass) evict_last, each CTA's own stationary
// tiles and the once-read dS image evict_first.
__device__ __forceinline__ uint64_t pol_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_normal() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
int attn_l2hint() {
  // default off: A/B on whole steps was neutral (attention backward -5 ms, the following GEMMs +20-40 ms:
  // evict_last attention tiles outlive the kernel in L2)
  static const int v = getenv("MARIO_ATTN_L2HINT") ? atoi(getenv("MARIO_ATTN_L2HINT")) : 0;
  return v;
}
__device__ __forceinline__ void tma_load_2d_h(void* dst, const void* tmap, uint64_t* bar, int c0, int c1, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%3, %4}], [%2], %5;"
      :: "r"(smem_u32(dst)), "l"(reinterpret_cast<uint64_t>(tmap)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s_h(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void tma_store_2d(const void* tmap, const void* src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];"
               :: "l"(reinterpret_cast<uint64_t>(tmap)), "r"(smem_u32(src)), "r"(c0), "r"(c1) : "memory");
}
__device__ __forceinline__ void bulk_commit_wait_read() {
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
// one 32-byte global store (sm_100: STG.256)
__device__ __forceinline__ void st_global_v8(void* p, const uint32_t (&v)[8]) {
  asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" :: "l"(p), "r"(v[0]), "r"(v[1]), "r"(v[2]),
               "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" :: "r"(id), "r"(n) : "memory"); }

// write 64 bf16 values (one 128-byte row) of a K-major SW128 tile with 128-byte rows
__device__ __forceinline__ void st_row_sw128(uint8_t* tile, int row, const float (&v)[64]) {
  uint8_t* rp = tile + row * 128;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    uint4 u;
    __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
    for (int e = 0; e < 4; ++e) h[e] = __floats2bfloat162_rn(v[8 * j + 2 * e], v[8 * j + 2 * e + 1]);
    *reinterpret_cast<uint4*>(rp + ((j ^ (row & 7)) << 4)) = u;
  }
}

// write 32 bf16 values = chunks [c0, c0+4) of one 128-byte row of a K-major SW128 tile
__device__ __forceinline__ void st_half_row_sw128(uint8_t* tile, int row, int c0, const float (&v)[32]) {
  uint8_t* rp = tile + row * 128;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint4 u;
    __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
    for (int e = 0; e < 4; ++e) h[e] = __floats2bfloat162_rn(v[8 * j + 2 * e], v[8 * j + 2 * e + 1]);
    *reinterpret_cast<uint4*>(rp + (((c0 + j) ^ (row & 7)) << 4)) = u;
  }
}

constexpr int kThreadsB = 320;
constexpr int kRing = 4;     // depth of the streamed-operand TMA ring (K/V or Q/dO tiles)
constexpr int kRingKV = 3;   // dK/dV kernel: 3 Q/dO stages leave room for double-buffered P^T / dS^T

template <int DH>
struct Smem {
  static constexpr int kBig = kRows * DH * 2;        // 128-row tile (K,V or Q,dO)
  static constexpr int kSmall = kCols * DH * 2;      // 64-row tile
  static constexpr int kP = kRows * kCols * 2;       // 128 x 64 bf16
};

// ------------------------------------------------------------------------ dK / dV
template <int DH>
__global__ void __launch_bounds__(kThreadsB, 1)
fa_bwd_dkdv_tc(const __grid_constant__ CUtensorMap tm_qkv128, const __grid_constant__ CUtensorMap tm_qkv64,
               const __grid_constant__ CUtensorMap tm_do64, const __grid_constant__ CUtensorMap tm_dqkv,
               const float* lse, const float* Dd, bf16* dqkv, int B, int s, int nh, int dbg, long long* trace,
               float qk_scale) {
  const bool bulk_ld = (s % kCols) == 0;
  using SM = Smem<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sK = smem;
  uint8_t* sV = sK + SM::kBig;
  // ring slot / buffer addresses as arithmetic (a runtime-indexed pointer array would live in local memory)
  auto sQ = [&](int r) { return sV + SM::kBig + 2 * r * SM::kSmall; };
  auto sG = [&](int r) { return sV + SM::kBig + 2 * r * SM::kSmall + SM::kSmall; };
  // P^T and dS^T double-buffered: tile idx + 1 is written while the dV/dK MMAs read tile idx
  auto sP = [&](int i) { return sV + SM::kBig + 2 * kRingKV * SM::kSmall + 2 * i * SM::kP; };
  auto sS = [&](int i) { return sV + SM::kBig + 2 * kRingKV * SM::kSmall + 2 * i * SM::kP + SM::kP; };
  // per ring slot: lse (natural log) and D of the slot's 64 queries, [kRingKV][2][64] fp32; TMA
  // bulk-copied with the Q/dO tile when s % 64 == 0, else staged by the softmax warps
  float* sLD = reinterpret_cast<float*>(sS(1) + SM::kP);
  uint64_t* bar = reinterpret_cast<uint64_t*>(sLD + kRingKV * 2 * kCols);
  uint64_t* kv_full = bar;                 // 1
  uint64_t* q_full = bar + 1;              // kRingKV
  uint64_t* q_empty = q_full + kRingKV;    // kRingKV
  uint64_t* s_full = q_empty + kRingKV;    // 2
  uint64_t* s_free = s_full + 2;           // 2
  uint64_t* p_full = s_free + 2;           // 2
  uint64_t* p_free = p_full + 2;           // 2
  uint64_t* acc_done = p_free + 2;         // 1
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_done + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  // heaviest first over all (sample, head) (key tile 0 sees every query tile); dbg bit 3: (sample, head)-major
  const int nt = (s + kRows - 1) / kRows, BH = B * nh;
  const int j = (dbg & 8) ? blockIdx.x % nt : blockIdx.x / BH, bh = (dbg & 8) ? blockIdx.x / nt : blockIdx.x % BH;
  const int kt = j, b = bh / nh, head = bh % nh;
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const int i0 = (kt * kRows) / kCols;
  const int nq = (s + kCols - 1) / kCols;
  const int ntiles = (dbg & 32) ? min(nq - i0, 1) : nq - i0;
  const float sl2 = qk_scale * LOG2E;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    tma_prefetch_desc(&tm_qkv64);
    tma_prefetch_desc(&tm_do64);
    mbar_init(kv_full, 1);
    for (int i = 0; i < kRingKV; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1); mbar_init(&s_free[i], 8); mbar_init(&p_full[i], 8); mbar_init(&p_free[i], 1);
    }
    mbar_init(acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_dV = tm, tm_dK = tm + DH, tm_S = tm + 2 * DH, tm_dP = tm + 2 * DH + 2 * kCols;

  if (ntiles <= 0) {  // keys entirely beyond the sample: nothing to do (dK = dV = 0 not needed: rows >= s)
    __syncthreads();
    if (warp == 1) tmem_dealloc<512>(tm);
    return;
  }

  if (warp == 0) {
    if (elect_one()) {
      const int row0 = b * s;
      if (dbg & 128) mbar_arrive(kv_full);
      else mbar_arrive_expect_tx(kv_full, 2 * SM::kBig);
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) {
        if (dbg & 128) break;
        tma_load_2d(sK + a * (kRows * 128), &tm_qkv128, kv_full, h + head * DH + a * 64, row0 + kt * kRows);
        tma_load_2d(sV + a * (kRows * 128), &tm_qkv128, kv_full, 2 * h + head * DH + a * 64, row0 + kt * kRows);
      }
      for (int idx = 0; idx < ntiles; ++idx) {
        const int st = idx % kRingKV;
        mbar_wait(&q_empty[st], ((idx / kRingKV) & 1) ^ 1);
        if (dbg & 16) { mbar_arrive(&q_full[st]); continue; }
        mbar_arrive_expect_tx(&q_full[st], 2 * SM::kSmall + (bulk_ld ? 2 * kCols * 4 : 0));
        const int qr = row0 + (i0 + idx) * kCols;
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_2d(sQ(st) + a * (kCols * 128), &tm_qkv64, &q_full[st], head * DH + a * 64, qr);
          tma_load_2d(sG(st) + a * (kCols * 128), &tm_do64, &q_full[st], head * DH + a * 64, qr);
        }
        if (bulk_ld) {
          const long o = static_cast<long>(head) * Ttok + qr;
          bulk_g2s(sLD + st * 2 * kCols, lse + o, kCols * 4, &q_full[st]);
          bulk_g2s(sLD + st * 2 * kCols + kCols, Dd + o, kCols * 4, &q_full[st]);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(128, kCols, 0, 0);   // S^T, dP^T: K-major A and B
    constexpr uint32_t id_a = umma_idesc_bf16(128, DH, 0, 1);      // dV, dK: B = Q/dO read MN-major
    mbar_wait(kv_full, 0);
    tc_fence_after();
    const bool tr = trace && blockIdx.x == 0 && lane == 0;
    auto issue_s = [&](int idx) {
      const int st = idx % kRingKV, buf = idx & 1;
      if (tr) trace[0 * 64 + idx] = clock64();
      mbar_wait(&q_full[st], (idx / kRingKV) & 1);
      mbar_wait(&s_free[buf], ((idx >> 1) & 1) ^ 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t k = smem_u32(sK), v = smem_u32(sV), q = smem_u32(sQ(st)), g = smem_u32(sG(st));
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          if (dbg & 2) break;
          const uint32_t ao = (kk >> 2) * (kRows * 128) + (kk & 3) * 32, bo = (kk >> 2) * (kCols * 128) + (kk & 3) * 32;
          umma_bf16(tm_S + buf * kCols, umma_desc_sw128(k + ao, 16, 1024), umma_desc_sw128(q + bo, 16, 1024), id_s, kk > 0);
          umma_bf16(tm_dP + buf * kCols, umma_desc_sw128(v + ao, 16, 1024), umma_desc_sw128(g + bo, 16, 1024), id_s, kk > 0);
        }
        umma_commit(&s_full[buf]);
      }
      __syncwarp();
      if (tr) trace[1 * 64 + idx] = clock64();
    };
    auto issue_acc = [&](int idx) {
      const int st = idx % kRingKV, pb = idx & 1;
      if (tr) trace[2 * 64 + idx] = clock64();
      mbar_wait(&p_full[pb], (idx >> 1) & 1);
      if (tr) trace[3 * 64 + idx] = clock64();
      tc_fence_after();
      if (elect_one()) {
        const uint32_t p = smem_u32(sP(pb)), ds = smem_u32(sS(pb)), q = smem_u32(sQ(st)), g = smem_u32(sG(st));
#pragma unroll
        for (int kk = 0; kk < kCols / 16; ++kk) {
          if (dbg & 4) break;
          const uint64_t pa = umma_desc_sw128(p + kk * 32, 16, 1024), sa = umma_desc_sw128(ds + kk * 32, 16, 1024);
          umma_bf16(tm_dV, pa, umma_desc_sw128(g + kk * 2048, kCols * 128, 1024), id_a, (idx | kk) != 0);
          umma_bf16(tm_dK, sa, umma_desc_sw128(q + kk * 2048, kCols * 128, 1024), id_a, (idx | kk) != 0);
        }
        umma_commit(&p_free[pb]);
        umma_commit(&q_empty[st]);
        if (idx == ntiles - 1) umma_commit(acc_done);
      }
      __syncwarp();
    };
    issue_s(0);
    for (int idx = 1; idx < ntiles; ++idx) {
      issue_s(idx);
      issue_acc(idx - 1);
    }
    issue_acc(ntiles - 1);
  } else {
    const int quarter = warp & 3, half = (warp - 2) >> 2;   // column half [32*half, 32*half+32)
    const int row = quarter * 32 + lane;             // key row within the tile
    const int key = kt * kRows + row;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const int tid = threadIdx.x - 64;                // 0..255
    for (int idx = 0; idx < ntiles; ++idx) {
      const int buf = idx & 1, i = i0 + idx, st = idx % kRingKV;
      float* ld = sLD + st * 2 * kCols;
      if (bulk_ld) {
        // the slot's lse / D came with its Q/dO tile (the slot is released only after this tile's
        // accumulate MMAs, which wait for this loop's p_full: no later phase can be pending)
        mbar_wait(&q_full[st], (idx / kRingKV) & 1);
      } else {
        // lse / D of this query tile into the slot (threads 0..63: lse, 64..127: D)
        if (tid < 128) {
          const int c = tid & 63, qq = i * kCols + c;
          const long r = static_cast<long>(b) * s + (qq < s ? qq : 0);
          ld[tid] = tid < 64 ? lse[static_cast<long>(head) * Ttok + r] : Dd[static_cast<long>(head) * Ttok + r];
        }
        named_bar(1, 256);
      }
      float lv[32], dv[32];
#pragma unroll
      for (int c = 0; c < 32; c += 4) {
        const float4 a = ld_shared_f4(ld + half * 32 + c);
        const float4 d = ld_shared_f4(ld + kCols + half * 32 + c);
        lv[c] = a.x * LOG2E; lv[c + 1] = a.y * LOG2E; lv[c + 2] = a.z * LOG2E; lv[c + 3] = a.w * LOG2E;
        dv[c] = d.x; dv[c + 1] = d.y; dv[c + 2] = d.z; dv[c + 3] = d.w;
      }
      const bool trs = trace && blockIdx.x == 0 && threadIdx.x == 64;
      if (trs) trace[4 * 64 + idx] = clock64();
      mbar_wait(&s_full[buf], (idx >> 1) & 1);
      if (trs) trace[5 * 64 + idx] = clock64();
      tc_fence_after();
      uint32_t sr[32], dr[32];
      tmem_ld_32x32b_x32(tm_S + buf * kCols + half * 32 + lane_off, sr);
      tmem_ld_32x32b_x32(tm_dP + buf * kCols + half * 32 + lane_off, dr);
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&s_free[buf]);
      float p[32], ds[32];
      if (dbg & 1) {
        mbar_wait(&p_free[buf], ((idx >> 1) & 1) ^ 1);
        __syncwarp();
        if (lane == 0) mbar_arrive(&p_full[buf]);
        continue;
      }
      // only tiles crossing the diagonal (queries < this block's last key) or the sequence end mask
      const bool edge = i * kCols < kt * kRows + kRows || i * kCols + kCols > s;
      if (edge) {
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const int cc = half * 32 + c;
          const int qq = i * kCols + cc;
          float pv = ex2(__uint_as_float(sr[c]) * sl2 - lv[c]);
          if (qq < key || qq >= s) pv = 0.f;
          p[c] = pv;
          ds[c] = pv * (__uint_as_float(dr[c]) - dv[c]);
        }
      } else {
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const float pv = ex2(__uint_as_float(sr[c]) * sl2 - lv[c]);
          p[c] = pv;
          ds[c] = pv * (__uint_as_float(dr[c]) - dv[c]);
        }
      }
      if (trs) trace[6 * 64 + idx] = clock64();
      mbar_wait(&p_free[buf], ((idx >> 1) & 1) ^ 1);   // the dV/dK MMAs of tile idx-2 consumed this buffer
      st_half_row_sw128(sP(buf), row, 4 * half, p);
      st_half_row_sw128(sS(buf), row, 4 * half, ds);
      fence_proxy_async();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[buf]);
      if (trs) trace[7 * 64 + idx] = clock64();
    }
    if (half == 1) goto done_dkdv;   // the epilogue uses one warp per lane quarter
    // epilogue: dV, dK rows of this thread's key
    mbar_wait(acc_done, 0);
    tc_fence_after();
    // tcgen05.ld is warp-collective (.sync.aligned): every lane loads, only valid keys store.
    // Full 128-key blocks (s % 128 == 0): rows go to the (now idle) P/dS buffers in the SW128 layout
    // and leave as four TMA tensor stores (coalesced); otherwise row-wise stores.
    const float scale = qk_scale;
    const bool tma_st = (s % kRows) == 0 && !(dbg & 64);
    auto stV = [&](int a) { return a ? sS(0) : sP(0); };
    auto stK = [&](int a) { return a ? sS(1) : sP(1); };
    const long krow_idx = static_cast<long>(b) * s + (key < s ? key : 0);
    bf16* krow = dqkv + krow_idx * (3 * h) + h + head * DH;
    bf16* vrow = krow + h;
#pragma unroll 1
    for (int c = 0; c < DH; c += 32) {
      uint32_t rv[32], rk[32];
      tmem_ld_32x32b_x32(tm_dV + c + lane_off, rv);
      tmem_ld_32x32b_x32(tm_dK + c + lane_off, rk);
      tmem_ld_wait();
      if (tma_st) {
        float fv[32], fk[32];
#pragma unroll
        for (int e = 0; e < 32; ++e) { fv[e] = __uint_as_float(rv[e]); fk[e] = __uint_as_float(rk[e]) * scale; }
        st_half_row_sw128(stV(c / 64), row, (c % 64) / 8, fv);
        st_half_row_sw128(stK(c / 64), row, (c % 64) / 8, fk);
      } else if (key < s && !(dbg & 64)) {
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          uint4 uv, uk;
          __nv_bfloat162* hv = reinterpret_cast<__nv_bfloat162*>(&uv);
          __nv_bfloat162* hk = reinterpret_cast<__nv_bfloat162*>(&uk);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            hv[e] = __floats2bfloat162_rn(__uint_as_float(rv[8 * q + 2 * e]), __uint_as_float(rv[8 * q + 2 * e + 1]));
            hk[e] = __floats2bfloat162_rn(__uint_as_float(rk[8 * q + 2 * e]) * scale,
                                          __uint_as_float(rk[8 * q + 2 * e + 1]) * scale);
          }
          *reinterpret_cast<uint4*>(vrow + c + 8 * q) = uv;
          *reinterpret_cast<uint4*>(krow + c + 8 * q) = uk;
        }
      }
    }
    if (tma_st) {
      fence_proxy_async();
      named_bar(2, 128);
      if (threadIdx.x == 64) {
        const int r0 = b * s + kt * kRows;
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_store_2d(&tm_dqkv, stV(a), 2 * h + head * DH + a * 64, r0);
          tma_store_2d(&tm_dqkv, stK(a), h + head * DH + a * 64, r0);
        }
        bulk_commit_wait_read();
      }
    }
  }
done_dkdv:
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
}

// ------------------------------------------------------------------------------ dQ
template <int DH>
__global__ void __launch_bounds__(kThreadsB, 1)
fa_bwd_dq_tc(const __grid_constant__ CUtensorMap tm_qkv128, const __grid_constant__ CUtensorMap tm_qkv64,
             const __grid_constant__ CUtensorMap tm_do128, const __grid_constant__ CUtensorMap tm_dqkv,
             const float* lse, const float* Dd, bf16* dqkv, int B, int s, int nh, int dbg, float qk_scale) {
  using SM = Smem<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sG = sQ + SM::kBig;
  auto sK = [&](int r) { return sG + SM::kBig + 2 * r * SM::kSmall; };
  auto sV = [&](int r) { return sG + SM::kBig + 2 * r * SM::kSmall + SM::kSmall; };
  // dS [128 q][64 keys], double-buffered
  auto sS = [&](int i) { return sG + SM::kBig + 2 * kRing * SM::kSmall + i * SM::kP; };
  uint64_t* bar = reinterpret_cast<uint64_t*>(sS(1) + SM::kP);
  uint64_t* q_fullb = bar;                // Q, dO loaded
  uint64_t* k_full = bar + 1;             // kRing
  uint64_t* k_empty = k_full + kRing;     // kRing
  uint64_t* s_full = k_empty + kRing;     // 2
  uint64_t* s_free = s_full + 2;          // 2
  uint64_t* p_full = s_free + 2;          // 2
  uint64_t* p_free = p_full + 2;          // 2
  uint64_t* acc_done = p_free + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_done + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  // heaviest first over all (sample, head) (the last query tile sees every key tile); dbg bit 3: (sample, head)-major
  const int nt = (s + kRows - 1) / kRows, BH = B * nh;
  const int j = (dbg & 8) ? blockIdx.x % nt : blockIdx.x / BH, bh = (dbg & 8) ? blockIdx.x / nt : blockIdx.x % BH;
  const int qt = nt - 1 - j, b = bh / nh, head = bh % nh;
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const int last_q = min(qt * kRows + kRows - 1, s - 1);
  const int ntiles = (dbg & 32) ? 1 : last_q / kCols + 1;   // key tiles 0 .. last_q/64
  const float sl2 = qk_scale * LOG2E;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    tma_prefetch_desc(&tm_qkv64);
    tma_prefetch_desc(&tm_do128);
    mbar_init(q_fullb, 1);
    for (int i = 0; i < kRing; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&s_full[i], 1); mbar_init(&s_free[i], 8); }
    for (int i = 0; i < 2; ++i) { mbar_init(&p_full[i], 8); mbar_init(&p_free[i], 1); }
    mbar_init(acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_dQ = tm, tm_S = tm + DH, tm_dP = tm + DH + 2 * kCols;

  if (warp == 0) {
    if (elect_one()) {
      const int row0 = b * s;
      if (dbg & 128) mbar_arrive(q_fullb);
      else mbar_arrive_expect_tx(q_fullb, 2 * SM::kBig);
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) {
        if (dbg & 128) break;
        tma_load_2d(sQ + a * (kRows * 128), &tm_qkv128, q_fullb, head * DH + a * 64, row0 + qt * kRows);
        tma_load_2d(sG + a * (kRows * 128), &tm_do128, q_fullb, head * DH + a * 64, row0 + qt * kRows);
      }
      for (int idx = 0; idx < ntiles; ++idx) {
        const int st = idx % kRing;
        mbar_wait(&k_empty[st], ((idx / kRing) & 1) ^ 1);
        if (dbg & 16) { mbar_arrive(&k_full[st]); continue; }
        mbar_arrive_expect_tx(&k_full[st], 2 * SM::kSmall);
        const int kr = row0 + idx * kCols;
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_2d(sK(st) + a * (kCols * 128), &tm_qkv64, &k_full[st], h + head * DH + a * 64, kr);
          tma_load_2d(sV(st) + a * (kCols * 128), &tm_qkv64, &k_full[st], 2 * h + head * DH + a * 64, kr);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(128, kCols, 0, 0);
    constexpr uint32_t id_a = umma_idesc_bf16(128, DH, 0, 1);   // dQ += dS K: B = K_j read MN-major
    mbar_wait(q_fullb, 0);
    tc_fence_after();
    auto issue_s = [&](int idx) {
      const int st = idx % kRing, buf = idx & 1;
      mbar_wait(&k_full[st], (idx / kRing) & 1);
      mbar_wait(&s_free[buf], ((idx >> 1) & 1) ^ 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t q = smem_u32(sQ), g = smem_u32(sG), k = smem_u32(sK(st)), v = smem_u32(sV(st));
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          if (dbg & 2) break;
          const uint32_t ao = (kk >> 2) * (kRows * 128) + (kk & 3) * 32, bo = (kk >> 2) * (kCols * 128) + (kk & 3) * 32;
          umma_bf16(tm_S + buf * kCols, umma_desc_sw128(q + ao, 16, 1024), umma_desc_sw128(k + bo, 16, 1024), id_s, kk > 0);
          umma_bf16(tm_dP + buf * kCols, umma_desc_sw128(g + ao, 16, 1024), umma_desc_sw128(v + bo, 16, 1024), id_s, kk > 0);
        }
        umma_commit(&s_full[buf]);
      }
      __syncwarp();
    };
    auto issue_acc = [&](int idx) {
      const int st = idx % kRing, pb = idx & 1;
      mbar_wait(&p_full[pb], (idx >> 1) & 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t ds = smem_u32(sS(pb)), k = smem_u32(sK(st));
#pragma unroll
        for (int kk = 0; kk < kCols / 16; ++kk)
          if (!(dbg & 4))
            umma_bf16(tm_dQ, umma_desc_sw128(ds + kk * 32, 16, 1024), umma_desc_sw128(k + kk * 2048, kCols * 128, 1024),
                      id_a, (idx | kk) != 0);
        umma_commit(&p_free[pb]);
        umma_commit(&k_empty[st]);
        if (idx == ntiles - 1) umma_commit(acc_done);
      }
      __syncwarp();
    };
    issue_s(0);
    for (int idx = 1; idx < ntiles; ++idx) {
      issue_s(idx);
      issue_acc(idx - 1);
    }
    issue_acc(ntiles - 1);
  } else {
    const int quarter = warp & 3, half = (warp - 2) >> 2;
    const int row = quarter * 32 + lane;
    const int q = qt * kRows + row;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const long gr = static_cast<long>(b) * s + (q < s ? q : 0);
    const float L = lse[static_cast<long>(head) * Ttok + gr] * LOG2E;
    const float Dr = Dd[static_cast<long>(head) * Ttok + gr];
    for (int idx = 0; idx < ntiles; ++idx) {
      const int buf = idx & 1;
      mbar_wait(&s_full[buf], (idx >> 1) & 1);
      tc_fence_after();
      uint32_t sr[32], dr[32];
      tmem_ld_32x32b_x32(tm_S + buf * kCols + half * 32 + lane_off, sr);
      tmem_ld_32x32b_x32(tm_dP + buf * kCols + half * 32 + lane_off, dr);
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&s_free[buf]);
      float ds[32];
      if (dbg & 1) {
        mbar_wait(&p_free[buf], ((idx >> 1) & 1) ^ 1);
        __syncwarp();
        if (lane == 0) mbar_arrive(&p_full[buf]);
        continue;
      }
      if (idx * kCols + kCols - 1 > qt * kRows) {   // tile crosses the diagonal: causal mask
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const int key = idx * kCols + half * 32 + c;
          float pv = ex2(__uint_as_float(sr[c]) * sl2 - L);
          if (key > q) pv = 0.f;
          ds[c] = pv * (__uint_as_float(dr[c]) - Dr);
        }
      } else {
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const float pv = ex2(__uint_as_float(sr[c]) * sl2 - L);
          ds[c] = pv * (__uint_as_float(dr[c]) - Dr);
        }
      }
      mbar_wait(&p_free[buf], ((idx >> 1) & 1) ^ 1);
      st_half_row_sw128(sS(buf), row, 4 * half, ds);
      fence_proxy_async();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[buf]);
    }
    if (half == 1) goto done_dq;
    mbar_wait(acc_done, 0);
    tc_fence_after();
    const float scale = qk_scale;
    const bool tma_st = (s % kRows) == 0 && !(dbg & 64);
    bf16* qrow = dqkv + gr * (3 * h) + head * DH;
#pragma unroll 1
    for (int c = 0; c < DH; c += 32) {
      uint32_t rq[32];
      tmem_ld_32x32b_x32(tm_dQ + c + lane_off, rq);
      tmem_ld_wait();
      if (tma_st) {   // rows into the idle dS buffers (SW128), then TMA tensor stores
        float fq[32];
#pragma unroll
        for (int e = 0; e < 32; ++e) fq[e] = __uint_as_float(rq[e]) * scale;
        st_half_row_sw128(sS(c / 64), row, (c % 64) / 8, fq);
      } else if (q < s && !(dbg & 64)) {
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          uint4 u;
          __nv_bfloat162* hq = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
          for (int f = 0; f < 4; ++f)
            hq[f] = __floats2bfloat162_rn(__uint_as_float(rq[8 * e + 2 * f]) * scale, __uint_as_float(rq[8 * e + 2 * f + 1]) * scale);
          *reinterpret_cast<uint4*>(qrow + c + 8 * e) = u;
        }
      }
    }
    if (tma_st) {
      fence_proxy_async();
      named_bar(2, 128);
      if (threadIdx.x == 64) {
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) tma_store_2d(&tm_dqkv, sS(a), head * DH + a * 64, b * s + qt * kRows);
        bulk_commit_wait_read();
      }
    }
  }
done_dq:
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
}

// ------------------------------------------------------------------- dK / dV, "TS"
// fa_bwd_dkdv_ts: the dK/dV kernel with P^T and dS^T kept in TMEM. The softmax threads (one key row
// = one TMEM lane each) pack P^T / dS^T to bf16 and tcgen05.st them over the S^T / dP^T columns they
// have just read (half h of the warps owns S columns [32h, 32h + 32) and writes its 16 packed columns
// at [32h, 32h + 16): no cross-warp hazard), and dV += P^T dO, dK += dS^T Q read their A operand
// from TMEM. This removes the P^T / dS^T shared-memory round trip (32 KB written + 32 KB read by the
// tensor core per tile) and frees 64 KB of shared memory for a 4-deep Q/dO ring: a ring slot is held
// from the S^T MMAs of its tile to the completion of its dV/dK MMAs, so the ring depth bounds how
// far the TMA runs ahead (the 3-deep ring of fa_bwd_dkdv_tc kept ~2000 cycles per tile at the
// cfg-2 shape, per the tools/attn_trace.py timeline). An S^T / dP^T buffer is released by the
// commit of the dV/dK MMAs that read the P^T / dS^T written into it.
constexpr int kRingTS = 4;
template <int DH>
__global__ void __launch_bounds__(kThreadsB, 1)
fa_bwd_dkdv_ts(const __grid_constant__ CUtensorMap tm_qkv128, const __grid_constant__ CUtensorMap tm_qkv64,
               const __grid_constant__ CUtensorMap tm_do64,
               const __grid_constant__ CUtensorMap tm_dqkv, const float* lse, const float* Dd, bf16* dqkv, int B,
               int s, int nh, uint8_t* dsimg, int l2hint, float qk_scale, long long* trace, int inorder) {
  const bool bulk_ld = (s % kCols) == 0;
  if (trace && threadIdx.x == 0 && blockIdx.x < 8192) {   // per-CTA (SM, start ns) for the trace tool
    uint64_t gt; uint32_t sm;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    trace[512 + 3 * blockIdx.x] = sm;
    trace[512 + 3 * blockIdx.x + 1] = static_cast<long long>(gt);
  }
  using SM = Smem<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sK = smem;
  uint8_t* sV = sK + SM::kBig;
  auto sQ = [&](int r) { return sV + SM::kBig + 2 * r * SM::kSmall; };
  auto sG = [&](int r) { return sV + SM::kBig + 2 * r * SM::kSmall + SM::kSmall; };
  float* sLD = reinterpret_cast<float*>(sV + SM::kBig + 2 * kRingTS * SM::kSmall);   // [ring][2][64]
  uint64_t* bar = reinterpret_cast<uint64_t*>(sLD + kRingTS * 2 * kCols);
  uint64_t* kv_full = bar;                 // 1
  uint64_t* q_full = bar + 1;              // kRingTS
  uint64_t* q_empty = q_full + kRingTS;    // kRingTS
  uint64_t* s_full = q_empty + kRingTS;    // 2
  uint64_t* s_free = s_full + 2;           // 2  (dV/dK MMA commit)
  uint64_t* p_full = s_free + 2;           // 2  (8 softmax warps)
  uint64_t* acc_done = p_full + 2;         // 1
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_done + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nt = (s + kRows - 1) / kRows, BH = B * nh;
  const int kt = blockIdx.x / BH, bh = blockIdx.x % BH, b = bh / nh, head = bh % nh;   // heaviest first
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const int i0 = (kt * kRows) / kCols;
  const int nq = (s + kCols - 1) / kCols;
  const int ntiles = nq - i0;
  const float sl2 = qk_scale * LOG2E;
  (void)nt;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    tma_prefetch_desc(&tm_qkv64);
    tma_prefetch_desc(&tm_do64);
    mbar_init(kv_full, 1);
    for (int i = 0; i < kRingTS; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&s_full[i], 1); mbar_init(&s_free[i], 1); mbar_init(&p_full[i], 8); }
    mbar_init(acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_dV = tm, tm_dK = tm + DH, tm_S = tm + 2 * DH, tm_dP = tm + 2 * DH + 2 * kCols;

  if (ntiles <= 0) {
    __syncthreads();
    if (warp == 1) tmem_dealloc<512>(tm);
    return;
  }

  if (warp == 0) {
    if (elect_one()) {
      const uint64_t pf_ = l2hint ? pol_first() : pol_normal(), pl_ = l2hint ? pol_last() : pol_normal();
      const int row0 = b * s;
      mbar_arrive_expect_tx(kv_full, 2 * SM::kBig);
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) {
        tma_load_2d_h(sK + a * (kRows * 128), &tm_qkv128, kv_full, h + head * DH + a * 64, row0 + kt * kRows, pf_);
        tma_load_2d_h(sV + a * (kRows * 128), &tm_qkv128, kv_full, 2 * h + head * DH + a * 64, row0 + kt * kRows, pf_);
      }
      for (int idx = 0; idx < ntiles; ++idx) {
        const int st = idx % kRingTS;
        mbar_wait(&q_empty[st], ((idx / kRingTS) & 1) ^ 1);
        mbar_arrive_expect_tx(&q_full[st], 2 * SM::kSmall + (bulk_ld ? 2 * kCols * 4 : 0));
        const int qr = row0 + (i0 + idx) * kCols;
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_2d_h(sQ(st) + a * (kCols * 128), &tm_qkv64, &q_full[st], head * DH + a * 64, qr, pl_);
          tma_load_2d_h(sG(st) + a * (kCols * 128), &tm_do64, &q_full[st], head * DH + a * 64, qr, pl_);
        }
        if (bulk_ld) {
          const long o = static_cast<long>(head) * Ttok + qr;
          bulk_g2s_h(sLD + st * 2 * kCols, lse + o, kCols * 4, &q_full[st], pl_);
          bulk_g2s_h(sLD + st * 2 * kCols + kCols, Dd + o, kCols * 4, &q_full[st], pl_);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(128, kCols, 0, 0);   // S^T, dP^T: K-major A and B
    constexpr uint32_t id_a = umma_idesc_bf16(128, DH, 0, 1);      // dV, dK: A from TMEM, B MN-major
    mbar_wait(kv_full, 0);
    tc_fence_after();
    const bool tr = trace && blockIdx.x == 0 && lane == 0;
    auto issue_s = [&](int idx) {
      const int st = idx % kRingTS, buf = idx & 1;
      if (tr) trace[0 * 64 + idx] = clock64();
      mbar_wait(&q_full[st], (idx / kRingTS) & 1);
      // inorder: S^T / dP^T of tile idx overwrite the P^T / dS^T columns the dV / dK MMAs of tile idx - 2
      // read; those were issued earlier by this thread, and tcgen05.mma executes in issue order, so
      // the tensor pipe needs no drain (commit -> mbarrier -> issue) between them
      if (!inorder) mbar_wait(&s_free[buf], ((idx >> 1) & 1) ^ 1);
      if (tr) trace[1 * 64 + idx] = clock64();
      tc_fence_after();
      if (elect_one()) {
        const uint32_t k = smem_u32(sK), v = smem_u32(sV), q = smem_u32(sQ(st)), g = smem_u32(sG(st));
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const uint32_t ao = (kk >> 2) * (kRows * 128) + (kk & 3) * 32, bo = (kk >> 2) * (kCols * 128) + (kk & 3) * 32;
          umma_bf16(tm_S + buf * kCols, umma_desc_sw128(k + ao, 16, 1024), umma_desc_sw128(q + bo, 16, 1024), id_s, kk > 0);
          umma_bf16(tm_dP + buf * kCols, umma_desc_sw128(v + ao, 16, 1024), umma_desc_sw128(g + bo, 16, 1024), id_s, kk > 0);
        }
        umma_commit(&s_full[buf]);
      }
      __syncwarp();
    };
    auto issue_acc = [&](int idx) {
      const int st = idx % kRingTS, buf = idx & 1;
      if (tr) trace[2 * 64 + idx] = clock64();
      mbar_wait(&p_full[buf], (idx >> 1) & 1);
      if (tr) trace[3 * 64 + idx] = clock64();
      tc_fence_after();
      if (elect_one()) {
        const uint32_t q = smem_u32(sQ(st)), g = smem_u32(sG(st));
#pragma unroll
        for (int kk = 0; kk < kCols / 16; ++kk) {
          // queries [16kk, 16kk + 16): packed columns (kk / 2) * 32 + (kk % 2) * 8 of the buffer
          const uint32_t ac = buf * kCols + (kk >> 1) * 32 + (kk & 1) * 8;
          umma_bf16_ts(tm_dV, tm_S + ac, umma_desc_sw128(g + kk * 2048, kCols * 128, 1024), id_a, (idx | kk) != 0);
          umma_bf16_ts(tm_dK, tm_dP + ac, umma_desc_sw128(q + kk * 2048, kCols * 128, 1024), id_a, (idx | kk) != 0);
        }
        umma_commit(&s_free[buf]);
        umma_commit(&q_empty[st]);
        if (idx == ntiles - 1) umma_commit(acc_done);
      }
      __syncwarp();
    };
    issue_s(0);
    for (int idx = 1; idx < ntiles; ++idx) {
      issue_s(idx);
      issue_acc(idx - 1);
    }
    issue_acc(ntiles - 1);
  } else {
    const int quarter = warp & 3, half = (warp - 2) >> 2;   // S columns [32 half, 32 half + 32)
    const int row = quarter * 32 + lane;                     // key row within the tile
    const int key = kt * kRows + row;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const int tid = threadIdx.x - 64;
    float lv[32], dv[32];
    // lse (pre-scaled by log2 e) and D of the tile's 32 queries of this half, from the ring slot
    auto load_ld = [&](int idx) {
      const int i = i0 + idx, st = idx % kRingTS;
      float* ld = sLD + st * 2 * kCols;
      if (bulk_ld) {
        mbar_wait(&q_full[st], (idx / kRingTS) & 1);
      } else {
        if (tid < 128) {
          const int c = tid & 63, qq = i * kCols + c;
          const long r = static_cast<long>(b) * s + (qq < s ? qq : 0);
          ld[tid] = tid < 64 ? lse[static_cast<long>(head) * Ttok + r] : Dd[static_cast<long>(head) * Ttok + r];
        }
        named_bar(1, 256);
      }
#pragma unroll
      for (int c = 0; c < 32; c += 4) {
        const float4 a = ld_shared_f4(ld + half * 32 + c);
        const float4 d = ld_shared_f4(ld + kCols + half * 32 + c);
        lv[c] = a.x * LOG2E; lv[c + 1] = a.y * LOG2E; lv[c + 2] = a.z * LOG2E; lv[c + 3] = a.w * LOG2E;
        dv[c] = d.x; dv[c + 1] = d.y; dv[c + 2] = d.z; dv[c + 3] = d.w;
      }
    };
    load_ld(0);
    for (int idx = 0; idx < ntiles; ++idx) {
      const int buf = idx & 1, i = i0 + idx;
      const bool trs = trace && blockIdx.x == 0 && threadIdx.x == 64;
      if (trs) trace[4 * 64 + idx] = clock64();
      mbar_wait(&s_full[buf], (idx >> 1) & 1);
      if (trs) trace[5 * 64 + idx] = clock64();
      tc_fence_after();
      uint32_t sr[32], dr[32];
      const uint32_t col = buf * kCols + half * 32 + lane_off;
      tmem_ld_32x32b_x32(tm_S + col, sr);
      tmem_ld_32x32b_x32(tm_dP + col, dr);
      tmem_ld_wait();
      if (trs) trace[6 * 64 + idx] = clock64();
      uint32_t pk[16], dk[16];
      float pv[32];
#pragma unroll
      for (int c = 0; c < 32; ++c) pv[c] = ex2(__uint_as_float(sr[c]) * sl2 - lv[c]);
      // causal / ragged mask only on the diagonal and last tiles, as one branch-free pass (a
      // per-element branch inside the loop above cost 16 branch regions on every tile)
      if (i * kCols < kt * kRows + kRows || i * kCols + kCols > s) {
        const int lo = key - (i * kCols + half * 32), hi = s - (i * kCols + half * 32);
#pragma unroll
        for (int c = 0; c < 32; ++c) pv[c] = (c < lo || c >= hi) ? 0.f : pv[c];
      }
#pragma unroll
      for (int c = 0; c < 32; c += 2) {
        const float p0 = pv[c], p1 = pv[c + 1];
        const float d0 = p0 * (__uint_as_float(dr[c]) - dv[c]), d1 = p1 * (__uint_as_float(dr[c + 1]) - dv[c + 1]);
        const __nv_bfloat162 pp = __floats2bfloat162_rn(p0, p1), dd = __floats2bfloat162_rn(d0, d1);
        pk[c / 2] = *reinterpret_cast<const uint32_t*>(&pp);
        dk[c / 2] = *reinterpret_cast<const uint32_t*>(&dd);
      }
      tmem_st_32x32b_x16(tm_S + col, pk);
      tmem_st_32x32b_x16(tm_dP + col, dk);
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (trs) trace[7 * 64 + idx] = clock64();
      if (lane == 0) mbar_arrive(&p_full[buf]);
      // the next tile's lse / D before this tile's dS-image stores: behind ~16 KB of global stores
      // per CTA in the LSU queue, these shared loads delayed the next tile's softmax by 400-800 clk
      if (idx + 1 < ntiles) load_ld(idx + 1);
      if (dsimg) {
        // dS for fa_bwd_dq_img: key row `key`, queries [64 i + 32 half, + 32) of query block i / 2,
        // written as the 128-byte row (key mod 64) of the MN-major SW128 image of dQ's A operand
        // (16-byte chunk c of row r at ((c ^ (r mod 8)) << 4), the layout TMA's 128B swizzle makes)
        const int qb = i >> 1, kt64 = key >> 6, r64 = key & 63;
        const size_t tri = static_cast<size_t>(s / kRows) * (s / kRows + 1);
        uint8_t* rowp = dsimg + ((static_cast<size_t>(bh) * tri + static_cast<size_t>(qb) * (qb + 1) + kt64) * 2 + (i & 1)) * 8192 +
                        r64 * 128;
        // logical chunks 2p, 2p + 1 land on the aligned physical pair (4 half + 2p) ^ (r mod 8 & 6): one
        // 32-byte store each (the lower half holds logical chunk 2p + (r & 1))
        const bool sw = (r64 & 1) != 0;
#pragma unroll
        for (int pp = 0; pp < 2; ++pp) {
          uint32_t v[8];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            v[e] = sw ? dk[8 * pp + 4 + e] : dk[8 * pp + e];
            v[4 + e] = sw ? dk[8 * pp + e] : dk[8 * pp + 4 + e];
          }
          st_global_v8(rowp + (((4 * half + 2 * pp) ^ (r64 & 6)) << 4), v);
        }
      }
    }
    if (half == 1) goto done_ts;
    mbar_wait(acc_done, 0);
    tc_fence_after();
    {
      const float scale = qk_scale;
      const bool tma_st = (s % kRows) == 0;
      // staging for the TMA stores: the (now idle) ring slots 0 and 1, four 128-row x 128-byte tiles
      auto stV = [&](int a) { return a ? sG(0) : sQ(0); };
      auto stK = [&](int a) { return a ? sG(1) : sQ(1); };
      const long krow_idx = static_cast<long>(b) * s + (key < s ? key : 0);
      bf16* krow = dqkv + krow_idx * (3 * h) + h + head * DH;
      bf16* vrow = krow + h;
#pragma unroll 1
      for (int c = 0; c < DH; c += 32) {
        uint32_t rv[32], rk[32];
        tmem_ld_32x32b_x32(tm_dV + c + lane_off, rv);
        tmem_ld_32x32b_x32(tm_dK + c + lane_off, rk);
        tmem_ld_wait();
        if (tma_st && kRingTS >= 2 && ntiles >= 2) {
          float fv[32], fk[32];
#pragma unroll
          for (int e = 0; e < 32; ++e) { fv[e] = __uint_as_float(rv[e]); fk[e] = __uint_as_float(rk[e]) * scale; }
          st_half_row_sw128(stV(c / 64), row, (c % 64) / 8, fv);
          st_half_row_sw128(stK(c / 64), row, (c % 64) / 8, fk);
        } else if (key < s) {
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            uint4 uv, uk;
            __nv_bfloat162* hv = reinterpret_cast<__nv_bfloat162*>(&uv);
            __nv_bfloat162* hk = reinterpret_cast<__nv_bfloat162*>(&uk);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              hv[e] = __floats2bfloat162_rn(__uint_as_float(rv[8 * q + 2 * e]), __uint_as_float(rv[8 * q + 2 * e + 1]));
              hk[e] = __floats2bfloat162_rn(__uint_as_float(rk[8 * q + 2 * e]) * scale,
                                            __uint_as_float(rk[8 * q + 2 * e + 1]) * scale);
            }
            *reinterpret_cast<uint4*>(vrow + c + 8 * q) = uv;
            *reinterpret_cast<uint4*>(krow + c + 8 * q) = uk;
          }
        }
      }
      if (tma_st && ntiles >= 2) {
        fence_proxy_async();
        named_bar(2, 128);
        if (threadIdx.x == 64) {
          const int r0 = b * s + kt * kRows;
#pragma unroll
          for (int a = 0; a < DH / 64; ++a) {
            tma_store_2d(&tm_dqkv, stV(a), 2 * h + head * DH + a * 64, r0);
            tma_store_2d(&tm_dqkv, stK(a), h + head * DH + a * 64, r0);
          }
          bulk_commit_wait_read();
        }
      }
    }
  }
done_ts:
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
  if (trace && threadIdx.x == 0 && blockIdx.x < 8192) {
    uint64_t gt;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
    trace[512 + 3 * blockIdx.x + 2] = static_cast<long long>(gt);
  }
}

// ----------------------------------------------------------------- dQ, persistent
// fa_bwd_dq_pers: the dQ kernel as a persistent grid (one CTA per SM) over work items (sample, head,
// 128-query tile) in the same heavy-first order, CTA c taking items c, c + grid, ... The per-CTA
// fixed cost of the one-item kernel (launch, TMEM allocation, the stationary Q/dO load, the dQ
// epilogue: ~30% of it at the cfg-2 shape) is paid once per SM: the producer streams the next
// item's Q/dO as soon as the last S/dP MMAs of the current one have read them, the dQ accumulator
// is double-buffered in TMEM (dQ0 | dQ1 | S x2 | dP x2 = 512 columns), and 4 dedicated epilogue
// warps drain dQ[n & 1] (tcgen05.ld -> scale -> bf16 -> global) while item n + 1 computes.
// Warps: 0 TMA, 1 MMA, 2..9 softmax (one query row per thread, 32 keys of the 64-key tile each),
// 10..13 epilogue. Counters (ring slot, S/dP buffer, dS buffer) run across items.
constexpr int kThreadsP = 448;
template <int DH>
__global__ void __launch_bounds__(kThreadsP, 1)
fa_bwd_dq_pers(const __grid_constant__ CUtensorMap tm_qkv128, const __grid_constant__ CUtensorMap tm_qkv64,
               const __grid_constant__ CUtensorMap tm_do128, const float* lse, const float* Dd, bf16* dqkv, int B,
               int s, int nh, float qk_scale) {
  using SM = Smem<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sG = sQ + SM::kBig;
  auto sK = [&](int r) { return sG + SM::kBig + 2 * r * SM::kSmall; };
  auto sV = [&](int r) { return sG + SM::kBig + 2 * r * SM::kSmall + SM::kSmall; };
  auto sS = [&](int i) { return sG + SM::kBig + 2 * kRing * SM::kSmall + i * SM::kP; };
  uint64_t* bar = reinterpret_cast<uint64_t*>(sS(1) + SM::kP);
  uint64_t* qd_full = bar;                // 1
  uint64_t* qd_empty = bar + 1;           // 1
  uint64_t* k_full = bar + 2;             // kRing
  uint64_t* k_empty = k_full + kRing;     // kRing
  uint64_t* s_full = k_empty + kRing;     // 2
  uint64_t* s_free = s_full + 2;          // 2
  uint64_t* p_full = s_free + 2;          // 2
  uint64_t* p_free = p_full + 2;          // 2
  uint64_t* acc_full = p_free + 2;        // 2
  uint64_t* acc_empty = acc_full + 2;     // 2
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_empty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nt = (s + kRows - 1) / kRows, BH = B * nh, W = nt * BH;
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const float sl2 = qk_scale * LOG2E;
  // item w -> (qt, b, head): heaviest query tiles first over all (sample, head)
  auto item = [&](int w, int& qt, int& b, int& head, int& ntiles) {
    const int j = w / BH, bh = w % BH;
    qt = nt - 1 - j; b = bh / nh; head = bh % nh;
    const int last_q = min(qt * kRows + kRows - 1, s - 1);
    ntiles = last_q / kCols + 1;
  };

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    tma_prefetch_desc(&tm_qkv64);
    tma_prefetch_desc(&tm_do128);
    mbar_init(qd_full, 1); mbar_init(qd_empty, 1);
    for (int i = 0; i < kRing; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1); mbar_init(&s_free[i], 8); mbar_init(&p_full[i], 8); mbar_init(&p_free[i], 1);
      mbar_init(&acc_full[i], 1); mbar_init(&acc_empty[i], 4);
    }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_dQ = tm, tm_S = tm + 2 * DH, tm_dP = tm + 2 * DH + 2 * kCols;

  if (warp == 0) {
    if (elect_one()) {
      int kc = 0, n = 0;
      for (int w = blockIdx.x; w < W; w += gridDim.x, ++n) {
        int qt, b, head, ntiles;
        item(w, qt, b, head, ntiles);
        const int row0 = b * s;
        mbar_wait(qd_empty, (n & 1) ^ 1);   // the previous item's S/dP MMAs are done with Q, dO
        mbar_arrive_expect_tx(qd_full, 2 * SM::kBig);
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_2d(sQ + a * (kRows * 128), &tm_qkv128, qd_full, head * DH + a * 64, row0 + qt * kRows);
          tma_load_2d(sG + a * (kRows * 128), &tm_do128, qd_full, head * DH + a * 64, row0 + qt * kRows);
        }
        for (int idx = 0; idx < ntiles; ++idx, ++kc) {
          const int st = kc % kRing;
          mbar_wait(&k_empty[st], ((kc / kRing) & 1) ^ 1);
          mbar_arrive_expect_tx(&k_full[st], 2 * SM::kSmall);
          const int kr = row0 + idx * kCols;
#pragma unroll
          for (int a = 0; a < DH / 64; ++a) {
            tma_load_2d(sK(st) + a * (kCols * 128), &tm_qkv64, &k_full[st], h + head * DH + a * 64, kr);
            tma_load_2d(sV(st) + a * (kCols * 128), &tm_qkv64, &k_full[st], 2 * h + head * DH + a * 64, kr);
          }
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(128, kCols, 0, 0);
    constexpr uint32_t id_a = umma_idesc_bf16(128, DH, 0, 1);   // dQ += dS K: B = K_j read MN-major
    int kc = 0, gc = 0, n = 0;
    for (int w = blockIdx.x; w < W; w += gridDim.x, ++n) {
      int qt, b, head, ntiles;
      item(w, qt, b, head, ntiles);
      const uint32_t dq_t = tm_dQ + (n & 1) * DH;
      mbar_wait(qd_full, n & 1);
      tc_fence_after();
      auto issue_s = [&](int idx) {
        const int st = (kc + idx) % kRing, g = gc + idx, buf = g & 1;
        mbar_wait(&k_full[st], ((kc + idx) / kRing) & 1);
        mbar_wait(&s_free[buf], ((g >> 1) & 1) ^ 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t q = smem_u32(sQ), gg = smem_u32(sG), k = smem_u32(sK(st)), v = smem_u32(sV(st));
#pragma unroll
          for (int kk = 0; kk < DH / 16; ++kk) {
            const uint32_t ao = (kk >> 2) * (kRows * 128) + (kk & 3) * 32, bo = (kk >> 2) * (kCols * 128) + (kk & 3) * 32;
            umma_bf16(tm_S + buf * kCols, umma_desc_sw128(q + ao, 16, 1024), umma_desc_sw128(k + bo, 16, 1024), id_s, kk > 0);
            umma_bf16(tm_dP + buf * kCols, umma_desc_sw128(gg + ao, 16, 1024), umma_desc_sw128(v + bo, 16, 1024), id_s, kk > 0);
          }
          umma_commit(&s_full[buf]);
          if (idx == ntiles - 1) umma_commit(qd_empty);   // Q/dO free once these MMAs complete
        }
        __syncwarp();
      };
      auto issue_acc = [&](int idx) {
        const int st = (kc + idx) % kRing, g = gc + idx, pb = g & 1;
        if (idx == 0) mbar_wait(&acc_empty[n & 1], ((n >> 1) & 1) ^ 1);   // dQ[n & 1] drained (item n - 2)
        mbar_wait(&p_full[pb], (g >> 1) & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t ds = smem_u32(sS(pb)), k = smem_u32(sK(st));
#pragma unroll
          for (int kk = 0; kk < kCols / 16; ++kk)
            umma_bf16(dq_t, umma_desc_sw128(ds + kk * 32, 16, 1024), umma_desc_sw128(k + kk * 2048, kCols * 128, 1024),
                      id_a, (idx | kk) != 0);
          umma_commit(&p_free[pb]);
          umma_commit(&k_empty[st]);
          if (idx == ntiles - 1) umma_commit(&acc_full[n & 1]);
        }
        __syncwarp();
      };
      issue_s(0);
      for (int idx = 1; idx < ntiles; ++idx) {
        issue_s(idx);
        issue_acc(idx - 1);
      }
      issue_acc(ntiles - 1);
      kc += ntiles;
      gc += ntiles;
    }
  } else if (warp < 10) {
    const int quarter = warp & 3, half = (warp - 2) >> 2;
    const int row = quarter * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    int gc = 0;
    for (int w = blockIdx.x; w < W; w += gridDim.x) {
      int qt, b, head, ntiles;
      item(w, qt, b, head, ntiles);
      const int q = qt * kRows + row;
      const long gr = static_cast<long>(b) * s + (q < s ? q : 0);
      const float L = lse[static_cast<long>(head) * Ttok + gr] * LOG2E;
      const float Dr = Dd[static_cast<long>(head) * Ttok + gr];
      for (int idx = 0; idx < ntiles; ++idx) {
        const int g = gc + idx, buf = g & 1;
        mbar_wait(&s_full[buf], (g >> 1) & 1);
        tc_fence_after();
        uint32_t sr[32], dr[32];
        tmem_ld_32x32b_x32(tm_S + buf * kCols + half * 32 + lane_off, sr);
        tmem_ld_32x32b_x32(tm_dP + buf * kCols + half * 32 + lane_off, dr);
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&s_free[buf]);
        float ds[32];
        if (idx * kCols + kCols - 1 > qt * kRows) {   // tile crosses the diagonal: causal mask
#pragma unroll
          for (int c = 0; c < 32; ++c) {
            const int key = idx * kCols + half * 32 + c;
            float pv = ex2(__uint_as_float(sr[c]) * sl2 - L);
            if (key > q) pv = 0.f;
            ds[c] = pv * (__uint_as_float(dr[c]) - Dr);
          }
        } else {
#pragma unroll
          for (int c = 0; c < 32; ++c) {
            const float pv = ex2(__uint_as_float(sr[c]) * sl2 - L);
            ds[c] = pv * (__uint_as_float(dr[c]) - Dr);
          }
        }
        mbar_wait(&p_free[buf], ((g >> 1) & 1) ^ 1);
        st_half_row_sw128(sS(buf), row, 4 * half, ds);
        fence_proxy_async();
        __syncwarp();
        if (lane == 0) mbar_arrive(&p_full[buf]);
      }
      gc += ntiles;
    }
  } else {
    // epilogue warps 10..13: TMEM lane quarter = warp & 3
    const int quarter = warp & 3;
    const int row = quarter * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const float scale = qk_scale;
    int n = 0;
    for (int w = blockIdx.x; w < W; w += gridDim.x, ++n) {
      int qt, b, head, ntiles;
      item(w, qt, b, head, ntiles);
      const int q = qt * kRows + row;
      bf16* qrow = dqkv + (static_cast<long>(b) * s + (q < s ? q : 0)) * (3 * h) + head * DH;
      mbar_wait(&acc_full[n & 1], (n >> 1) & 1);
      tc_fence_after();
#pragma unroll 1
      for (int c = 0; c < DH; c += 32) {
        uint32_t rq[32];
        tmem_ld_32x32b_x32(tm_dQ + (n & 1) * DH + c + lane_off, rq);
        tmem_ld_wait();
        if (c + 32 == DH) {   // every column of dQ[n & 1] is in registers: release it to the MMA warp
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&acc_empty[n & 1]);
        }
        if (q < s) {
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            uint4 u;
            __nv_bfloat162* hq = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
            for (int f = 0; f < 4; ++f)
              hq[f] = __floats2bfloat162_rn(__uint_as_float(rq[8 * e + 2 * f]) * scale,
                                            __uint_as_float(rq[8 * e + 2 * f + 1]) * scale);
            *reinterpret_cast<uint4*>(qrow + c + 8 * e) = u;
          }
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
}

// ------------------------------------------------------------------ dQ from the dS image
// fa_bwd_dq_img: dQ = dS K / sqrt(dh) with dS taken from the image fa_bwd_dkdv_ts wrote (when the
// caller provides the workspace), so nothing is recomputed: 1 MMA per tile instead of the 3 of the
// recomputing dQ kernels (S = Q K^T and dP = dO V^T again, plus the softmax). Image layout per
// (sample, head) and 128-query block qb: the 2 qb + 2 key tiles of 64 (causal) at index
// qb (qb + 1) + kt, each 2 x 8 KB boxes (queries [0,64) / [64,128) of the block) holding 64 key rows
// x 64 queries, MN-major with the 128-byte swizzle -- exactly the shared-memory image of the MMA's
// A operand (M = queries, K = keys), so the producer moves it with one 16 KB bulk copy.
// Persistent (one CTA per SM) over items (query block, sample, head), heaviest first. Warps: 0 TMA,
// 1 MMA (dQ double-buffered in TMEM), 2..5 epilogue (one query row per thread).
constexpr int kThreadsI = 192;
#ifndef MARIO_DQI_RING
#define MARIO_DQI_RING 3
#endif
constexpr int kRingI = MARIO_DQI_RING;   // 2 CTAs per SM (TMEM 2 x 256 columns)
template <int DH>
struct SmemI {
  static constexpr int kA = kRows * kCols * 2;       // 16 KB dS image tile
  static constexpr int kK = kCols * DH * 2;          // K tile (64 keys)
  static constexpr int kStage = kA + kK;
  static constexpr int kBytes = kRingI * kStage + 256 + 1024;
};
template <int DH>
__global__ void __launch_bounds__(kThreadsI, 1)
fa_bwd_dq_img(const __grid_constant__ CUtensorMap tm_qkv64, const uint8_t* __restrict__ dsimg, bf16* dqkv, int B, int s,
              int nh, int l2hint, float qk_scale, float* bpart) {
  using SI = SmemI<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + kRingI * SI::kStage);
  uint64_t* full = bar;                    // kRingI
  uint64_t* empty = full + kRingI;         // kRingI
  uint64_t* acc_full = empty + kRingI;     // 2
  uint64_t* acc_empty = acc_full + 2;      // 2
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_empty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nt = s / kRows, BH = B * nh, W = nt * BH;
  const int h = nh * DH;
  const size_t tri = static_cast<size_t>(nt) * (nt + 1);
  auto item = [&](int w, int& qb, int& bh, int& ntiles) {
    qb = nt - 1 - w / BH; bh = w % BH;
    ntiles = 2 * qb + 2;
  };
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv64);
    for (int i = 0; i < kRingI; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&acc_full[i], 1); mbar_init(&acc_empty[i], 4); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<2 * DH>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;

  if (warp == 0) {
    if (elect_one()) {
      const uint64_t pf_ = l2hint ? pol_first() : pol_normal(), pl_ = l2hint ? pol_last() : pol_normal();
      int kc = 0;
      for (int w = blockIdx.x; w < W; w += gridDim.x) {
        int qb, bh, ntiles;
        item(w, qb, bh, ntiles);
        const int b = bh / nh, head = bh % nh;
        const uint8_t* img = dsimg + (static_cast<size_t>(bh) * tri + static_cast<size_t>(qb) * (qb + 1)) * SI::kA;
        for (int kt = 0; kt < ntiles; ++kt, ++kc) {
          const int st = kc % kRingI;
          uint8_t* sa = smem + st * SI::kStage;
          mbar_wait(&empty[st], ((kc / kRingI) & 1) ^ 1);
          mbar_arrive_expect_tx(&full[st], SI::kStage);
          bulk_g2s_h(sa, img + static_cast<size_t>(kt) * SI::kA, SI::kA, &full[st], pf_);
#pragma unroll
          for (int a = 0; a < DH / 64; ++a)
            tma_load_2d_h(sa + SI::kA + a * (kCols * 128), &tm_qkv64, &full[st], h + head * DH + a * 64, b * s + kt * kCols,
                          pl_);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id = umma_idesc_bf16(128, DH, 1, 1);   // A = dS image (MN-major), B = K_j (MN-major)
    int kc = 0, n = 0;
    for (int w = blockIdx.x; w < W; w += gridDim.x, ++n) {
      int qb, bh, ntiles;
      item(w, qb, bh, ntiles);
      const uint32_t acc = tm + (n & 1) * DH;
      mbar_wait(&acc_empty[n & 1], ((n >> 1) & 1) ^ 1);
      tc_fence_after();
      for (int kt = 0; kt < ntiles; ++kt, ++kc) {
        const int st = kc % kRingI;
        mbar_wait(&full[st], (kc / kRingI) & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t sa = smem_u32(smem + st * SI::kStage), sk = sa + SI::kA;
#pragma unroll
          for (int kk = 0; kk < kCols / 16; ++kk)
            umma_bf16(acc, umma_desc_sw128(sa + kk * 2048, 8192, 1024), umma_desc_sw128(sk + kk * 2048, kCols * 128, 1024),
                      id, (kt | kk) != 0);
          umma_commit(&empty[st]);
          if (kt == ntiles - 1) umma_commit(&acc_full[n & 1]);
        }
        __syncwarp();
      }
    }
  } else {
    const int quarter = warp & 3;
    const int row = quarter * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const float scale = qk_scale;
    int n = 0;
    for (int w = blockIdx.x; w < W; w += gridDim.x, ++n) {
      int qb, bh, ntiles;
      item(w, qb, bh, ntiles);
      const int b = bh / nh, head = bh % nh;
      bf16* qrow = dqkv + (static_cast<long>(b) * s + qb * kRows + row) * (3 * h) + head * DH;
      mbar_wait(&acc_full[n & 1], (n >> 1) & 1);
      tc_fence_after();
#pragma unroll 1
      for (int c = 0; c < DH; c += 32) {
        uint32_t rq[32];
        tmem_ld_32x32b_x32(tm + (n & 1) * DH + c + lane_off, rq);
        tmem_ld_wait();
        if (c + 32 == DH) {
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&acc_empty[n & 1]);
        }
        float cs[32];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          uint4 u;
          __nv_bfloat162* hq = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
          for (int f = 0; f < 4; ++f) {
            hq[f] = __floats2bfloat162_rn(__uint_as_float(rq[8 * e + 2 * f]) * scale,
                                          __uint_as_float(rq[8 * e + 2 * f + 1]) * scale);
            const float2 back = __bfloat1622float2(hq[f]);
            cs[8 * e + 2 * f] = back.x;
            cs[8 * e + 2 * f + 1] = back.y;
          }
          *reinterpret_cast<uint4*>(qrow + c + 8 * e) = u;
        }
        if (bpart) {
          // column sums of this warp's 32 stored rows x 32 columns (the q-bias gradient partial of its
          // 32-row block): a transposing butterfly, 16 + 8 + 4 + 2 + 1 shuffles; at each step a lane
          // keeps the half of its columns its lane bit selects and adds the partner's copy of that half,
          // so lane l ends with column l (fixed order: deterministic). The kernel is DRAM-bound on the
          // image, so these shuffles run in its shadow.
#pragma unroll
          for (int o = 16; o >= 1; o >>= 1) {
            const bool up = (lane & o) != 0;
#pragma unroll
            for (int j = 0; j < o; ++j) {
              const float send = up ? cs[j] : cs[j + o];
              const float keep = up ? cs[j + o] : cs[j];
              cs[j] = keep + __shfl_xor_sync(0xffffffffu, send, o);
            }
          }
          bpart[((static_cast<long>(b) * s + qb * kRows) / 32 + quarter) * (3 * h) + head * DH + c + lane] = cs[0];
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<2 * DH>(tm);
}

// ------------------------------------------------------------ dK / dV, 128-query tiles ("N128")
// fa_bwd_dkdv_n128: the dK/dV kernel with S^T / dP^T MMAs of N = 128 queries. Measured
// (tools/mma_rate.cu, one CTA per SM, back-to-back issue): an M128 K16 tcgen05.mma takes ~72 clk at
// N = 128 and ~74 clk at N = 64 -- the N = 64 S^T / dP^T of fa_bwd_dkdv_ts run at 43% of the tensor
// core's rate, which is what bounded that kernel (its tensor pipe is busy ~1900 clk per 64-query tile).
// At N = 128 the four products of a tile (S^T, dP^T; dV += P^T dO, dK += dS^T Q with P^T / dS^T
// from TMEM) are all ~full-rate MMAs. TMEM: dV | dK | S^T (128 cols) | dP^T (128 cols) = 512 at dh
// 128, so S^T / dP^T are single-buffered; the MMA thread issues S(i), dP(i), then dV(i) once P(i)
// is in TMEM, dK(i) once dS(i) is, then S(i + 1), dP(i + 1) right behind them: tcgen05.mma executes
// in issue order, so S(i + 1) cannot overwrite the P^T(i) columns before dV(i) has read them (the
// same reliance as MARIO_ATTN_BWD_INORDER of fa_bwd_dkdv_ts, measured bitwise equal). The softmax
// (8 warps: TMEM lane quarter = warp & 3, query half = 64 columns) computes P(i) while dP(i) runs and
// dS(i) while dV(i) runs. One CTA per item: a persistent form (snake item order, which balances the
// causal item weights like dynamic dispatch; next item's S/dP MMAs overlapping the dV/dK epilogue) is
// bitwise equal but measured slower, 256.6 -> 260.8 us, because its epilogue must store dV/dK from
// registers (ring slot 0, the TMA-store staging here, is then in use): 16-byte stores across 32 rows
// per warp instruction cost 13 us over the TMA store (profiles/r02/attn_bwd_pers_ab.jsonl).
// Same arithmetic in the same order as fa_bwd_dkdv_ts: dQKV bitwise equal
// (tools/ab_n128.sh); attention backward 267.4 -> 256.6 us at the cfg-2 shape, 433.8 -> 417.7 us at
// B 1, s 4096, 32 heads. Polynomial exponentials for a share of P (as the forward) measured neutral or
// slower here, so the SFU is not this kernel's pace. Writes the same dS image as fa_bwd_dkdv_ts (one
// 8 KB box per query half). s % 128 == 0 only.
constexpr int kRingN = 2;
template <int DH>
struct SmemN {
  static constexpr int kTile = kRows * DH * 2;                 // 128-row K, V, Q or dO tile
  static constexpr int kLD = 2 * kRows * 4;                    // lse, D of a 128-query tile
  static constexpr int kBytes = 2 * kTile + kRingN * 2 * kTile + kRingN * kLD + 256 + 1024;
};
template <int DH>
__global__ void __launch_bounds__(kThreadsB, 1)
fa_bwd_dkdv_n128(const __grid_constant__ CUtensorMap tm_qkv128, const __grid_constant__ CUtensorMap tm_do128,
                 const __grid_constant__ CUtensorMap tm_dqkv, const float* lse, const float* Dd, bf16* dqkv, int B,
                 int s, int nh, uint8_t* dsimg, float qk_scale, float* bpart) {
  using SN = SmemN<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sK = smem;
  uint8_t* sV = sK + SN::kTile;
  auto sQ = [&](int r) { return sV + SN::kTile + r * 2 * SN::kTile; };
  auto sG = [&](int r) { return sV + SN::kTile + r * 2 * SN::kTile + SN::kTile; };
  float* sLD = reinterpret_cast<float*>(sV + SN::kTile + kRingN * 2 * SN::kTile);   // [ring][2][128]
  uint64_t* bar = reinterpret_cast<uint64_t*>(sLD + kRingN * 2 * kRows);
  uint64_t* kv_full = bar;                 // 1
  uint64_t* q_full = bar + 1;              // kRingN
  uint64_t* q_empty = q_full + kRingN;     // kRingN
  uint64_t* s_full = q_empty + kRingN;     // 1  S^T(i) in TMEM
  uint64_t* dp_full = s_full + 1;          // 1  dP^T(i) in TMEM
  uint64_t* p_full = dp_full + 1;          // 1  P^T(i) packed (8 softmax warps)
  uint64_t* ds_full = p_full + 1;          // 1  dS^T(i) packed (8 softmax warps)
  uint64_t* acc_done = ds_full + 1;        // 1
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_done + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int BH = B * nh;
  const int kt = blockIdx.x / BH, bh = blockIdx.x % BH, b = bh / nh, head = bh % nh;   // heaviest first
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const int nq = s / kRows;
  const int ntiles = nq - kt;              // query tiles kt .. nq - 1 (tile kt is the diagonal)
  const float sl2 = qk_scale * LOG2E;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    tma_prefetch_desc(&tm_do128);
    mbar_init(kv_full, 1);
    for (int i = 0; i < kRingN; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
    mbar_init(s_full, 1); mbar_init(dp_full, 1); mbar_init(p_full, 8); mbar_init(ds_full, 8); mbar_init(acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_dV = tm, tm_dK = tm + DH, tm_S = tm + 2 * DH, tm_dP = tm + 2 * DH + kRows;

  if (warp == 0) {
    if (elect_one()) {
      const int row0 = b * s;
      mbar_arrive_expect_tx(kv_full, 2 * SN::kTile);
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) {
        tma_load_2d(sK + a * (kRows * 128), &tm_qkv128, kv_full, h + head * DH + a * 64, row0 + kt * kRows);
        tma_load_2d(sV + a * (kRows * 128), &tm_qkv128, kv_full, 2 * h + head * DH + a * 64, row0 + kt * kRows);
      }
      for (int idx = 0; idx < ntiles; ++idx) {
        const int st = idx % kRingN;
        mbar_wait(&q_empty[st], ((idx / kRingN) & 1) ^ 1);
        mbar_arrive_expect_tx(&q_full[st], 2 * SN::kTile + SN::kLD);
        const int qr = row0 + (kt + idx) * kRows;
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_2d(sQ(st) + a * (kRows * 128), &tm_qkv128, &q_full[st], head * DH + a * 64, qr);
          tma_load_2d(sG(st) + a * (kRows * 128), &tm_do128, &q_full[st], head * DH + a * 64, qr);
        }
        const long o = static_cast<long>(head) * Ttok + qr;
        bulk_g2s(sLD + st * 2 * kRows, lse + o, kRows * 4, &q_full[st]);
        bulk_g2s(sLD + st * 2 * kRows + kRows, Dd + o, kRows * 4, &q_full[st]);
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(128, kRows, 0, 0);   // S^T, dP^T: K-major A and B, N = 128
    constexpr uint32_t id_a = umma_idesc_bf16(128, DH, 0, 1);      // dV, dK: A from TMEM, B MN-major
    mbar_wait(kv_full, 0);
    tc_fence_after();
    for (int idx = 0; idx < ntiles; ++idx) {
      const int st = idx % kRingN, par = idx & 1;
      mbar_wait(&q_full[st], (idx / kRingN) & 1);
      tc_fence_after();
      const uint32_t k = smem_u32(sK), v = smem_u32(sV), q = smem_u32(sQ(st)), g = smem_u32(sG(st));
      if (elect_one()) {
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const uint32_t o = (kk >> 2) * (kRows * 128) + (kk & 3) * 32;
          umma_bf16(tm_S, umma_desc_sw128(k + o, 16, 1024), umma_desc_sw128(q + o, 16, 1024), id_s, kk > 0);
        }
        umma_commit(s_full);
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const uint32_t o = (kk >> 2) * (kRows * 128) + (kk & 3) * 32;
          umma_bf16(tm_dP, umma_desc_sw128(v + o, 16, 1024), umma_desc_sw128(g + o, 16, 1024), id_s, kk > 0);
        }
        umma_commit(dp_full);
      }
      __syncwarp();
      mbar_wait(p_full, par);
      tc_fence_after();
      if (elect_one()) {
#pragma unroll
        for (int kk = 0; kk < kRows / 16; ++kk) {
          // queries [16kk, 16kk + 16): half kk / 4 packed them at columns 64 (kk / 4) + 8 (kk % 4)
          const uint32_t ac = (kk >> 2) * 64 + (kk & 3) * 8;
          umma_bf16_ts(tm_dV, tm_S + ac, umma_desc_sw128(g + kk * 2048, kRows * 128, 1024), id_a, (idx | kk) != 0);
        }
      }
      __syncwarp();
      mbar_wait(ds_full, par);
      tc_fence_after();
      if (elect_one()) {
#pragma unroll
        for (int kk = 0; kk < kRows / 16; ++kk) {
          const uint32_t ac = (kk >> 2) * 64 + (kk & 3) * 8;
          umma_bf16_ts(tm_dK, tm_dP + ac, umma_desc_sw128(q + kk * 2048, kRows * 128, 1024), id_a, (idx | kk) != 0);
        }
        umma_commit(&q_empty[st]);
        if (idx == ntiles - 1) umma_commit(acc_done);
      }
      __syncwarp();
    }
  } else {
    const int quarter = warp & 3, half = (warp - 2) >> 2;   // S^T columns (queries) [64 half, 64 half + 64)
    const int row = quarter * 32 + lane;                     // key row within the block
    const int key = kt * kRows + row;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const uint32_t col = half * 64 + lane_off;
    for (int idx = 0; idx < ntiles; ++idx) {
      const int i = kt + idx, st = idx % kRingN, par = idx & 1;
      const float* ld = sLD + st * 2 * kRows + half * 64;
      mbar_wait(&q_full[st], (idx / kRingN) & 1);   // lse / D of this tile (the MMA thread saw it complete)
      mbar_wait(s_full, par);
      tc_fence_after();
      float p[64];
      {
        uint32_t sr[32];
#pragma unroll
        for (int hh = 0; hh < 2; ++hh) {
          tmem_ld_32x32b_x32(tm_S + col + hh * 32, sr);
          tmem_ld_wait();
#pragma unroll
          for (int c = 0; c < 32; c += 4) {
            const float4 l4 = ld_shared_f4(ld + hh * 32 + c);
            const float lv[4] = {l4.x * LOG2E, l4.y * LOG2E, l4.z * LOG2E, l4.w * LOG2E};
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const int cc = hh * 32 + c + e;
              p[cc] = ex2(__uint_as_float(sr[c + e]) * sl2 - lv[e]);
            }
          }
        }
      }
      if (i == kt) {   // diagonal tile: P^T[key][q] = 0 for q < key
        const int lo = row - half * 64;
#pragma unroll
        for (int c = 0; c < 64; ++c) p[c] = c < lo ? 0.f : p[c];
      }
      {
        uint32_t pk[32];
#pragma unroll
        for (int c = 0; c < 64; c += 2) {
          const __nv_bfloat162 pp = __floats2bfloat162_rn(p[c], p[c + 1]);
          pk[c / 2] = *reinterpret_cast<const uint32_t*>(&pp);
        }
        tmem_st_32x32b_x32(tm_S + col, pk);
        tmem_st_wait();
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(p_full);
      mbar_wait(dp_full, par);
      tc_fence_after();
      uint32_t dk[32];
      {
        uint32_t dr[32];
#pragma unroll
        for (int hh = 0; hh < 2; ++hh) {
          tmem_ld_32x32b_x32(tm_dP + col + hh * 32, dr);
          tmem_ld_wait();
#pragma unroll
          for (int c = 0; c < 32; c += 4) {
            const float4 d4 = ld_shared_f4(ld + kRows + hh * 32 + c);
            const int cc = hh * 32 + c;
            const float d0 = p[cc] * (__uint_as_float(dr[c]) - d4.x), d1 = p[cc + 1] * (__uint_as_float(dr[c + 1]) - d4.y);
            const float d2 = p[cc + 2] * (__uint_as_float(dr[c + 2]) - d4.z), d3 = p[cc + 3] * (__uint_as_float(dr[c + 3]) - d4.w);
            const __nv_bfloat162 a0 = __floats2bfloat162_rn(d0, d1), a1 = __floats2bfloat162_rn(d2, d3);
            dk[cc / 2] = *reinterpret_cast<const uint32_t*>(&a0);
            dk[cc / 2 + 1] = *reinterpret_cast<const uint32_t*>(&a1);
          }
        }
      }
      tmem_st_32x32b_x32(tm_dP + col, dk);
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(ds_full);
      if (dsimg) {
        // dS image (fa_bwd_dq_img's A operand): query block i, 64-key tile key / 64, box = query half;
        // key row (key mod 64) as the 128-byte row of an MN-major SW128 tile (16-byte chunk c of row r
        // at ((c ^ (r mod 8)) << 4)); chunks 2p, 2p + 1 land on the aligned pair (2p ^ (r & 6)), swapped
        // when r is odd: one 32-byte store per pair
        const int kt64 = key >> 6, r64 = key & 63;
        const size_t tri = static_cast<size_t>(nq) * (nq + 1);
        uint8_t* rowp = dsimg + ((static_cast<size_t>(bh) * tri + static_cast<size_t>(i) * (i + 1) + kt64) * 2 + half) * 8192 +
                        r64 * 128;
        const bool sw = (r64 & 1) != 0;
#pragma unroll
        for (int pp = 0; pp < 4; ++pp) {
          uint32_t v8[8];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            v8[e] = sw ? dk[8 * pp + 4 + e] : dk[8 * pp + e];
            v8[4 + e] = sw ? dk[8 * pp + e] : dk[8 * pp + 4 + e];
          }
          st_global_v8(rowp + (((2 * pp) ^ (r64 & 6)) << 4), v8);
        }
      }
    }
    // epilogue: dV and dK (scaled by 1/sqrt(dh)) through the idle ring slot 0 as SW128 K-major tiles
    // of 128 rows x 64 columns, TMA-stored; the two query halves take half of the columns each
    mbar_wait(acc_done, 0);
    tc_fence_after();
    auto stV = [&](int a) { return sQ(0) + a * (kRows * 128); };
    auto stK = [&](int a) { return sG(0) + a * (kRows * 128); };
#pragma unroll 1
    for (int c = half * (DH / 2); c < (half + 1) * (DH / 2); c += 32) {
      uint32_t rv[32], rk[32];
      tmem_ld_32x32b_x32(tm_dV + c + lane_off, rv);
      tmem_ld_32x32b_x32(tm_dK + c + lane_off, rk);
      tmem_ld_wait();
      float fv[32], fk[32];
#pragma unroll
      for (int e = 0; e < 32; ++e) { fv[e] = __uint_as_float(rv[e]); fk[e] = __uint_as_float(rk[e]) * qk_scale; }
      st_half_row_sw128(stV(c / 64), row, (c % 64) / 8, fv);
      st_half_row_sw128(stK(c / 64), row, (c % 64) / 8, fk);
    }
    fence_proxy_async();
    named_bar(1, 256);
    if (threadIdx.x == 64) {
      const int r0 = b * s + kt * kRows;
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) {
        tma_store_2d(&tm_dqkv, stV(a), 2 * h + head * DH + a * 64, r0);
        tma_store_2d(&tm_dqkv, stK(a), h + head * DH + a * 64, r0);
      }
      bulk_commit_wait_read();
    }
    if (bpart) {
      // column sums of the staged bf16 dV / dK tiles (exactly what is stored), per 32-row block in
      // row order: bpart[(token / 32)][3h] gets the qkv-bias gradient partials of the k and v columns.
      // Thread t: 16-byte chunk column j = t % 32 (8 columns of dV, then dK) over the 32 rows of row
      // block t / 32 -- a warp reads whole 128-byte swizzled rows (4 wavefronts per instruction).
      // Read alongside the TMA store: both only read the staging tiles.
      const int t = threadIdx.x - 64, j = t % 32, q = t / 32;
      constexpr int kChunks = 2 * DH / 8;
      if (j < kChunks && q < kRows / 32) {
        const bool isK = j >= DH / 8;
        const int cc = isK ? j - DH / 8 : j;            // chunk within the tile's row (8 columns)
        const uint8_t* tile = isK ? stK(cc / 8) : stV(cc / 8);
        float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll 4
        for (int r = 32 * q; r < 32 * q + 32; ++r) {
          const uint4 u = *reinterpret_cast<const uint4*>(tile + r * 128 + (((cc % 8) ^ (r & 7)) << 4));
          const __nv_bfloat162* hh = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float2 f = __bfloat1622float2(hh[e]);
            acc[2 * e] += f.x;
            acc[2 * e + 1] += f.y;
          }
        }
        float* dst = bpart + ((static_cast<long>(b) * s + kt * kRows) / 32 + q) * (3 * h) + (isK ? h : 2 * h) +
                     head * DH + cc * 8;
        *reinterpret_cast<float4*>(dst) = make_float4(acc[0], acc[1], acc[2], acc[3]);
        *reinterpret_cast<float4*>(dst + 4) = make_float4(acc[4], acc[5], acc[6], acc[7]);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
}

// ------------------------------------------------------------------- dQ, 128-key tiles
// fa_bwd_dq_n128: the recomputing dQ kernel (no dS image: cfg 5's s = 16384, whose image would be
// 10.8 GB, and callers without a workspace) on 128-key tiles, the mirror of fa_bwd_dkdv_n128: one CTA
// per 128 queries (TMEM lanes), heaviest query blocks first; S = Q K_j^T and dP = dO V_j^T as M128 N128
// K16 MMAs (the N = 64 tiles of fa_bwd_dq_pers run at 43% of the tensor rate), dS = P (dP - D) packed
// to bf16 in place over dP by 8 softmax warps (lane quarter x 64-key half; lse and D are row constants
// in registers), dQ += dS K_j with A from TMEM. TMEM dQ | S | dP. The MMA thread issues S(j+1) as soon
// as the softmax has S(j) in registers (s_free), dQ(j) once dS(j) is in TMEM, then dP(j+1): dP(j+1)
// overwrites the dS(j) columns only after dQ(j) read them (tcgen05.mma executes in issue order).
// K/V tiles stream through a 2-deep ring; the dQ tile goes out through the idle Q/dO staging by TMA.
// Same arithmetic in the same order as fa_bwd_dq_pers (dQ bitwise equal). s % 128 == 0 only.
template <int DH>
struct SmemQN {
  static constexpr int kTile = kRows * DH * 2;                 // 128-row Q, dO, K or V tile
  static constexpr int kBytes = 2 * kTile + kRingN * 2 * kTile + 256 + 1024;
};
template <int DH>
__global__ void __launch_bounds__(kThreadsB, 1)
fa_bwd_dq_n128(const __grid_constant__ CUtensorMap tm_qkv128, const __grid_constant__ CUtensorMap tm_do128,
               const __grid_constant__ CUtensorMap tm_dqkv, const float* lse, const float* Dd, int B, int s, int nh,
               float qk_scale) {
  using SQ = SmemQN<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sG = sQ + SQ::kTile;
  auto sK = [&](int r) { return sG + SQ::kTile + r * 2 * SQ::kTile; };
  auto sV = [&](int r) { return sG + SQ::kTile + r * 2 * SQ::kTile + SQ::kTile; };
  uint64_t* bar = reinterpret_cast<uint64_t*>(sG + SQ::kTile + kRingN * 2 * SQ::kTile);
  uint64_t* qd_full = bar;                 // 1
  uint64_t* kv_full = bar + 1;             // kRingN
  uint64_t* kv_empty = kv_full + kRingN;   // kRingN
  uint64_t* s_full = kv_empty + kRingN;    // 1  S(j) in TMEM
  uint64_t* s_free = s_full + 1;           // 1  S(j) read by the softmax (8 warps)
  uint64_t* dp_full = s_free + 1;          // 1  dP(j) in TMEM
  uint64_t* ds_full = dp_full + 1;         // 1  dS(j) packed (8 warps)
  uint64_t* acc_done = ds_full + 1;        // 1
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_done + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int BH = B * nh, nt = s / kRows;
  const int qb = nt - 1 - static_cast<int>(blockIdx.x) / BH, bh = blockIdx.x % BH, b = bh / nh, head = bh % nh;
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const int ntiles = qb + 1;               // key tiles 0 .. qb (tile qb is the diagonal)
  const float sl2 = qk_scale * LOG2E;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    tma_prefetch_desc(&tm_do128);
    mbar_init(qd_full, 1);
    for (int i = 0; i < kRingN; ++i) { mbar_init(&kv_full[i], 1); mbar_init(&kv_empty[i], 1); }
    mbar_init(s_full, 1); mbar_init(s_free, 8); mbar_init(dp_full, 1); mbar_init(ds_full, 8); mbar_init(acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_dQ = tm, tm_S = tm + DH, tm_dP = tm + DH + kRows;

  if (warp == 0) {
    if (elect_one()) {
      const int row0 = b * s;
      mbar_arrive_expect_tx(qd_full, 2 * SQ::kTile);
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) {
        tma_load_2d(sQ + a * (kRows * 128), &tm_qkv128, qd_full, head * DH + a * 64, row0 + qb * kRows);
        tma_load_2d(sG + a * (kRows * 128), &tm_do128, qd_full, head * DH + a * 64, row0 + qb * kRows);
      }
      for (int j = 0; j < ntiles; ++j) {
        const int st = j % kRingN;
        mbar_wait(&kv_empty[st], ((j / kRingN) & 1) ^ 1);
        mbar_arrive_expect_tx(&kv_full[st], 2 * SQ::kTile);
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_2d(sK(st) + a * (kRows * 128), &tm_qkv128, &kv_full[st], h + head * DH + a * 64, row0 + j * kRows);
          tma_load_2d(sV(st) + a * (kRows * 128), &tm_qkv128, &kv_full[st], 2 * h + head * DH + a * 64, row0 + j * kRows);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(128, kRows, 0, 0);   // S, dP: K-major A and B, N = 128
    constexpr uint32_t id_a = umma_idesc_bf16(128, DH, 0, 1);      // dQ: A = dS from TMEM, B = K MN-major
    mbar_wait(qd_full, 0);
    tc_fence_after();
    const uint32_t q = smem_u32(sQ), gg = smem_u32(sG);
    auto issue_s = [&](int j) {   // S(j) = Q K_j^T
      const int st = j % kRingN;
      mbar_wait(&kv_full[st], (j / kRingN) & 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t k = smem_u32(sK(st));
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const uint32_t o = (kk >> 2) * (kRows * 128) + (kk & 3) * 32;
          umma_bf16(tm_S, umma_desc_sw128(q + o, 16, 1024), umma_desc_sw128(k + o, 16, 1024), id_s, kk > 0);
        }
        umma_commit(s_full);
      }
      __syncwarp();
    };
    auto issue_dp = [&](int j) {   // dP(j) = dO V_j^T (K/V of tile j already waited for by issue_s)
      const int st = j % kRingN;
      if (elect_one()) {
        const uint32_t v = smem_u32(sV(st));
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const uint32_t o = (kk >> 2) * (kRows * 128) + (kk & 3) * 32;
          umma_bf16(tm_dP, umma_desc_sw128(gg + o, 16, 1024), umma_desc_sw128(v + o, 16, 1024), id_s, kk > 0);
        }
        umma_commit(dp_full);
      }
      __syncwarp();
    };
    issue_s(0);
    issue_dp(0);
    for (int j = 0; j < ntiles; ++j) {
      const int st = j % kRingN;
      if (j + 1 < ntiles) {
        mbar_wait(s_free, j & 1);   // the softmax holds S(j) in registers
        issue_s(j + 1);
      }
      mbar_wait(ds_full, j & 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t k = smem_u32(sK(st));
#pragma unroll
        for (int kk = 0; kk < kRows / 16; ++kk) {
          // keys [16kk, 16kk + 16): half kk / 4 packed them at columns 64 (kk / 4) + 8 (kk % 4)
          const uint32_t ac = (kk >> 2) * 64 + (kk & 3) * 8;
          umma_bf16_ts(tm_dQ, tm_dP + ac, umma_desc_sw128(k + kk * 2048, kRows * 128, 1024), id_a, (j | kk) != 0);
        }
        umma_commit(&kv_empty[st]);
        if (j == ntiles - 1) umma_commit(acc_done);
      }
      __syncwarp();
      if (j + 1 < ntiles) issue_dp(j + 1);
    }
  } else {
    const int quarter = warp & 3, half = (warp - 2) >> 2;   // S columns (keys) [64 half, 64 half + 64)
    const int row = quarter * 32 + lane;                     // query row within the block
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const uint32_t col = half * 64 + lane_off;
    const long gr = static_cast<long>(b) * s + qb * kRows + row;
    const float L = lse[static_cast<long>(head) * Ttok + gr] * LOG2E;
    const float Dr = Dd[static_cast<long>(head) * Ttok + gr];
    for (int j = 0; j < ntiles; ++j) {
      const int par = j & 1;
      mbar_wait(s_full, par);
      tc_fence_after();
      float p[64];
      {
        uint32_t sr[64];
        tmem_ld_32x32b_x32(tm_S + col, *reinterpret_cast<uint32_t(*)[32]>(&sr[0]));
        tmem_ld_32x32b_x32(tm_S + col + 32, *reinterpret_cast<uint32_t(*)[32]>(&sr[32]));
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(s_free);
#pragma unroll
        for (int c = 0; c < 64; ++c) p[c] = ex2(__uint_as_float(sr[c]) * sl2 - L);
      }
      if (j == qb) {   // diagonal tile: P[q][key] = 0 for key > q
        const int hi = row - half * 64;
#pragma unroll
        for (int c = 0; c < 64; ++c) p[c] = c > hi ? 0.f : p[c];
      }
      mbar_wait(dp_full, par);
      tc_fence_after();
      uint32_t dk[32];
      {
        uint32_t dr[32];
#pragma unroll
        for (int hh = 0; hh < 2; ++hh) {
          tmem_ld_32x32b_x32(tm_dP + col + hh * 32, dr);
          tmem_ld_wait();
#pragma unroll
          for (int c = 0; c < 32; c += 2) {
            const int cc = hh * 32 + c;
            const __nv_bfloat162 d2 = __floats2bfloat162_rn(p[cc] * (__uint_as_float(dr[c]) - Dr),
                                                            p[cc + 1] * (__uint_as_float(dr[c + 1]) - Dr));
            dk[cc / 2] = *reinterpret_cast<const uint32_t*>(&d2);
          }
        }
      }
      tmem_st_32x32b_x32(tm_dP + col, dk);
      tmem_st_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(ds_full);
    }
    // epilogue: dQ (scaled by 1/sqrt(dh)) through the idle Q / dO tiles as SW128 K-major 128 x 64 tiles,
    // TMA-stored; the two halves take half of the columns each
    mbar_wait(acc_done, 0);
    tc_fence_after();
    auto stQ = [&](int a) { return a < 2 ? sQ + a * (kRows * 128) : sG + (a - 2) * (kRows * 128); };
#pragma unroll 1
    for (int c0 = half * (DH / 2); c0 < (half + 1) * (DH / 2); c0 += 32) {
      uint32_t rq[32];
      tmem_ld_32x32b_x32(tm_dQ + c0 + lane_off, rq);
      tmem_ld_wait();
      float fq[32];
#pragma unroll
      for (int e = 0; e < 32; ++e) fq[e] = __uint_as_float(rq[e]) * qk_scale;
      st_half_row_sw128(stQ(c0 / 64), row, (c0 % 64) / 8, fq);
    }
    fence_proxy_async();
    named_bar(1, 256);
    if (threadIdx.x == 64) {
      const int r0 = b * s + qb * kRows;
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) tma_store_2d(&tm_dqkv, stQ(a), head * DH + a * 64, r0);
      bulk_commit_wait_read();
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
}

// >= 116 KB so that one CTA owns the SM (each allocates all 512 TMEM columns)
constexpr int at_least_one_sm(int b) { return b < 116 * 1024 ? 116 * 1024 : b; }
template <int DH>
constexpr int smem_dkdv() { return at_least_one_sm(2 * Smem<DH>::kBig + 2 * kRingKV * Smem<DH>::kSmall + 4 * Smem<DH>::kP + kRingKV * 2 * kCols * 4 + 256 + 1024); }
template <int DH>
constexpr int smem_dq() { return at_least_one_sm(2 * Smem<DH>::kBig + 2 * kRing * Smem<DH>::kSmall + 2 * Smem<DH>::kP + 256 + 1024); }
template <int DH>
constexpr int smem_dkdv_ts() { return at_least_one_sm(2 * Smem<DH>::kBig + 2 * kRingTS * Smem<DH>::kSmall + kRingTS * 2 * kCols * 4 + 256 + 1024); }
int g_attn_dq_pers = 1;   // MARIO_ATTN_DQ_PERS=0 selects the one-item-per-CTA dQ kernel

template <int DH>
bool launch(const bf16* qkv, const bf16* dO, const float* lse, const float* Dd, bf16* dqkv, int B, int s, int nh,
            uint8_t* dsimg, cudaStream_t st, float qk_scale, float* bpart, bool* bpart_done) {
  if (bpart_done) *bpart_done = false;
  const int h = nh * DH;
  const long T = static_cast<long>(B) * s;
  CUtensorMap m128, m64, d64, d128, g128;
  if (!make_tmap_bf16_2d(&m128, qkv, 3 * h, T, 3 * h, 64, 128) || !make_tmap_bf16_2d(&m64, qkv, 3 * h, T, 3 * h, 64, 64) ||
      !make_tmap_bf16_2d(&d64, dO, h, T, h, 64, 64) || !make_tmap_bf16_2d(&d128, dO, h, T, h, 64, 128) ||
      !make_tmap_bf16_2d(&g128, dqkv, 3 * h, T, 3 * h, 64, 128))
    return false;
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(fa_bwd_dkdv_tc<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_dkdv<DH>());
    cudaFuncSetAttribute(fa_bwd_dq_tc<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_dq<DH>());
    set = true;
  }
  dim3 grid(B * nh * ((s + kRows - 1) / kRows));
  // experiment knob (results are wrong when bits 0-2 or 4 are set): bit 0 skips the softmax
  // arithmetic and P/dS stores, bit 1 skips the S/dP MMAs, bit 2 skips the accumulate MMAs, bit 3
  // orders CTAs (sample, head)-major, bit 4 skips the streamed TMA loads
  const char* dbgs = getenv("MARIO_ATTN_DBG");
  const int dbg = dbgs ? atoi(dbgs) : 0;
  const char* only = getenv("MARIO_ATTN_TC_ONLY");   // debugging aid: "dkdv" or "dq"
  if (!only || only[1] == 'k')
  {
    static long long* trace = nullptr;
    const bool want_trace = getenv("MARIO_ATTN_TRACE") != nullptr;
    constexpr size_t kTraceWords = 8 * 64 + 3 * 8192;
    if (want_trace && !trace) { cudaMalloc(&trace, kTraceWords * sizeof(long long)); cudaMemset(trace, 0, kTraceWords * sizeof(long long)); }
    static const bool ts = getenv("MARIO_ATTN_DKDV_TS") ? atoi(getenv("MARIO_ATTN_DKDV_TS")) != 0 : true;
    if (dsimg && (s % kRows) != 0) dsimg = nullptr;
    if (!(ts && dbg == 0)) dsimg = nullptr;
    if (ts && dbg == 0) {
      static bool tset = false;
      if (!tset) {
        cudaFuncSetAttribute(fa_bwd_dkdv_ts<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_dkdv_ts<DH>());
        tset = true;
      }
      static const int inorder = getenv("MARIO_ATTN_BWD_INORDER") ? atoi(getenv("MARIO_ATTN_BWD_INORDER")) : 0;
      // 128-query tiles (fa_bwd_dkdv_n128) where s % 128 == 0 (MARIO_ATTN_DKDV_N128 = 0: the 64-query-
      // tile kernel, also the traced one)
      static const int n128 = getenv("MARIO_ATTN_DKDV_N128") ? atoi(getenv("MARIO_ATTN_DKDV_N128")) : 1;
      if (n128 && (s % kRows) == 0 && !want_trace) {
        static bool nset = false;
        if (!nset) {
          cudaFuncSetAttribute(fa_bwd_dkdv_n128<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, SmemN<DH>::kBytes);
          nset = true;
        }
        // the qkv-bias column partials come from this kernel (k, v) and fa_bwd_dq_img (q): both or none
        const bool bp = bpart && dsimg && (!only || only[1] == 'k');
        fa_bwd_dkdv_n128<DH><<<grid, kThreadsB, SmemN<DH>::kBytes, st>>>(m128, d128, g128, lse, Dd, dqkv, B, s, nh,
                                                                           dsimg, qk_scale, bp ? bpart : nullptr);
        if (bp && bpart_done) *bpart_done = true;
      } else
      fa_bwd_dkdv_ts<DH><<<grid, kThreadsB, smem_dkdv_ts<DH>(), st>>>(m128, m64, d64, g128, lse, Dd, dqkv, B, s, nh,
                                                                        dsimg, attn_l2hint(), qk_scale,
                                                                        want_trace ? trace : nullptr, inorder);
    } else {
      fa_bwd_dkdv_tc<DH><<<grid, kThreadsB, smem_dkdv<DH>(), st>>>(m128, m64, d64, g128, lse, Dd, dqkv, B, s, nh, dbg,
                                                                     want_trace ? trace : nullptr, qk_scale);
    }
    if (want_trace) {
      long long h[8 * 64];
      cudaStreamSynchronize(st);
      cudaMemcpy(h, trace, sizeof(h), cudaMemcpyDeviceToHost);
      const long long t0 = h[0];
      fprintf(stderr, "tile   s_req    s_go  acc_req  acc_go | sm_req   sm_go   sm_ld  sm_done\n");
      for (int i = 0; i < 32; ++i)
        fprintf(stderr, "%3d %8lld %8lld %8lld %8lld | %8lld %8lld %8lld %8lld\n", i, h[i] - t0, h[64 + i] - t0,
                h[128 + i] - t0, h[192 + i] - t0, h[256 + i] - t0, h[320 + i] - t0, h[384 + i] - t0, h[448 + i] - t0);
      const char* dump = getenv("MARIO_ATTN_TRACE_CTAS");   // file for the per-CTA (sm, start, end) records
      if (dump && grid.x <= 8192) {
        std::vector<long long> c(3 * grid.x);
        cudaMemcpy(c.data(), trace + 512, c.size() * sizeof(long long), cudaMemcpyDeviceToHost);
        if (FILE* f = fopen(dump, "w")) {
          for (unsigned j = 0; j < grid.x; ++j) fprintf(f, "%u %lld %lld %lld\n", j, c[3 * j], c[3 * j + 1], c[3 * j + 2]);
          fclose(f);
        }
      }
    }
  }
  static const bool pers = getenv("MARIO_ATTN_DQ_PERS") ? atoi(getenv("MARIO_ATTN_DQ_PERS")) != 0 : g_attn_dq_pers != 0;
  if (only && only[1] == 'q') dsimg = nullptr;
  if (dsimg && (!only || only[1] == 'q')) {
    static bool iset = false;
    if (!iset) {
      cudaFuncSetAttribute(fa_bwd_dq_img<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, SmemI<DH>::kBytes);
      iset = true;
    }
    const int sms = device_sm_count();
    const int items = B * nh * (s / kRows);
    static const int per_sm = getenv("MARIO_DQI_CTAS") ? atoi(getenv("MARIO_DQI_CTAS")) : 2;
    const int grid_i = items < per_sm * sms ? items : per_sm * sms;
    fa_bwd_dq_img<DH><<<grid_i, kThreadsI, SmemI<DH>::kBytes, st>>>(m64, dsimg, dqkv, B, s, nh, attn_l2hint(),
                                                                     qk_scale, (bpart_done && *bpart_done) ? bpart : nullptr);
  } else if (!only || only[1] == 'q') {
    // 128-key tiles (fa_bwd_dq_n128) where s % 128 == 0: 1835 -> 1601 us for the whole backward at B 1,
    // s 16384, 8 heads; 532 -> 489 us at s 4096 (dQ bitwise equal); MARIO_ATTN_DQ_N128=0: fa_bwd_dq_pers
    static const int qn128 = getenv("MARIO_ATTN_DQ_N128") ? atoi(getenv("MARIO_ATTN_DQ_N128")) : 1;
    if (qn128 && dbg == 0 && (s % kRows) == 0) {
      static bool qset = false;
      if (!qset) {
        cudaFuncSetAttribute(fa_bwd_dq_n128<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, SmemQN<DH>::kBytes);
        qset = true;
      }
      fa_bwd_dq_n128<DH><<<B * nh * (s / kRows), kThreadsB, SmemQN<DH>::kBytes, st>>>(m128, d128, g128, lse, Dd, B, s,
                                                                                      nh, qk_scale);
    } else if (pers && dbg == 0) {
      static bool pset = false;
      if (!pset) {
        cudaFuncSetAttribute(fa_bwd_dq_pers<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_dq<DH>());
        pset = true;
      }
      const int sms = device_sm_count();
      const int items = B * nh * ((s + kRows - 1) / kRows);
      fa_bwd_dq_pers<DH><<<items < sms ? items : sms, kThreadsP, smem_dq<DH>(), st>>>(m128, m64, d128, lse, Dd, dqkv,
                                                                                         B, s, nh, qk_scale);
    } else {
      fa_bwd_dq_tc<DH><<<grid, kThreadsB, smem_dq<DH>(), st>>>(m128, m64, d128, g128, lse, Dd, dqkv, B, s, nh, dbg,
                                                               qk_scale);
    }
  }
  note_launch(2);
  return true;
}


// ------------------------------------------------------------------------------ forward
// One CTA per 128 queries (TMEM lanes); loop over 64-key tiles j <= last query:
//   MMA thread: S_j = Q K_j^T (M128 N64) into a double-buffered TMEM pair, PV_j = P_j V_j
//   (M128 N=dh, fresh accumulator per tile, double-buffered) once P_j is in smem.
//   4 softmax warps (one query row per thread): online max/sum, P_j (bf16, swizzled smem),
//   and O (fp32 registers) += PV_{j-1} one tile late so the PV MMA latency is hidden:
//   O <- O * exp(m_{j-2} - m_{j-1}) + PV_{j-1}.
template <int DH>
__global__ void __launch_bounds__(kThreadsB, 1)
fa_fwd_tc(const __grid_constant__ CUtensorMap tm_qkv128, const __grid_constant__ CUtensorMap tm_qkv64, bf16* O,
          float* lse, int B, int s, int nh, float qk_scale) {
  using SM = Smem<DH>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK[kRing];
  uint8_t* sV[kRing];
  for (int r = 0; r < kRing; ++r) { sK[r] = sQ + SM::kBig + 2 * r * SM::kSmall; sV[r] = sK[r] + SM::kSmall; }
  uint8_t* sP[2] = {sQ + SM::kBig + 2 * kRing * SM::kSmall, sQ + SM::kBig + 2 * kRing * SM::kSmall + SM::kP};
  float* xch = reinterpret_cast<float*>(sP[1] + SM::kP);   // [2 halves][128 rows] max / sum exchange
  uint64_t* bar = reinterpret_cast<uint64_t*>(xch + 2 * kRows);
  uint64_t* q_fullb = bar;                // 1
  uint64_t* k_full = bar + 1;             // kRing
  uint64_t* k_empty = k_full + kRing;     // kRing
  uint64_t* s_full = k_empty + kRing;     // 2
  uint64_t* s_free = s_full + 2;          // 2
  uint64_t* p_full = s_free + 2;          // 2
  uint64_t* o_full = p_full + 2;          // 2  (PV_j done: also frees P_j smem)
  uint64_t* o_free = o_full + 2;          // 2  (softmax read PV_j out of TMEM)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(o_free + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int qt = blockIdx.x, b = blockIdx.y / nh, head = blockIdx.y % nh;
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const int last_q = min(qt * kRows + kRows - 1, s - 1);
  const int ntiles = last_q / kCols + 1;
  const float sl2 = qk_scale * LOG2E;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    tma_prefetch_desc(&tm_qkv64);
    mbar_init(q_fullb, 1);
    for (int i = 0; i < kRing; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1); mbar_init(&s_free[i], 8);
      mbar_init(&p_full[i], 8); mbar_init(&o_full[i], 1); mbar_init(&o_free[i], 8);
    }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_S = tm, tm_O = tm + 2 * kCols;   // S[2] x 64 cols, PV[2] x DH cols

  if (warp == 0) {
    if (elect_one()) {
      const int row0 = b * s;
      mbar_arrive_expect_tx(q_fullb, SM::kBig);
#pragma unroll
      for (int a = 0; a < DH / 64; ++a)
        tma_load_2d(sQ + a * (kRows * 128), &tm_qkv128, q_fullb, head * DH + a * 64, row0 + qt * kRows);
      for (int j = 0; j < ntiles; ++j) {
        const int st = j % kRing;
        mbar_wait(&k_empty[st], ((j / kRing) & 1) ^ 1);
        mbar_arrive_expect_tx(&k_full[st], 2 * SM::kSmall);
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_2d(sK[st] + a * (kCols * 128), &tm_qkv64, &k_full[st], h + head * DH + a * 64, row0 + j * kCols);
          tma_load_2d(sV[st] + a * (kCols * 128), &tm_qkv64, &k_full[st], 2 * h + head * DH + a * 64, row0 + j * kCols);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(128, kCols, 0, 0);
    constexpr uint32_t id_o = umma_idesc_bf16(128, DH, 0, 1);   // PV: B = V_j read MN-major
    mbar_wait(q_fullb, 0);
    tc_fence_after();
    auto issue_s = [&](int j) {
      const int st = j % kRing, b2 = j & 1;
      mbar_wait(&k_full[st], (j / kRing) & 1);
      mbar_wait(&s_free[b2], ((j >> 1) & 1) ^ 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t q = smem_u32(sQ), k = smem_u32(sK[st]);
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const uint32_t ao = (kk >> 2) * (kRows * 128) + (kk & 3) * 32, bo = (kk >> 2) * (kCols * 128) + (kk & 3) * 32;
          umma_bf16(tm_S + b2 * kCols, umma_desc_sw128(q + ao, 16, 1024), umma_desc_sw128(k + bo, 16, 1024), id_s, kk > 0);
        }
        umma_commit(&s_full[b2]);
      }
      __syncwarp();
    };
    auto issue_pv = [&](int j) {
      const int st = j % kRing, b2 = j & 1;
      mbar_wait(&p_full[b2], (j >> 1) & 1);
      mbar_wait(&o_free[b2], ((j >> 1) & 1) ^ 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t p = smem_u32(sP[b2]), v = smem_u32(sV[st]);
#pragma unroll
        for (int kk = 0; kk < kCols / 16; ++kk)
          umma_bf16(tm_O + b2 * DH, umma_desc_sw128(p + kk * 32, 16, 1024),
                    umma_desc_sw128(v + kk * 2048, kCols * 128, 1024), id_o, kk > 0);
        umma_commit(&o_full[b2]);
        umma_commit(&k_empty[st]);
      }
      __syncwarp();
    };
    issue_s(0);
    for (int j = 1; j < ntiles; ++j) {
      issue_s(j);
      issue_pv(j - 1);
    }
    issue_pv(ntiles - 1);
  } else {
    // 8 softmax warps: warps w and w+4 share TMEM lane quarter (w & 3); `half` selects the 32 S
    // columns of each key tile and the DH/2 O columns this warp owns. The row max is exchanged
    // through smem each tile (64-thread named barrier per quarter); row sums stay partial.
    const int quarter = warp & 3, half = (warp - 2) >> 2;
    const int row = quarter * 32 + lane;
    const int q = qt * kRows + row;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    constexpr int HD = DH / 2;
    float o[HD];
#pragma unroll
    for (int d = 0; d < HD; ++d) o[d] = 0.f;
    float m_run = -INFINITY, l_run = 0.f;
    auto fold = [&](int j, float m_j, float m_before) {
      const int st = j & 1;
      mbar_wait(&o_full[st], (j >> 1) & 1);
      tc_fence_after();
      const float c = ex2(m_before - m_j);
#pragma unroll
      for (int c0 = 0; c0 < HD; c0 += 32) {
        uint32_t r[32];
        tmem_ld_32x32b_x32(tm_O + st * DH + half * HD + c0 + lane_off, r);
        tmem_ld_wait();
#pragma unroll
        for (int e = 0; e < 32; ++e) o[c0 + e] = o[c0 + e] * c + __uint_as_float(r[e]);
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&o_free[st]);
    };
    float m_pending = -INFINITY, m_folded = -INFINITY;
    for (int j = 0; j < ntiles; ++j) {
      const int st = j & 1;
      mbar_wait(&s_full[st], (j >> 1) & 1);
      tc_fence_after();
      uint32_t sr[32];
      tmem_ld_32x32b_x32(tm_S + st * kCols + half * 32 + lane_off, sr);
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&s_free[st]);
      // max over the raw scores (sl2 > 0), masked to -inf only on tiles crossing the diagonal;
      // then p = 2^(s * sl2 - m) as one FFMA + one MUFU per element
      float mr = -INFINITY;
      if (j * kCols + kCols - 1 > qt * kRows) {
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const int key = j * kCols + half * 32 + c;
          if (key > q) sr[c] = __float_as_uint(-INFINITY);
          mr = fmaxf(mr, __uint_as_float(sr[c]));
        }
      } else {
#pragma unroll
        for (int c = 0; c < 32; ++c) mr = fmaxf(mr, __uint_as_float(sr[c]));
      }
      const float mx = fmaxf(m_run, mr * sl2);
      st_shared_f32(&xch[half * kRows + row], mx);
      named_bar(2 + quarter, 64);
      const float m_new = fmaxf(mx, ld_shared_f32(&xch[(half ^ 1) * kRows + row]));   // finite: key 0 <= q
      named_bar(2 + quarter, 64);                                                      // xch reusable next tile
      float p[32], ls = 0.f;
#pragma unroll
      for (int c = 0; c < 32; ++c) {
        p[c] = ex2(fmaf(__uint_as_float(sr[c]), sl2, -m_new));
        ls += p[c];
      }
      l_run = l_run * ex2(m_run - m_new) + ls;
      m_run = m_new;
      st_half_row_sw128(sP[st], row, 4 * half, p);
      fence_proxy_async();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[st]);
      if (j > 0) {
        fold(j - 1, m_pending, m_folded);
        m_folded = m_pending;
      }
      m_pending = m_new;
    }
    fold(ntiles - 1, m_pending, m_folded);
    // total row sum = both halves' partial sums (same running max)
    st_shared_f32(&xch[half * kRows + row], l_run);
    named_bar(2 + quarter, 64);
    const float l_tot = l_run + ld_shared_f32(&xch[(half ^ 1) * kRows + row]);
    const float inv = 1.f / l_tot;
    if (q < s) {
      bf16* orow = O + (static_cast<long>(b) * s + q) * h + head * DH + half * HD;
#pragma unroll
      for (int d = 0; d < HD; d += 8) {
        uint4 u;
        __nv_bfloat162* hh = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
        for (int e = 0; e < 4; ++e) hh[e] = __floats2bfloat162_rn(o[d + 2 * e] * inv, o[d + 2 * e + 1] * inv);
        *reinterpret_cast<uint4*>(orow + d) = u;
      }
      if (half == 0) lse[static_cast<long>(head) * Ttok + static_cast<long>(b) * s + q] = (m_run + log2f(l_tot)) / LOG2E;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
}

// ------------------------------------------------------------- forward, two Q tiles
// fa_fwd2_tc: one CTA = 256 queries (Q tiles t = 0, 1 of 128 rows) of one (sample, head); keys in
// tiles of 128. Warpgroup 0: warp 0 TMA, warp 1 MMA (one elected thread), warps 2-3 idle; it
// gives registers away (setmaxnreg 56) to warpgroups 1 and 2 (224), the softmax of Q tile 0 and 1
// (one thread per query row, the whole 128-key S row in registers: no cross-thread max exchange). TMEM: S_0, S_1 (128 columns each), O_0, O_1 (DH each). The MMA
// warp interleaves the two tiles (S_0(j+1), S_1(j+1), PV_0(j), PV_1(j)) so one tile's softmax
// overlaps the other's MMAs. O accumulates in TMEM; the running max is only raised (and O, l
// rescaled in TMEM) when a row's max grows by more than 2^8 (warp-uniform decision), so most tiles
// need no correction. K/V tiles stream through a 3-slot TMA ring in the MMA's consumption order
// K0, K1, V0, K2, V1, ..., V_{n-1}. Causal: Q tile 0 of query block qb sees key tiles 0..2qb,
// tile 1 sees 0..2qb+1; only the last (diagonal) tile of each is masked.
constexpr int kF2Q = 128;        // rows per Q tile
constexpr int kF2N = 128;        // keys per tile
constexpr int kF2Threads = 384;
#ifndef MARIO_F2_STAGES
#define MARIO_F2_STAGES 3   // K/V ring depth of the two-Q-tile forward (A/B: NVCC_EXTRA=-DMARIO_F2_STAGES=n)
#endif
constexpr int kF2Stages = MARIO_F2_STAGES;
// per-thread register split after setmaxnreg: TMA / MMA warps vs the two softmax warpgroups
// (4 x 32 x CTRL + 8 x 32 x SMAX <= 65536)
#ifndef MARIO_F2_CTRL_REGS
#define MARIO_F2_CTRL_REGS "88"
#define MARIO_F2_SMAX_REGS "208"
#endif
#ifndef MARIO_F2_DBG
#define MARIO_F2_DBG 0   // 1: softmax exponentials replaced by an FMA (timing experiment only, wrong results)
#endif
#ifndef MARIO_POLY_EX2
#define MARIO_POLY_EX2 1
#endif
constexpr bool kPolyEx2 = MARIO_POLY_EX2 != 0;   // every 4th softmax exponential on the FMA pipe

template <int DH>
struct SmemF2 {
  static constexpr int kTile = kF2Q * DH * 2;       // a Q, K or V tile (bf16)
  static constexpr int kP = kF2Q * kF2N * 2;        // P tile (bf16)
  static constexpr int kBytes = 2 * kTile + kF2Stages * kTile + 2 * kP + 256 + 1024;
};

// which tile the i-th ring item is (load order == MMA consumption order)
__device__ __forceinline__ void f2_item(int i, int n, bool& is_v, int& j) {
  if (i == 0) { is_v = false; j = 0; return; }
  if (i == 2 * n - 1) { is_v = true; j = n - 1; return; }
  const int t = (i + 1) >> 1;       // i = 2t - 1 -> K_t, i = 2t -> V_{t-1}
  if (i & 1) { is_v = false; j = t; } else { is_v = true; j = t - 1; }
}

template <int DH>
__global__ void __launch_bounds__(kF2Threads, 1)
fa_fwd2_tc(const __grid_constant__ CUtensorMap tm_qkv128, bf16* O, float* lse, int B, int s, int nh, int g_l2hint,
           float qk_scale, long long* trace) {
  using SM = SmemF2<DH>;
  // trace (MARIO_ATTN_FWD_TRACE): per CTA (sm, start, end) globaltimer ns, for tools/attn_fwd_trace.py
  if (trace && threadIdx.x == 0) {
    uint64_t gt; uint32_t smid;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    trace[3 * blockIdx.x] = smid;
    trace[3 * blockIdx.x + 1] = static_cast<long long>(gt);
  }
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                                   // [2][kTile]
  uint8_t* sRing = sQ + 2 * SM::kTile;                  // [kF2Stages][kTile]
  uint8_t* sP = sRing + kF2Stages * SM::kTile;          // [2][kP]
  uint64_t* bar = reinterpret_cast<uint64_t*>(sP + 2 * SM::kP);
  uint64_t* q_full = bar;                          // 1
  uint64_t* full = bar + 1;                        // kF2Stages
  uint64_t* empty = full + kF2Stages;              // kF2Stages
  uint64_t* s_full = empty + kF2Stages;            // 2
  uint64_t* s_free = s_full + 2;                   // 2
  uint64_t* p_full = s_free + 2;                   // 2
  uint64_t* o_done = p_full + 2;                   // 2
  uint64_t* q_empty = o_done + 2;                  // 1  (persistent: the item's S MMAs are done with Q)
  uint64_t* o_free = q_empty + 1;                  // 2  (persistent: the epilogue has read O_t)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(o_free + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int BH = B * nh, nqb = (s + 2 * kF2Q - 1) / (2 * kF2Q);
  const int h = nh * DH;
  const long Ttok = static_cast<long>(B) * s;
  const float sl2 = qk_scale * LOG2E;
  // work items w = (query block, sample, head), heaviest query blocks first; a grid smaller than the
  // item count runs persistently, CTA c taking items in snake order (round r: r*G + c, or
  // r*G + G-1-c on odd rounds), which balances the causal item weights like dynamic dispatch. Item
  // n+1's Q load, K/V loads and S MMAs overlap item n's last PV and epilogue; barrier phases run on
  // across items (per-tile step bases). One CTA per item runs the same code for one round.
  const int W = nqb * BH, G = gridDim.x, cta = blockIdx.x;
  auto item_of = [=](int r) { const int w = r * G + ((r & 1) ? G - 1 - cta : cta); return w < W ? w : -1; };

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tm_qkv128);
    mbar_init(q_full, 1);
    for (int i = 0; i < kF2Stages; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int t = 0; t < 2; ++t) {
      mbar_init(&s_full[t], 1); mbar_init(&s_free[t], 4); mbar_init(&p_full[t], 4); mbar_init(&o_done[t], 1);
      mbar_init(&o_free[t], 4);
    }
    mbar_init(q_empty, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = *tmem_slot;
  const uint32_t tm_S0 = tm, tm_O0 = tm + 2 * kF2N;

  if (warp < 4) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 " MARIO_F2_CTRL_REGS ";");
  if (warp == 0) {
    if (elect_one()) {
      const uint64_t pf_ = g_l2hint ? pol_first() : pol_normal(), pl_ = g_l2hint ? pol_last() : pol_normal();
      int gi = 0;   // ring items across work items
      for (int n = 0;; ++n) {
        const int w = item_of(n);
        if (w < 0) break;
        const int qb = nqb - 1 - w / BH, bh = w % BH, b = bh / nh, head = bh % nh;
        const int q0 = qb * 2 * kF2Q, n1 = 2 * qb + 2, row0 = b * s;
        if (n > 0) mbar_wait(q_empty, (n - 1) & 1);   // the previous item's S MMAs have read Q
        mbar_arrive_expect_tx(q_full, 2 * SM::kTile);
#pragma unroll
        for (int t = 0; t < 2; ++t)
#pragma unroll
          for (int a = 0; a < DH / 64; ++a)
            tma_load_2d_h(sQ + t * SM::kTile + a * (kF2Q * 128), &tm_qkv128, q_full, head * DH + a * 64,
                          row0 + q0 + t * kF2Q, pf_);
        for (int i = 0; i < 2 * n1; ++i, ++gi) {
          bool is_v;
          int j;
          f2_item(i, n1, is_v, j);
          const int st = gi % kF2Stages;
          mbar_wait(&empty[st], ((gi / kF2Stages) & 1) ^ 1);
          mbar_arrive_expect_tx(&full[st], SM::kTile);
          uint8_t* dst = sRing + st * SM::kTile;
#pragma unroll
          for (int a = 0; a < DH / 64; ++a)
            tma_load_2d_h(dst + a * (kF2N * 128), &tm_qkv128, &full[st], (is_v ? 2 * h : h) + head * DH + a * 64,
                          row0 + j * kF2N, pl_);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t id_s = umma_idesc_bf16(kF2Q, kF2N, 0, 0);
    constexpr uint32_t id_o = umma_idesc_bf16(kF2Q, DH, 0, 1);   // B = V read MN-major
    int item = 0;                 // ring items across work items
    int base0 = 0, base1 = 0;     // per-tile S / PV count of the previous work items (barrier phases)
    for (int n = 0;; ++n) {
    const int w = item_of(n);
    if (w < 0) break;
    const int qb = nqb - 1 - w / BH;
    const int n0 = 2 * qb + 1, n1 = 2 * qb + 2;
    mbar_wait(q_full, n & 1);
    tc_fence_after();
    auto issue_s = [&](int j) {
      const int st = item % kF2Stages;
      mbar_wait(&full[st], (item / kF2Stages) & 1);
      for (int t = 0; t < 2; ++t) {
        if (t == 0 && j >= n0) continue;
        mbar_wait(&s_free[t], (((t ? base1 : base0) + j) & 1) ^ 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t q = smem_u32(sQ + t * SM::kTile), k = smem_u32(sRing + st * SM::kTile);
#pragma unroll
          for (int kk = 0; kk < DH / 16; ++kk) {
            const uint32_t ao = (kk >> 2) * (kF2Q * 128) + (kk & 3) * 32, bo = (kk >> 2) * (kF2N * 128) + (kk & 3) * 32;
            umma_bf16(tm_S0 + t * kF2N, umma_desc_sw128(q + ao, 16, 1024), umma_desc_sw128(k + bo, 16, 1024), id_s,
                      kk > 0);
          }
          umma_commit(&s_full[t]);
        }
        __syncwarp();
      }
      if (elect_one()) umma_commit(&empty[st]);
      __syncwarp();
      ++item;
    };
    auto issue_pv = [&](int j) {
      const int st = item % kF2Stages;
      mbar_wait(&full[st], (item / kF2Stages) & 1);
      for (int t = 0; t < 2; ++t) {
        if (t == 0 && j >= n0) continue;
        if (j == 0 && n > 0) mbar_wait(&o_free[t], (n - 1) & 1);   // the previous item's O_t read out
        mbar_wait(&p_full[t], ((t ? base1 : base0) + j) & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t p = smem_u32(sP + t * SM::kP), v = smem_u32(sRing + st * SM::kTile);
#pragma unroll
          for (int kk = 0; kk < kF2N / 16; ++kk) {
            const uint32_t ao = (kk >> 2) * (kF2Q * 128) + (kk & 3) * 32;
            umma_bf16(tm_O0 + t * DH, umma_desc_sw128(p + ao, 16, 1024),
                      umma_desc_sw128(v + kk * 2048, kF2N * 128, 1024), id_o, (j | kk) != 0);
          }
          umma_commit(&o_done[t]);
        }
        __syncwarp();
      }
      if (elect_one()) umma_commit(&empty[st]);
      __syncwarp();
      ++item;
    };
    issue_s(0);
    for (int j = 0; j < n1; ++j) {
      if (j + 1 < n1) issue_s(j + 1);
      if (j + 1 == n1 - 1 || (j == 0 && n1 == 1)) {   // every S MMA of the item issued: Q free when done
        if (elect_one()) umma_commit(q_empty);
        __syncwarp();
      }
      issue_pv(j);
    }
    base0 += n0;
    base1 += n1;
    }
  }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 " MARIO_F2_SMAX_REGS ";");
    const int t = (warp - 4) >> 2, quarter = warp & 3;
    const int row = quarter * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quarter * 32) << 16;
    const uint32_t tS = tm_S0 + t * kF2N + lane_off, tO = tm_O0 + t * DH + lane_off;
    uint8_t* myP = sP + t * SM::kP;
    int bs = 0;   // this tile's S / PV count of the previous work items
    for (int n = 0;; ++n) {
    const int w = item_of(n);
    if (w < 0) break;
    const int qb = nqb - 1 - w / BH;
    const int q = qb * 2 * kF2Q + t * kF2Q + row;
    const int nt = t == 0 ? 2 * qb + 1 : 2 * qb + 2;
    float m_used = -INFINITY, l = 0.f;
    for (int j = 0; j < nt; ++j) {
      mbar_wait(&s_full[t], (bs + j) & 1);
      tc_fence_after();
      uint32_t xr[kF2N];
#pragma unroll
      for (int c0 = 0; c0 < kF2N; c0 += 32) tmem_ld_32x32b_x32(tS + c0, *reinterpret_cast<uint32_t(*)[32]>(&xr[c0]));
      tmem_ld_wait();
      float* x = reinterpret_cast<float*>(xr);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&s_free[t]);   // S_t may be overwritten by the next tile's MMA
      if (j == nt - 1) {                         // diagonal tile: causal mask
#pragma unroll
        for (int c = 0; c < kF2N; ++c)
          if (j * kF2N + c > q) x[c] = -INFINITY;
      }
      float mr = x[0];
#pragma unroll
      for (int c = 1; c < kF2N; ++c) mr = fmaxf(mr, x[c]);
      const float m_cand = mr * sl2;
      bool waited = false;
      if (j == 0) {
        m_used = m_cand;                          // finite: key 0 <= q
      } else if (__any_sync(0xffffffffu, m_cand > m_used + 8.f)) {
        // raise the running max: O_t (after PV_t(j-1)) and l rescaled by 2^(m_old - m_new)
        mbar_wait(&o_done[t], (bs + j - 1) & 1);
        tc_fence_after();
        waited = true;
        const float m_new = fmaxf(m_used, m_cand);
        const float f = ex2(m_used - m_new);
        l *= f;
        m_used = m_new;
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 32) {
          uint32_t r[32];
          tmem_ld_32x32b_x32(tO + c0, r);
          tmem_ld_wait();
#pragma unroll
          for (int e = 0; e < 32; ++e) r[e] = __float_as_uint(__uint_as_float(r[e]) * f);
          tmem_st_32x32b_x32(tO + c0, r);
        }
        tmem_st_wait();
      }
      float ls = 0.f;
#pragma unroll
      for (int c = 0; c < kF2N; ++c) {
        const float arg = fmaf(x[c], sl2, -m_used);
#if MARIO_F2_DBG   // experiment: exponentials replaced by an FMA (wrong results) to time the softmax share
        x[c] = arg * 0.0009765625f + 1.f;
#else
        x[c] = (kPolyEx2 && (c & 3) == 3) ? ex2_poly(arg) : ex2(arg);
#endif
        ls += x[c];
      }
      l += ls;
      if (j > 0 && !waited) {                     // P_t smem is free once PV_t(j-1) completed
        mbar_wait(&o_done[t], (bs + j - 1) & 1);
      }
#pragma unroll
      for (int c0 = 0; c0 < kF2N; c0 += 32)
        st_half_row_sw128(myP + (c0 / 64) * (kF2Q * 128), row, (c0 % 64) / 8, *reinterpret_cast<float(*)[32]>(&x[c0]));
      fence_proxy_async();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[t]);
    }
    mbar_wait(&o_done[t], (bs + nt - 1) & 1);
    tc_fence_after();
    const float inv = 1.f / l;
    const int bh = w % BH, b = bh / nh, head = bh % nh;
    bf16* orow = O + (static_cast<long>(b) * s + (q < s ? q : 0)) * h + head * DH;
#pragma unroll 1
    for (int c0 = 0; c0 < DH; c0 += 32) {
      uint32_t r[32];
      tmem_ld_32x32b_x32(tO + c0, r);
      tmem_ld_wait();
      if (c0 + 32 == DH) {   // every column of O_t in registers: the next item's PV_t may overwrite it
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&o_free[t]);
      }
      if (q < s) {
#pragma unroll
        for (int d = 0; d < 32; d += 8) {
          uint4 u;
          __nv_bfloat162* hh = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
          for (int e = 0; e < 4; ++e)
            hh[e] = __floats2bfloat162_rn(__uint_as_float(r[d + 2 * e]) * inv, __uint_as_float(r[d + 2 * e + 1]) * inv);
          *reinterpret_cast<uint4*>(orow + c0 + d) = u;
        }
      }
    }
    if (q < s) lse[static_cast<long>(head) * Ttok + static_cast<long>(b) * s + q] = (m_used + log2f(l)) / LOG2E;
    bs += nt;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tm);
  if (trace && threadIdx.x == 0) {
    uint64_t gt;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
    trace[3 * blockIdx.x + 2] = static_cast<long long>(gt);
  }
}

template <int DH>
bool launch_fwd2_tc(const bf16* qkv, bf16* O, float* lse, int B, int s, int nh, cudaStream_t st, float qk_scale) {
  const int h = nh * DH;
  const long T = static_cast<long>(B) * s;
  CUtensorMap m128;
  if (!make_tmap_bf16_2d(&m128, qkv, 3 * h, T, 3 * h, 64, 128)) return false;
  constexpr int smem = SmemF2<DH>::kBytes < 116 * 1024 ? 116 * 1024 : SmemF2<DH>::kBytes;
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(fa_fwd2_tc<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    set = true;
  }
  const int nqb = (s + 2 * kF2Q - 1) / (2 * kF2Q);
  const int items = nqb * B * nh;
  // persistent (default; MARIO_ATTN_FWD_PERS=0: one CTA per item): one CTA per SM the launching thread
  // may use (its green-context partition in the emulated pipeline). The item -> CTA map does not change
  // any item's arithmetic: O and lse are bitwise those of the one-CTA-per-item launch. Measured 85.5 ->
  // 81.1 us at the cfg-2 shape (profiles/r02/attn_fwd_pers_ab.jsonl).
  static const int pers = getenv("MARIO_ATTN_FWD_PERS") ? atoi(getenv("MARIO_ATTN_FWD_PERS")) : 1;
  const int sms = device_sm_count();
  const int grid = (pers && items > sms) ? sms : items;
  static const char* tfile = getenv("MARIO_ATTN_FWD_TRACE");
  static long long* trace = nullptr;
  if (tfile && !trace) cudaMalloc(&trace, 3 * 65536 * sizeof(long long));
  fa_fwd2_tc<DH><<<grid, kF2Threads, smem, st>>>(m128, O, lse, B, s, nh, attn_l2hint(), qk_scale,
                                                 (tfile && grid <= 65536) ? trace : nullptr);
  if (tfile && grid <= 65536) {
    std::vector<long long> c(3 * grid);
    cudaStreamSynchronize(st);
    cudaMemcpy(c.data(), trace, c.size() * sizeof(long long), cudaMemcpyDeviceToHost);
    if (FILE* f = fopen(tfile, "w")) {
      for (int j = 0; j < grid; ++j) fprintf(f, "%d %lld %lld %lld\n", j, c[3 * j], c[3 * j + 1], c[3 * j + 2]);
      fclose(f);
    }
  }
  note_launch();
  return true;
}

template <int DH>
constexpr int smem_fwd() { return at_least_one_sm(Smem<DH>::kBig + 2 * kRing * Smem<DH>::kSmall + 2 * Smem<DH>::kP + 2 * kRows * 4 + 256 + 1024); }

template <int DH>
bool launch_fwd_tc(const bf16* qkv, bf16* O, float* lse, int B, int s, int nh, cudaStream_t st, float qk_scale) {
  const int h = nh * DH;
  const long T = static_cast<long>(B) * s;
  CUtensorMap m128, m64;
  if (!make_tmap_bf16_2d(&m128, qkv, 3 * h, T, 3 * h, 64, 128) || !make_tmap_bf16_2d(&m64, qkv, 3 * h, T, 3 * h, 64, 64))
    return false;
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(fa_fwd_tc<DH>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_fwd<DH>());
    set = true;
  }
  dim3 grid((s + kRows - 1) / kRows, B * nh);
  fa_fwd_tc<DH><<<grid, kThreadsB, smem_fwd<DH>(), st>>>(m128, m64, O, lse, B, s, nh, qk_scale);
  note_launch();
  return true;
}

}  // namespace

bool flash_attn_bwd_tc_supported(int dh, int B, int s, int nh) {
  return (dh == 64 || dh == 128) && ((nh * dh) % 64 == 0);
}

bool flash_attn_fwd_tc(const bf16* qkv, bf16* O, float* lse, int B, int s, int nh, int dh, cudaStream_t st,
                       float qk_scale) {
  if (qk_scale <= 0.f) qk_scale = rsqrtf(static_cast<float>(dh));
  // g_attn_variant: -1 auto (two-Q-tile kernel unless it would launch fewer CTAs than SMs: the
  // one-Q-tile kernel has twice as many), 2 force the one-Q-tile kernel, 3 force the two-Q-tile one.
  // The choice uses the whole GPU's SM count, not the thread's SM budget: the two kernels round
  // differently, and a stage must compute the same bits on an SM partition as in loopback.
  const int sms = device_sm_count_full();
  const long ctas2 = static_cast<long>((s + 2 * kF2Q - 1) / (2 * kF2Q)) * B * nh;
  if (g_attn_variant == 2 || (g_attn_variant != 3 && ctas2 < sms)) {
    if (dh == 128) return launch_fwd_tc<128>(qkv, O, lse, B, s, nh, st, qk_scale);
    if (dh == 64) return launch_fwd_tc<64>(qkv, O, lse, B, s, nh, st, qk_scale);
    return false;
  }
  if (dh == 128) return launch_fwd2_tc<128>(qkv, O, lse, B, s, nh, st, qk_scale);
  if (dh == 64) return launch_fwd2_tc<64>(qkv, O, lse, B, s, nh, st, qk_scale);
  return false;
}

// Returns false if the configuration is unsupported (caller falls back to the mma.sync kernels).
bool flash_attn_bwd_tc(const bf16* qkv, const bf16* dO, const float* lse, const float* Dd, bf16* dqkv, int B, int s,
                       int nh, int dh, void* ds_ws, size_t ds_ws_bytes, cudaStream_t st, float qk_scale, float* bpart,
                       bool* bpart_done) {
  if (bpart_done) *bpart_done = false;
  if (qk_scale <= 0.f) qk_scale = rsqrtf(static_cast<float>(dh));
  uint8_t* img = ds_ws && ds_ws_bytes >= flash_attn_bwd_ds_bytes(dh, B, s, nh) ? static_cast<uint8_t*>(ds_ws) : nullptr;
  if (dh == 128) return launch<128>(qkv, dO, lse, Dd, dqkv, B, s, nh, img, st, qk_scale, bpart, bpart_done);
  if (dh == 64) return launch<64>(qkv, dO, lse, Dd, dqkv, B, s, nh, img, st, qk_scale, bpart, bpart_done);
  return false;
}

// bytes of the dS image fa_bwd_dq_img reads (0: that path does not apply to this shape)
size_t flash_attn_bwd_ds_bytes(int dh, int B, int s, int nh) {
  if ((dh != 64 && dh != 128) || s % kRows != 0 || (nh * dh) % 64 != 0) return 0;
  const size_t nt = static_cast<size_t>(s / kRows);
  return static_cast<size_t>(B) * nh * nt * (nt + 1) * SmemI<128>::kA;
}

}  // namespace mario
