// K5-K15 — norms, attention, RoPE, SwiGLU, softmax-CE, embedding, reductions.
// Formulas: SURVEY §8(c) c1 (readings A1/A2), same definitions as oracle/model.py but an
// independent implementation (no shared code).
#include <cfloat>
#include <cstdint>
#include <cstdlib>
#include <type_traits>

#include "layers.h"
#include "kstats.h"

#include "kernels.h"

namespace mario {
namespace {

__device__ __forceinline__ float ldf(const float* p) { return *p; }
__device__ __forceinline__ float ldf(const __nv_bfloat16* p) { return __bfloat162float(*p); }
__device__ __forceinline__ void stf(float* p, float v) { *p = v; }
__device__ __forceinline__ void stf(__nv_bfloat16* p, float v) { *p = __float2bfloat16_rn(v); }

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

inline int cdiv(long a, long b) { return static_cast<int>((a + b - 1) / b); }
}  // namespace

// 3: warp-per-row v2 forward + row-pipelined backward; 2: row-pipelined (rowpipe.cu); 1: block-per-row-tile;
// 0: warp-per-row (A/B; env MARIO_NORM_VARIANT sets the initial value)
// Measured (tools/norm_fwd_perf.py, T = 8192): the v2 forward 20.6 -> 18.6 us (LN) / 18.6 -> 16.6 us
// (RMS) at n = 2048, 37.0 -> 35.4 us (LN) at 4096, slower at 5120 (41.3 -> 48.4 us), so variant 3
// takes widths <= 4096 and the row pipeline the rest.
int g_norm_tile = getenv("MARIO_NORM_VARIANT") ? atoi(getenv("MARIO_NORM_VARIANT")) : 3;

namespace {

// ------------------------------------------------------------------ embedding
template <class T>
__global__ void embed_fwd_k(const int32_t* tok, int ld_tok, int B, int s, const T* wte, const T* wpe, T* H, int h) {
  const long n = static_cast<long>(B) * s * h;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < n; i += static_cast<long>(gridDim.x) * blockDim.x) {
    const long r = i / h;
    const int c = static_cast<int>(i % h);
    const int b = static_cast<int>(r / s), t = static_cast<int>(r % s);
    const int x = tok[static_cast<long>(b) * ld_tok + t];
    float v = ldf(wte + static_cast<long>(x) * h + c);
    if (wpe) v += ldf(wpe + static_cast<long>(t) * h + c);
    stf(H + i, v);
  }
}

// bf16, h % 8 == 0: 16-byte chunks, 32-bit index math (the scalar kernel's 64-bit divisions per
// element made it 73 us per micro-batch at cfg 2); same fp32 sum and rounding, bitwise equal
__global__ void embed_fwd_v8_k(const int32_t* tok, int ld_tok, int s, const __nv_bfloat16* wte,
                               const __nv_bfloat16* wpe, __nv_bfloat16* H, int h8, int n8) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n8; i += gridDim.x * blockDim.x) {
    const int r = i / h8, c8 = i - r * h8;
    const int b = r / s, t = r - b * s;
    const int x = tok[static_cast<long>(b) * ld_tok + t];
    const uint4 a = reinterpret_cast<const uint4*>(wte)[static_cast<long>(x) * h8 + c8];
    uint4 o;
    const __nv_bfloat162* ha = reinterpret_cast<const __nv_bfloat162*>(&a);
    __nv_bfloat162* ho = reinterpret_cast<__nv_bfloat162*>(&o);
    if (wpe) {
      const uint4 p = reinterpret_cast<const uint4*>(wpe)[static_cast<long>(t) * h8 + c8];
      const __nv_bfloat162* hp = reinterpret_cast<const __nv_bfloat162*>(&p);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 fa = __bfloat1622float2(ha[e]), fp = __bfloat1622float2(hp[e]);
        ho[e] = __floats2bfloat162_rn(fa.x + fp.x, fa.y + fp.y);
      }
    } else {
      o = a;
    }
    reinterpret_cast<uint4*>(H)[i] = o;
  }
}

// one block bitonic sort of keys (token * T + index) in shared memory
__global__ void embed_sort_k(const int32_t* tok, int ld_tok, int B, int s, long long* keys_out, int npow2) {
  extern __shared__ long long sk[];
  const int T = B * s;
  for (int i = threadIdx.x; i < npow2; i += blockDim.x) {
    if (i < T) {
      const int b = i / s, t = i % s;
      sk[i] = static_cast<long long>(tok[static_cast<long>(b) * ld_tok + t]) * T + i;
    } else {
      sk[i] = LLONG_MAX;
    }
  }
  __syncthreads();
  for (int k = 2; k <= npow2; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < npow2; i += blockDim.x) {
        const int ixj = i ^ j;
        if (ixj > i) {
          const bool up = (i & k) == 0;
          const long long a = sk[i], c = sk[ixj];
          if ((a > c) == up) { sk[i] = c; sk[ixj] = a; }
        }
      }
      __syncthreads();
    }
  }
  for (int i = threadIdx.x; i < T; i += blockDim.x) keys_out[i] = sk[i];
}

// Longer micro-batches (B*s > kSortChunk, e.g. s > 16384 at mbs 1): every CTA bitonic-sorts one
// chunk of kSortChunk keys in shared memory, then merge passes double the sorted run length. Keys
// are unique (the position is part of the key), so the order is fully determined: each element's
// output index is its index in its own run plus the number of keys of the partner run that are
// smaller (binary search), with no atomics.
constexpr int kSortChunk = 16384;
__global__ void embed_sort_chunk_k(const int32_t* tok, int ld_tok, int s, int Ttok, long long* keys_out) {
  extern __shared__ long long sk[];
  const int c0 = blockIdx.x * kSortChunk;
  for (int i = threadIdx.x; i < kSortChunk; i += blockDim.x) {
    const int g = c0 + i;
    if (g < Ttok) {
      const int b = g / s, t = g % s;
      sk[i] = static_cast<long long>(tok[static_cast<long>(b) * ld_tok + t]) * Ttok + g;
    } else {
      sk[i] = LLONG_MAX;
    }
  }
  __syncthreads();
  for (int k = 2; k <= kSortChunk; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < kSortChunk; i += blockDim.x) {
        const int ixj = i ^ j;
        if (ixj > i) {
          const bool up = (i & k) == 0;
          const long long a = sk[i], c = sk[ixj];
          if ((a > c) == up) { sk[i] = c; sk[ixj] = a; }
        }
      }
      __syncthreads();
    }
  }
  for (int i = threadIdx.x; i < kSortChunk && c0 + i < Ttok; i += blockDim.x) keys_out[c0 + i] = sk[i];
}

__global__ void embed_merge_k(const long long* in, long long* out, int n, int width) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int run = i / width, pair0 = (run & ~1) * width;
  const bool left = (run & 1) == 0;
  const int own0 = left ? pair0 : pair0 + width;
  const int oth0 = left ? pair0 + width : pair0;
  const int oth_n = max(0, min(width, n - oth0));
  const long long k = in[i];
  int lo = 0, hi = oth_n;   // number of partner keys < k
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (in[oth0 + mid] < k) lo = mid + 1; else hi = mid;
  }
  out[pair0 + (i - own0) + lo] = k;
}

template <class T>
__global__ void embed_segsum_k(const long long* keys, int Ttok, const T* dH, int h, float* dwte) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) / 32, lane = threadIdx.x % 32;
  if (warp >= Ttok) return;
  const long long v = keys[warp] / Ttok;
  if (warp > 0 && keys[warp - 1] / Ttok == v) return;   // not a segment start
  for (int c = lane; c < h; c += 32) {
    float acc = 0.f;
    for (int j = warp; j < Ttok && keys[j] / Ttok == v; ++j) acc += ldf(dH + (keys[j] % Ttok) * h + c);
    dwte[v * h + c] += acc;
  }
}

// bf16, h % 8 == 0: one warp per segment (sorted positions sharing a token). The warp reads the
// segment's keys 32 at a time (one division per key, ballot for the segment end), and each lane then
// owns 8 consecutive columns per 16-byte load, adding the segment's rows in position order (the same
// order as the scalar kernel: bitwise-identical sums for segments of up to 32 positions). The scalar
// kernel re-divided every key for every column (179 us per micro-batch at cfg 2).
__global__ void embed_segsum_v8_k(const long long* keys, int Ttok, const __nv_bfloat16* dH, int h, float* dwte) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) / 32, lane = threadIdx.x % 32;
  if (warp >= Ttok) return;
  const long long v = keys[warp] / Ttok;
  if (warp > 0 && keys[warp - 1] / Ttok == v) return;
  float* out = dwte + v * h;
  for (int j0 = warp; j0 < Ttok;) {
    // this chunk of up to 32 segment members: lane i holds position of member j0 + i
    const int j = j0 + lane;
    const long long kj = j < Ttok ? keys[j] : LLONG_MAX;
    const bool in = j < Ttok && kj / Ttok == v;
    const unsigned m = __ballot_sync(0xffffffffu, in);
    const int cnt = __popc(~m) ? __ffs(~m) - 1 : 32;   // members are a prefix of the chunk
    const int pos = in ? static_cast<int>(kj % Ttok) : 0;
    for (int c8 = lane; c8 < h / 8; c8 += 32) {
      float acc[8];
      const float4 o0 = *reinterpret_cast<const float4*>(out + c8 * 8);
      const float4 o1 = *reinterpret_cast<const float4*>(out + c8 * 8 + 4);
      float sum[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
      for (int i = 0; i < cnt; ++i) {
        const int p = __shfl_sync(0xffffffffu, pos, i);
        const uint4 u = *reinterpret_cast<const uint4*>(dH + static_cast<long>(p) * h + c8 * 8);
        const __nv_bfloat162* hv = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float2 f = __bfloat1622float2(hv[e]);
          sum[2 * e] += f.x;
          sum[2 * e + 1] += f.y;
        }
      }
      acc[0] = o0.x + sum[0]; acc[1] = o0.y + sum[1]; acc[2] = o0.z + sum[2]; acc[3] = o0.w + sum[3];
      acc[4] = o1.x + sum[4]; acc[5] = o1.y + sum[5]; acc[6] = o1.z + sum[6]; acc[7] = o1.w + sum[7];
      *reinterpret_cast<float4*>(out + c8 * 8) = make_float4(acc[0], acc[1], acc[2], acc[3]);
      *reinterpret_cast<float4*>(out + c8 * 8 + 4) = make_float4(acc[4], acc[5], acc[6], acc[7]);
    }
    if (cnt < 32) break;
    j0 += 32;
  }
}

// fp32 dH (the bf16 model's fp32 residual-gradient stream, reading A30), h % 4 == 0: the v8
// kernel's segment walk with 4 columns per 16-byte load; same per-column summation order.
__global__ void embed_segsum_f4_k(const long long* keys, int Ttok, const float* dH, int h, float* dwte) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) / 32, lane = threadIdx.x % 32;
  if (warp >= Ttok) return;
  const long long v = keys[warp] / Ttok;
  if (warp > 0 && keys[warp - 1] / Ttok == v) return;
  float* out = dwte + v * h;
  for (int j0 = warp; j0 < Ttok;) {
    const int j = j0 + lane;
    const long long kj = j < Ttok ? keys[j] : LLONG_MAX;
    const bool in = j < Ttok && kj / Ttok == v;
    const unsigned m = __ballot_sync(0xffffffffu, in);
    const int cnt = __popc(~m) ? __ffs(~m) - 1 : 32;
    const int pos = in ? static_cast<int>(kj % Ttok) : 0;
    for (int c4 = lane; c4 < h / 4; c4 += 32) {
      float4 acc = *reinterpret_cast<const float4*>(out + c4 * 4);
      float4 sum = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int i = 0; i < cnt; ++i) {
        const int p = __shfl_sync(0xffffffffu, pos, i);
        const float4 u = *reinterpret_cast<const float4*>(dH + static_cast<long>(p) * h + c4 * 4);
        sum.x += u.x; sum.y += u.y; sum.z += u.z; sum.w += u.w;
      }
      acc.x += sum.x; acc.y += sum.y; acc.z += sum.z; acc.w += sum.w;
      *reinterpret_cast<float4*>(out + c4 * 4) = acc;
    }
    if (cnt < 32) break;
    j0 += 32;
  }
}

template <class T>
__global__ void embed_pos_bwd_k(const T* dH, int B, int s, int h, float* dwpe) {
  const long n = static_cast<long>(s) * h;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < n; i += static_cast<long>(gridDim.x) * blockDim.x) {
    const long t = i / h;
    const int c = static_cast<int>(i % h);
    float acc = 0.f;
    for (int b = 0; b < B; ++b) acc += ldf(dH + (static_cast<long>(b) * s + t) * h + c);
    dwpe[i] += acc;
  }
}

// bf16, h % 8 == 0: dwpe[t] += sum_b dH[b, t] in 16-byte chunks (same order: b ascending), 32-bit index math
__global__ void embed_pos_bwd_v8_k(const __nv_bfloat16* dH, int B, int s, int h8, float* dwpe) {
  const int n8 = s * h8;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n8; i += gridDim.x * blockDim.x) {
    float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
    for (int b = 0; b < B; ++b) {
      const uint4 u = reinterpret_cast<const uint4*>(dH)[static_cast<long>(b) * n8 + i];
      const __nv_bfloat162* hv = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 f = __bfloat1622float2(hv[e]);
        acc[2 * e] += f.x;
        acc[2 * e + 1] += f.y;
      }
    }
    float4* o = reinterpret_cast<float4*>(dwpe) + 2 * static_cast<long>(i);
    const float4 a = o[0], c = o[1];
    o[0] = make_float4(a.x + acc[0], a.y + acc[1], a.z + acc[2], a.w + acc[3]);
    o[1] = make_float4(c.x + acc[4], c.y + acc[5], c.z + acc[6], c.w + acc[7]);
  }
}

// ---------------------------------------------------------------------- norms
template <class T, bool RMS>
__global__ void norm_fwd_k(const T* x, const float* g, const float* b, T* y, float* stats, int rows, int n, float eps) {
  const int row = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (row >= rows) return;
  const T* xr = x + static_cast<long>(row) * n;
  float mean = 0.f;
  if (!RMS) {
    float s = 0.f;
    for (int c = lane; c < n; c += 32) s += ldf(xr + c);
    mean = warp_sum(s) / n;
  }
  float v = 0.f;
  for (int c = lane; c < n; c += 32) { const float d = ldf(xr + c) - mean; v += d * d; }
  const float rstd = rsqrtf(warp_sum(v) / n + eps);
  T* yr = y + static_cast<long>(row) * n;
  for (int c = lane; c < n; c += 32) {
    float o = (ldf(xr + c) - mean) * rstd * g[c];
    if (!RMS) o += b[c];
    stf(yr + c, o);
  }
  if (lane == 0) { stats[2 * row] = mean; stats[2 * row + 1] = rstd; }
}

// Row cached in registers: NV uint4 (8 bf16) per lane covers n <= 256 * NV.
template <bool RMS, int NV>
__global__ void norm_fwd_reg_k(const __nv_bfloat16* x, const float* g, const float* b, __nv_bfloat16* y, float* stats,
                               int rows, int n, float eps) {
  const int row = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (row >= rows) return;
  const __nv_bfloat16* xr = x + static_cast<long>(row) * n;
  uint4 v[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = (i * 32 + lane) * 8;
    v[i] = c < n ? *reinterpret_cast<const uint4*>(xr + c) : make_uint4(0, 0, 0, 0);
  }
  float mean = 0.f;
  if (!RMS) {
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < NV; ++i) {
      const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&v[i]);
#pragma unroll
      for (int j = 0; j < 8; ++j) s += __bfloat162float(hv[j]);
    }
    mean = warp_sum(s) / n;
  }
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = (i * 32 + lane) * 8;
    if (c >= n) continue;
    const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&v[i]);
#pragma unroll
    for (int j = 0; j < 8; ++j) { const float d = __bfloat162float(hv[j]) - mean; q += d * d; }
  }
  const float rstd = rsqrtf(warp_sum(q) / n + eps);
  __nv_bfloat16* yr = y + static_cast<long>(row) * n;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = (i * 32 + lane) * 8;
    if (c >= n) continue;
    const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&v[i]);
    const float4 g0 = *reinterpret_cast<const float4*>(g + c), g1 = *reinterpret_cast<const float4*>(g + c + 4);
    const float gg[8] = {g0.x, g0.y, g0.z, g0.w, g1.x, g1.y, g1.z, g1.w};
    float bb[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    if (!RMS) {
      const float4 b0 = *reinterpret_cast<const float4*>(b + c), b1 = *reinterpret_cast<const float4*>(b + c + 4);
      bb[0] = b0.x; bb[1] = b0.y; bb[2] = b0.z; bb[3] = b0.w; bb[4] = b1.x; bb[5] = b1.y; bb[6] = b1.z; bb[7] = b1.w;
    }
    uint4 o;
    __nv_bfloat16* ho = reinterpret_cast<__nv_bfloat16*>(&o);
#pragma unroll
    for (int j = 0; j < 8; ++j) ho[j] = __float2bfloat16_rn((__bfloat162float(hv[j]) - mean) * rstd * gg[j] + bb[j]);
    *reinterpret_cast<uint4*>(yr + c) = o;
  }
  if (lane == 0) { stats[2 * row] = mean; stats[2 * row + 1] = rstd; }
}

template <int NV>
__global__ void norm_bwd_dx_reg_k(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                                  const __nv_bfloat16* dres, __nv_bfloat16* dx, int rows, int n, int rms) {
  const int row = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (row >= rows) return;
  const long o = static_cast<long>(row) * n;
  const float mean = stats[2 * row], rstd = stats[2 * row + 1];
  uint4 vd[NV], vx[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = (i * 32 + lane) * 8;
    vd[i] = c < n ? *reinterpret_cast<const uint4*>(dy + o + c) : make_uint4(0, 0, 0, 0);
    vx[i] = c < n ? *reinterpret_cast<const uint4*>(x + o + c) : make_uint4(0, 0, 0, 0);
  }
  float sg = 0.f, sgx = 0.f;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = (i * 32 + lane) * 8;
    if (c >= n) continue;
    const __nv_bfloat16* hd = reinterpret_cast<const __nv_bfloat16*>(&vd[i]);
    const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&vx[i]);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float gp = __bfloat162float(hd[j]) * g[c + j];
      sg += gp;
      sgx += gp * (__bfloat162float(hx[j]) - mean) * rstd;
    }
  }
  sg = rms ? 0.f : warp_sum(sg) / n;
  sgx = warp_sum(sgx) / n;
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const int c = (i * 32 + lane) * 8;
    if (c >= n) continue;
    const __nv_bfloat16* hd = reinterpret_cast<const __nv_bfloat16*>(&vd[i]);
    const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&vx[i]);
    uint4 ur = make_uint4(0, 0, 0, 0);
    if (dres) ur = *reinterpret_cast<const uint4*>(dres + o + c);
    const __nv_bfloat16* hr = reinterpret_cast<const __nv_bfloat16*>(&ur);
    uint4 uo;
    __nv_bfloat16* ho = reinterpret_cast<__nv_bfloat16*>(&uo);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float gp = __bfloat162float(hd[j]) * g[c + j];
      const float xh = (__bfloat162float(hx[j]) - mean) * rstd;
      float d = (gp - sg - xh * sgx) * rstd;
      if (dres) d += __bfloat162float(hr[j]);
      ho[j] = __float2bfloat16_rn(d);
    }
    *reinterpret_cast<uint4*>(dx + o + c) = uo;
  }
}

template <bool RMS>
__global__ void norm_fwd_v8_k(const __nv_bfloat16* x, const float* g, const float* b, __nv_bfloat16* y, float* stats,
                              int rows, int n, float eps) {
  const int row = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (row >= rows) return;
  const __nv_bfloat16* xr = x + static_cast<long>(row) * n;
  float mean = 0.f;
  if (!RMS) {
    float s = 0.f;
    for (int c = lane * 8; c < n; c += 256) {
      const uint4 u = *reinterpret_cast<const uint4*>(xr + c);
      const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&u);
#pragma unroll
      for (int j = 0; j < 8; ++j) s += __bfloat162float(hv[j]);
    }
    mean = warp_sum(s) / n;
  }
  float v = 0.f;
  for (int c = lane * 8; c < n; c += 256) {
    const uint4 u = *reinterpret_cast<const uint4*>(xr + c);
    const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&u);
#pragma unroll
    for (int j = 0; j < 8; ++j) { const float d = __bfloat162float(hv[j]) - mean; v += d * d; }
  }
  const float rstd = rsqrtf(warp_sum(v) / n + eps);
  __nv_bfloat16* yr = y + static_cast<long>(row) * n;
  for (int c = lane * 8; c < n; c += 256) {
    const uint4 u = *reinterpret_cast<const uint4*>(xr + c);
    const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&u);
    uint4 o;
    __nv_bfloat16* ho = reinterpret_cast<__nv_bfloat16*>(&o);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      float t = (__bfloat162float(hv[j]) - mean) * rstd * g[c + j];
      if (!RMS) t += b[c + j];
      ho[j] = __float2bfloat16_rn(t);
    }
    *reinterpret_cast<uint4*>(yr + c) = o;
  }
  if (lane == 0) { stats[2 * row] = mean; stats[2 * row + 1] = rstd; }
}

__global__ void norm_bwd_dx_v8_k(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                                 const __nv_bfloat16* dres, __nv_bfloat16* dx, int rows, int n, int rms) {
  const int row = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (row >= rows) return;
  const long o = static_cast<long>(row) * n;
  const float mean = stats[2 * row], rstd = stats[2 * row + 1];
  float sg = 0.f, sgx = 0.f;
  for (int c = lane * 8; c < n; c += 256) {
    const uint4 ud = *reinterpret_cast<const uint4*>(dy + o + c);
    const uint4 ux = *reinterpret_cast<const uint4*>(x + o + c);
    const __nv_bfloat16* hd = reinterpret_cast<const __nv_bfloat16*>(&ud);
    const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&ux);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float gp = __bfloat162float(hd[j]) * g[c + j];
      sg += gp;
      sgx += gp * (__bfloat162float(hx[j]) - mean) * rstd;
    }
  }
  sg = rms ? 0.f : warp_sum(sg) / n;
  sgx = warp_sum(sgx) / n;
  for (int c = lane * 8; c < n; c += 256) {
    const uint4 ud = *reinterpret_cast<const uint4*>(dy + o + c);
    const uint4 ux = *reinterpret_cast<const uint4*>(x + o + c);
    const __nv_bfloat16* hd = reinterpret_cast<const __nv_bfloat16*>(&ud);
    const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&ux);
    uint4 ur = make_uint4(0, 0, 0, 0);
    if (dres) ur = *reinterpret_cast<const uint4*>(dres + o + c);
    const __nv_bfloat16* hr = reinterpret_cast<const __nv_bfloat16*>(&ur);
    uint4 uo;
    __nv_bfloat16* ho = reinterpret_cast<__nv_bfloat16*>(&uo);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float gp = __bfloat162float(hd[j]) * g[c + j];
      const float xh = (__bfloat162float(hx[j]) - mean) * rstd;
      float d = (gp - sg - xh * sgx) * rstd;
      if (dres) d += __bfloat162float(hr[j]);
      ho[j] = __float2bfloat16_rn(d);
    }
    *reinterpret_cast<uint4*>(dx + o + c) = uo;
  }
}

template <class T>
__global__ void norm_bwd_dx_k(const T* dy, const T* x, const float* stats, const float* g, const T* dres, T* dx,
                              int rows, int n, int rms) {
  const int row = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (row >= rows) return;
  const long o = static_cast<long>(row) * n;
  const float mean = stats[2 * row], rstd = stats[2 * row + 1];
  float sg = 0.f, sgx = 0.f;
  for (int c = lane; c < n; c += 32) {
    const float gp = ldf(dy + o + c) * g[c];
    const float xh = (ldf(x + o + c) - mean) * rstd;
    sg += gp;
    sgx += gp * xh;
  }
  sg = warp_sum(sg) / n;
  sgx = warp_sum(sgx) / n;
  if (rms) sg = 0.f;
  for (int c = lane; c < n; c += 32) {
    const float gp = ldf(dy + o + c) * g[c];
    const float xh = (ldf(x + o + c) - mean) * rstd;
    float d = (gp - sg - xh * sgx) * rstd;
    if (dres) d += ldf(dres + o + c);
    stf(dx + o + c, d);
  }
}

// bf16 norm backward with the fp32 residual-gradient stream (any n; the row-pipelined kernel's
// fallback): dx = norm'(dy) + (dres32 | dres) written as bf16 and, if dx32, as fp32.
__global__ void norm_bwd_mixed_k(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                                 const __nv_bfloat16* dres, const float* dres32, __nv_bfloat16* dx, float* dx32,
                                 int rows, int n, int rms) {
  const int row = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (row >= rows) return;
  const long o = static_cast<long>(row) * n;
  const float mean = stats[2 * row], rstd = stats[2 * row + 1];
  float sg = 0.f, sgx = 0.f;
  for (int c = lane; c < n; c += 32) {
    const float gp = __bfloat162float(dy[o + c]) * g[c];
    const float xh = (__bfloat162float(x[o + c]) - mean) * rstd;
    sg += gp;
    sgx += gp * xh;
  }
  sg = warp_sum(sg) / n;
  sgx = warp_sum(sgx) / n;
  if (rms) sg = 0.f;
  for (int c = lane; c < n; c += 32) {
    const float gp = __bfloat162float(dy[o + c]) * g[c];
    const float xh = (__bfloat162float(x[o + c]) - mean) * rstd;
    float d = (gp - sg - xh * sgx) * rstd;
    if (dres32) d += dres32[o + c];
    else if (dres) d += __bfloat162float(dres[o + c]);
    dx[o + c] = __float2bfloat16_rn(d);
    if (dx32) dx32[o + c] = d;
  }
}

template <class T>
__global__ void colsum_partial_k(const T* a, const T* x, const float* stats, int rows, int n, int lda, int mode,
                                 float* partial, int nblk) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  const int blk = blockIdx.y;
  const int r0 = static_cast<int>(static_cast<long>(rows) * blk / nblk);
  const int r1 = static_cast<int>(static_cast<long>(rows) * (blk + 1) / nblk);
  float s0 = 0.f, s1 = 0.f;
  for (int r = r0; r < r1; ++r) {
    const float dy = ldf(a + static_cast<long>(r) * lda + c);
    if (mode == 0) { s0 += dy; continue; }
    const float xh = (ldf(x + static_cast<long>(r) * n + c) - stats[2 * r]) * stats[2 * r + 1];
    s0 += dy * xh;
    s1 += dy;
  }
  partial[static_cast<long>(blk) * n + c] = s0;
  if (mode == 1) partial[static_cast<long>(nblk + blk) * n + c] = s1;
}

// bf16, n % 8 == 0: each thread owns 8 consecutive columns (16-byte loads).
__global__ void colsum_partial_v8_k(const __nv_bfloat16* a, const __nv_bfloat16* x, const float* stats, int rows,
                                    int n, int lda, int mode, float* partial, int nblk) {
  const int c8 = (blockIdx.x * blockDim.x + threadIdx.x) * 8;
  if (c8 >= n) return;
  const int blk = blockIdx.y;
  const int r0 = static_cast<int>(static_cast<long>(rows) * blk / nblk);
  const int r1 = static_cast<int>(static_cast<long>(rows) * (blk + 1) / nblk);
  float s0[8] = {0, 0, 0, 0, 0, 0, 0, 0}, s1[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  for (int r = r0; r < r1; ++r) {
    const uint4 ua = *reinterpret_cast<const uint4*>(a + static_cast<long>(r) * lda + c8);
    const __nv_bfloat16* ha = reinterpret_cast<const __nv_bfloat16*>(&ua);
    if (mode == 0) {
#pragma unroll
      for (int j = 0; j < 8; ++j) s0[j] += __bfloat162float(ha[j]);
      continue;
    }
    const uint4 ux = *reinterpret_cast<const uint4*>(x + static_cast<long>(r) * n + c8);
    const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&ux);
    const float mu = stats[2 * r], rs = stats[2 * r + 1];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float dy = __bfloat162float(ha[j]);
      s0[j] += dy * ((__bfloat162float(hx[j]) - mu) * rs);
      s1[j] += dy;
    }
  }
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    partial[static_cast<long>(blk) * n + c8 + j] = s0[j];
    if (mode == 1) partial[static_cast<long>(nblk + blk) * n + c8 + j] = s1[j];
  }
}

__global__ void __launch_bounds__(256) colsum_partial_v2_k(const __nv_bfloat16* a, const __nv_bfloat16* x,
                                                           const float* stats, int rows, int n, int lda, int mode,
                                                           float* partial, int nblk) {
  __shared__ float red[2][8][256 + 8];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int c8 = blockIdx.x * 256 + lane * 8;
  const int blk = blockIdx.y;
  const int r0 = static_cast<int>(static_cast<long>(rows) * blk / nblk);
  const int r1 = static_cast<int>(static_cast<long>(rows) * (blk + 1) / nblk);
  float s0[8] = {0, 0, 0, 0, 0, 0, 0, 0}, s1[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  if (c8 < n && mode == 0) {
    // plain column sums (a bias gradient): 8 rows' 16-byte loads in flight per warp, added in row
    // order (the one-load-per-iteration loop was latency-bound at ~2 TB/s on the 100 MB dQKV)
    int r = r0 + warp;
    for (; r + 56 < r1; r += 64) {
      uint4 u[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) u[k] = __ldg(reinterpret_cast<const uint4*>(a + static_cast<long>(r + 8 * k) * lda + c8));
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const __nv_bfloat16* ha = reinterpret_cast<const __nv_bfloat16*>(&u[k]);
#pragma unroll
        for (int j = 0; j < 8; ++j) s0[j] += __bfloat162float(ha[j]);
      }
    }
    for (; r < r1; r += 8) {
      const uint4 ua = *reinterpret_cast<const uint4*>(a + static_cast<long>(r) * lda + c8);
      const __nv_bfloat16* ha = reinterpret_cast<const __nv_bfloat16*>(&ua);
#pragma unroll
      for (int j = 0; j < 8; ++j) s0[j] += __bfloat162float(ha[j]);
    }
  } else if (c8 < n) {
    for (int r = r0 + warp; r < r1; r += 8) {
      const uint4 ua = *reinterpret_cast<const uint4*>(a + static_cast<long>(r) * lda + c8);
      const __nv_bfloat16* ha = reinterpret_cast<const __nv_bfloat16*>(&ua);
      const uint4 ux = *reinterpret_cast<const uint4*>(x + static_cast<long>(r) * n + c8);
      const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&ux);
      const float mu = stats[2 * r], rs = stats[2 * r + 1];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const float dy = __bfloat162float(ha[j]);
        s0[j] += dy * ((__bfloat162float(hx[j]) - mu) * rs);
        s1[j] += dy;
      }
    }
  }
#pragma unroll
  for (int j = 0; j < 8; ++j) { red[0][warp][lane * 8 + j] = s0[j]; red[1][warp][lane * 8 + j] = s1[j]; }
  __syncthreads();
  const int c = threadIdx.x;                // one column of the 256 per thread
  const int col = blockIdx.x * 256 + c;
  if (col < n) {
    float t0 = 0.f, t1 = 0.f;
#pragma unroll
    for (int w = 0; w < 8; ++w) { t0 += red[0][w][c]; t1 += red[1][w][c]; }
    partial[static_cast<long>(blk) * n + col] = t0;
    if (mode == 1) partial[static_cast<long>(nblk + blk) * n + col] = t1;
  }
}

// out_k[c] += sum_b partial[k * nblk + b][c] for k = blockIdx.y (a null out_k: nothing). Block =
// 32 columns x 16 warps: warp w sums row blocks w, w + 16, ... with 4 loads in flight, then the
// 16 warp sums are added in fixed order (deterministic). The grid spans n / 32 x arrays CTAs, so a
// [256][8192] partial (fc1.b) is read by 256 CTAs instead of 32 threads-per-column chains.
__global__ void __launch_bounds__(512) colsum_reduce_k(const float* __restrict__ partial, int nblk, int n,
                                                       float* out0, float* out1, float* out2) {
  __shared__ float red[16][33];
  const int k = blockIdx.y;
  float* o = k == 0 ? out0 : (k == 1 ? out1 : out2);
  if (!o) return;   // uniform over the block
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int c = blockIdx.x * 32 + lane;
  // 8 independent loads in flight per thread (the partials are L2-resident; with 4 the reduction of a
  // norm backward's 444 x n x 3 partials was latency-bound at ~1.6 TB/s)
  float a[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  if (c < n) {
    const float* p = partial + static_cast<long>(k) * nblk * n + c;
    int b = w;
    for (; b + 112 < nblk; b += 128) {
      float v[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) v[j] = p[static_cast<long>(b + 16 * j) * n];
#pragma unroll
      for (int j = 0; j < 8; ++j) a[j] += v[j];
    }
    for (int j = 0; b < nblk; b += 16, j = (j + 1) & 7) a[j] += p[static_cast<long>(b) * n];
  }
  red[w][lane] = ((a[0] + a[1]) + (a[2] + a[3])) + ((a[4] + a[5]) + (a[6] + a[7]));
  __syncthreads();
  if (w == 0 && c < n) {
    float t = 0.f;
#pragma unroll
    for (int i = 0; i < 16; ++i) t += red[i][lane];
    o[c] += t;
  }
}

// Block-per-row-tile norm backward (bf16, n = 8 * VPT * nthreads, nthreads % 32 == 0). Thread t owns
// the 16-byte chunks t, t + nthreads, ... of every row (coalesced), R rows are in flight per
// iteration, row sums are reduced warp -> shared memory -> block, and each thread keeps its
// columns' gradient sums in registers across the CTA's contiguous row range. One wave of CTAs.
// (A forward of the same shape measured no faster than the warp-per-row kernels: not used.)
__device__ __forceinline__ void load_g8(const float* g, int c, float (&o)[8]) {
  const float4 a = *reinterpret_cast<const float4*>(g + c), b = *reinterpret_cast<const float4*>(g + c + 4);
  o[0] = a.x; o[1] = a.y; o[2] = a.z; o[3] = a.w; o[4] = b.x; o[5] = b.y; o[6] = b.z; o[7] = b.w;
}

// dx = norm'(dy) (+ dres), and, fused, the column partial sums of this CTA's contiguous row range:
// partial[0][blk] = sum dy * xhat (d gamma), partial[1][blk] = sum dy (d beta, LN only),
// partial[2][blk] = sum dx (the stored, rounded output: the bias gradient of the linear layer that
// produced the residual, when sum_out).
template <int VPT, int R>
__global__ void __launch_bounds__(VPT == 1 ? 512 : 384) norm_bwd_tile_k(const __nv_bfloat16* dy, const __nv_bfloat16* x,
                                                       const float* stats, const float* g,
                                                       const __nv_bfloat16* dres, __nv_bfloat16* dx, int rows, int n,
                                                       int rms, float* partial, int nblk, int sum_out) {
  __shared__ float red[2][2][R][32];
  const int nt = blockDim.x, t = threadIdx.x, w = t / 32, lane = t % 32, nw = nt / 32;
  const int blk = blockIdx.x;
  const int rb = static_cast<int>(static_cast<long>(rows) * blk / nblk);
  const int re = static_cast<int>(static_cast<long>(rows) * (blk + 1) / nblk);
  float gg[VPT][8], ag[VPT][8], ab[VPT][8], ao[VPT][8];
#pragma unroll
  for (int v = 0; v < VPT; ++v) {
    load_g8(g, (t + v * nt) * 8, gg[v]);
#pragma unroll
    for (int j = 0; j < 8; ++j) { ag[v][j] = 0.f; ab[v][j] = 0.f; ao[v][j] = 0.f; }
  }
  int it = 0;
  for (int r0 = rb; r0 < re; r0 += R, ++it) {
    uint4 ud[R][VPT], ux[R][VPT];
    float mean[R], rstd[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const bool ok = r0 + r < re;
      mean[r] = ok ? stats[2 * (r0 + r)] : 0.f;
      rstd[r] = ok ? stats[2 * (r0 + r) + 1] : 0.f;
#pragma unroll
      for (int v = 0; v < VPT; ++v) {
        const long o = static_cast<long>(r0 + r) * n + (t + v * nt) * 8;
        ud[r][v] = ok ? *reinterpret_cast<const uint4*>(dy + o) : make_uint4(0, 0, 0, 0);
        ux[r][v] = ok ? *reinterpret_cast<const uint4*>(x + o) : make_uint4(0, 0, 0, 0);
      }
    }
    const int pb = it & 1;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      float sg = 0.f, sgx = 0.f;
#pragma unroll
      for (int v = 0; v < VPT; ++v) {
        const __nv_bfloat16* hd = reinterpret_cast<const __nv_bfloat16*>(&ud[r][v]);
        const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&ux[r][v]);
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const float d = __bfloat162float(hd[j]);
          const float xh = (__bfloat162float(hx[j]) - mean[r]) * rstd[r];
          const float gp = d * gg[v][j];
          sg += gp;
          sgx += gp * xh;
          ag[v][j] += d * xh;
          ab[v][j] += d;
        }
      }
      sg = warp_sum(sg);
      sgx = warp_sum(sgx);
      if (lane == 0) { red[pb][0][r][w] = sg; red[pb][1][r][w] = sgx; }
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (r0 + r >= re) break;
      float sg = 0.f, sgx = 0.f;
      for (int i = 0; i < nw; ++i) { sg += red[pb][0][r][i]; sgx += red[pb][1][r][i]; }
      sg = rms ? 0.f : sg / n;
      sgx /= n;
#pragma unroll
      for (int v = 0; v < VPT; ++v) {
        const long o = static_cast<long>(r0 + r) * n + (t + v * nt) * 8;
        uint4 ur = make_uint4(0, 0, 0, 0);
        if (dres) ur = *reinterpret_cast<const uint4*>(dres + o);
        const __nv_bfloat16* hd = reinterpret_cast<const __nv_bfloat16*>(&ud[r][v]);
        const __nv_bfloat16* hx = reinterpret_cast<const __nv_bfloat16*>(&ux[r][v]);
        const __nv_bfloat16* hr = reinterpret_cast<const __nv_bfloat16*>(&ur);
        uint4 uo;
        __nv_bfloat16* ho = reinterpret_cast<__nv_bfloat16*>(&uo);
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const float xh = (__bfloat162float(hx[j]) - mean[r]) * rstd[r];
          float d = (__bfloat162float(hd[j]) * gg[v][j] - sg - xh * sgx) * rstd[r];
          if (dres) d += __bfloat162float(hr[j]);
          ho[j] = __float2bfloat16_rn(d);
          ao[v][j] += __bfloat162float(ho[j]);
        }
        *reinterpret_cast<uint4*>(dx + o) = uo;
      }
    }
  }
  if (!partial) return;
#pragma unroll
  for (int v = 0; v < VPT; ++v) {
    const int c = (t + v * nt) * 8;
    float* p0 = partial + static_cast<long>(blk) * n + c;
    float* p1 = partial + static_cast<long>(nblk + blk) * n + c;
    float* p2 = partial + static_cast<long>(2 * nblk + blk) * n + c;
    *reinterpret_cast<float4*>(p0) = make_float4(ag[v][0], ag[v][1], ag[v][2], ag[v][3]);
    *reinterpret_cast<float4*>(p0 + 4) = make_float4(ag[v][4], ag[v][5], ag[v][6], ag[v][7]);
    if (!rms) {
      *reinterpret_cast<float4*>(p1) = make_float4(ab[v][0], ab[v][1], ab[v][2], ab[v][3]);
      *reinterpret_cast<float4*>(p1 + 4) = make_float4(ab[v][4], ab[v][5], ab[v][6], ab[v][7]);
    }
    if (sum_out) {
      *reinterpret_cast<float4*>(p2) = make_float4(ao[v][0], ao[v][1], ao[v][2], ao[v][3]);
      *reinterpret_cast<float4*>(p2 + 4) = make_float4(ao[v][4], ao[v][5], ao[v][6], ao[v][7]);
    }
  }
}

// out_k[c] += sum_b partial[k][b][c] for the non-null outputs. Block = 32 columns x 8 warps: warp w
// sums blocks w, w + 8, ... (coalesced 128-byte rows), then the 8 warp sums are added in fixed
// order (deterministic).
__global__ void __launch_bounds__(256) colsum_final3_k(const float* partial, int nblk, int n, float* out0, float* out1,
                                                       float* out2) {
  __shared__ float red[3][8][33];
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int c = blockIdx.x * 32 + lane;
  float s0 = 0.f, s1 = 0.f, s2 = 0.f;
  if (c < n) {
    for (int b = w; b < nblk; b += 8) {
      s0 += partial[static_cast<long>(b) * n + c];
      if (out1) s1 += partial[static_cast<long>(nblk + b) * n + c];
      if (out2) s2 += partial[static_cast<long>(2 * nblk + b) * n + c];
    }
  }
  red[0][w][lane] = s0; red[1][w][lane] = s1; red[2][w][lane] = s2;
  __syncthreads();
  if (w < 3 && c < n) {
    float t = 0.f;
#pragma unroll
    for (int i = 0; i < 8; ++i) t += red[w][i][lane];
    float* o = w == 0 ? out0 : (w == 1 ? out1 : out2);
    if (o) o[c] += t;
  }
}

// VPT (16-byte chunks per thread) for the tile kernels, 0 when the width does not tile
inline int tile_vpt(int n) {
  if (n % 8) return 0;
  const int ch = n / 8;
  for (int v = 1; v <= 4; v *= 2)
    if (ch % v == 0 && (ch / v) % 32 == 0 && ch / v <= (v == 1 ? 512 : 384)) return v;
  return 0;
}

// the device's full SM count, NOT the launching thread's budget: the row partition of the column
// reductions below follows it, so their fp32 partial sums (and the bits of the bias / gain
// gradients) do not depend on the SM partition a stage runs on (emulated pipeline, set_sm_budget)
int device_sms() { return device_sm_count_full(); }

template <class K>
int resident_grid(K kernel, int threads) {
  int occ = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, 0);
  return device_sms() * (occ < 1 ? 1 : occ);
}

// returns false when the shape does not tile (caller falls back to the row kernels)
bool norm_bwd_tile(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                   const __nv_bfloat16* dres, __nv_bfloat16* dx, int rows, int n, int rms, float* dg, float* db,
                   float* dsum, float* partial, size_t partial_floats, cudaStream_t st) {
  const int vpt = tile_vpt(n);
  if (!vpt || vpt > 2) return false;
  const int nt = n / 8 / vpt;
  const int R = vpt == 1 ? 4 : 2;
  int nblk = vpt == 1 ? resident_grid(norm_bwd_tile_k<1, 4>, nt) : resident_grid(norm_bwd_tile_k<2, 2>, nt);
  if (dg) {
    const long cap = static_cast<long>(partial_floats / (3 * static_cast<size_t>(n)));
    if (cap < 1) return false;
    nblk = nblk < cap ? nblk : static_cast<int>(cap);
  }
  const int need = cdiv(rows, R);
  nblk = nblk < need ? nblk : need;
  if (nblk < 1) return true;
  float* part = dg ? partial : nullptr;
  const int so = dsum ? 1 : 0;
  if (vpt == 1) norm_bwd_tile_k<1, 4><<<nblk, nt, 0, st>>>(dy, x, stats, g, dres, dx, rows, n, rms, part, nblk, so);
  else norm_bwd_tile_k<2, 2><<<nblk, nt, 0, st>>>(dy, x, stats, g, dres, dx, rows, n, rms, part, nblk, so);
  note_launch();
  if (dg) {
    colsum_final3_k<<<cdiv(n, 32), 256, 0, st>>>(partial, nblk, n, dg, rms ? nullptr : db, dsum);
    note_launch();
  }
  return true;
}

// ------------------------------------------------------------------ attention
// One warp per (query row, head); keys in chunks of 32 (one per lane); online softmax.
template <class T>
__global__ void attn_fwd_k(const T* qkv, T* O, float* lse, int B, int s, int nh, int dh) {
  __shared__ float qs[8][128];
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const long gw = static_cast<long>(blockIdx.x) * 8 + w;
  const long Ttok = static_cast<long>(B) * s;
  if (gw >= Ttok * nh) return;
  const int head = static_cast<int>(gw % nh);
  const long r = gw / nh;
  const int t = static_cast<int>(r % s);
  const long base = r - t;  // first row of this sample
  const int h = nh * dh, ld = 3 * h;
  const float scale = rsqrtf(static_cast<float>(dh));
  for (int d = lane; d < dh; d += 32) qs[w][d] = ldf(qkv + r * ld + head * dh + d);
  __syncwarp();
  float m = -INFINITY, l = 0.f, o[4] = {0.f, 0.f, 0.f, 0.f};
  for (int c0 = 0; c0 <= t; c0 += 32) {
    const int u = c0 + lane;
    float sc = -INFINITY;
    if (u <= t) {
      const T* kr = qkv + (base + u) * ld + h + head * dh;
      float acc = 0.f;
      for (int d = 0; d < dh; ++d) acc += qs[w][d] * ldf(kr + d);
      sc = acc * scale;
    }
    const float mn = fmaxf(m, warp_max(sc));
    const float corr = __expf(m - mn);
    const float p = (u <= t) ? __expf(sc - mn) : 0.f;
    l = l * corr + warp_sum(p);
#pragma unroll
    for (int i = 0; i < 4; ++i) o[i] *= corr;
    const int nv = min(32, t - c0 + 1);
    for (int j = 0; j < nv; ++j) {
      const float pj = __shfl_sync(0xffffffffu, p, j);
      const T* vr = qkv + (base + c0 + j) * ld + 2 * h + head * dh;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int d = lane + 32 * i;
        if (d < dh) o[i] += pj * ldf(vr + d);
      }
    }
    m = mn;
  }
  const float inv = 1.f / l;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int d = lane + 32 * i;
    if (d < dh) stf(O + r * h + head * dh + d, o[i] * inv);
  }
  if (lane == 0) lse[static_cast<long>(head) * Ttok + r] = m + logf(l);
}

template <class T>
__global__ void attn_bwd_dq_k(const T* qkv, const T* O, const T* dO, const float* lse, T* dqkv, float* Dsc, int B,
                              int s, int nh, int dh) {
  __shared__ float qs[8][128], gs[8][128];
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const long gw = static_cast<long>(blockIdx.x) * 8 + w;
  const long Ttok = static_cast<long>(B) * s;
  if (gw >= Ttok * nh) return;
  const int head = static_cast<int>(gw % nh);
  const long r = gw / nh;
  const int t = static_cast<int>(r % s);
  const long base = r - t;
  const int h = nh * dh, ld = 3 * h;
  const float scale = rsqrtf(static_cast<float>(dh));
  float Dp = 0.f;
  for (int d = lane; d < dh; d += 32) {
    qs[w][d] = ldf(qkv + r * ld + head * dh + d);
    const float g = ldf(dO + r * h + head * dh + d);
    gs[w][d] = g;
    Dp += g * ldf(O + r * h + head * dh + d);
  }
  const float D = warp_sum(Dp);
  __syncwarp();
  const float L = lse[static_cast<long>(head) * Ttok + r];
  float dq[4] = {0.f, 0.f, 0.f, 0.f};
  for (int c0 = 0; c0 <= t; c0 += 32) {
    const int u = c0 + lane;
    float ds = 0.f;
    if (u <= t) {
      const T* kr = qkv + (base + u) * ld + h + head * dh;
      const T* vr = qkv + (base + u) * ld + 2 * h + head * dh;
      float sc = 0.f, dp = 0.f;
      for (int d = 0; d < dh; ++d) { sc += qs[w][d] * ldf(kr + d); dp += gs[w][d] * ldf(vr + d); }
      const float p = __expf(sc * scale - L);
      ds = p * (dp - D);
    }
    const int nv = min(32, t - c0 + 1);
    for (int j = 0; j < nv; ++j) {
      const float dsj = __shfl_sync(0xffffffffu, ds, j);
      const T* kr = qkv + (base + c0 + j) * ld + h + head * dh;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int d = lane + 32 * i;
        if (d < dh) dq[i] += dsj * ldf(kr + d);
      }
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int d = lane + 32 * i;
    if (d < dh) stf(dqkv + r * ld + head * dh + d, dq[i] * scale);
  }
  if (lane == 0) Dsc[static_cast<long>(head) * Ttok + r] = D;
}

template <class T>
__global__ void attn_bwd_dkdv_k(const T* qkv, const T* dO, const float* lse, const float* Dsc, T* dqkv, int B, int s,
                                int nh, int dh) {
  __shared__ float ks[8][128], vs[8][128];
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const long gw = static_cast<long>(blockIdx.x) * 8 + w;
  const long Ttok = static_cast<long>(B) * s;
  if (gw >= Ttok * nh) return;
  const int head = static_cast<int>(gw % nh);
  const long r = gw / nh;  // key row
  const int u = static_cast<int>(r % s);
  const long base = r - u;
  const int h = nh * dh, ld = 3 * h;
  const float scale = rsqrtf(static_cast<float>(dh));
  for (int d = lane; d < dh; d += 32) {
    ks[w][d] = ldf(qkv + r * ld + h + head * dh + d);
    vs[w][d] = ldf(qkv + r * ld + 2 * h + head * dh + d);
  }
  __syncwarp();
  float dk[4] = {0.f, 0.f, 0.f, 0.f}, dv[4] = {0.f, 0.f, 0.f, 0.f};
  for (int c0 = u; c0 < s; c0 += 32) {
    const int t = c0 + lane;
    float p = 0.f, ds = 0.f;
    if (t < s) {
      const long rt = base + t;
      const T* qr = qkv + rt * ld + head * dh;
      const T* gr = dO + rt * h + head * dh;
      float sc = 0.f, dp = 0.f;
      for (int d = 0; d < dh; ++d) { sc += ldf(qr + d) * ks[w][d]; dp += ldf(gr + d) * vs[w][d]; }
      p = __expf(sc * scale - lse[static_cast<long>(head) * Ttok + rt]);
      ds = p * (dp - Dsc[static_cast<long>(head) * Ttok + rt]);
    }
    const int nv = min(32, s - c0);
    for (int j = 0; j < nv; ++j) {
      const float pj = __shfl_sync(0xffffffffu, p, j);
      const float dsj = __shfl_sync(0xffffffffu, ds, j);
      const long rt = base + c0 + j;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int d = lane + 32 * i;
        if (d < dh) {
          dv[i] += pj * ldf(dO + rt * h + head * dh + d);
          dk[i] += dsj * ldf(qkv + rt * ld + head * dh + d);
        }
      }
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int d = lane + 32 * i;
    if (d < dh) {
      stf(dqkv + r * ld + h + head * dh + d, dk[i] * scale);
      stf(dqkv + r * ld + 2 * h + head * dh + d, dv[i]);
    }
  }
}

// ----------------------------------------------------------------------- RoPE
template <class T>
__global__ void rope_k(T* qkv, int B, int s, int nh, int dh, float base, int inverse) {
  const int half = dh / 2;
  const long n = static_cast<long>(B) * s * nh * half;
  const int h = nh * dh;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < n; i += static_cast<long>(gridDim.x) * blockDim.x) {
    const int j = static_cast<int>(i % half);
    const long rh = i / half;
    const int head = static_cast<int>(rh % nh);
    const long r = rh / nh;
    const int t = static_cast<int>(r % s);
    const double theta = pow(static_cast<double>(base), -2.0 * j / dh);
    double sn, cs;
    sincos(t * theta, &sn, &cs);
    const float c = static_cast<float>(cs), sgn = inverse ? -1.f : 1.f;
    const float si = sgn * static_cast<float>(sn);
    for (int part = 0; part < 2; ++part) {  // q, then k
      T* p = qkv + r * 3 * h + part * h + head * dh;
      const float x1 = ldf(p + j), x2 = ldf(p + j + half);
      stf(p + j, x1 * c - x2 * si);
      stf(p + j + half, x1 * si + x2 * c);
    }
  }
}

// RoPE angle table (c, s)[t][j] = (cos, sin)(t * base^(-2j/dh)), the angles in double precision and
// rounded to fp32 exactly as rope_k computes them per element (so the two paths agree bitwise).
__global__ void rope_table_k(float2* tab, int s, int dh, float base) {
  const int half = dh / 2;
  const long n = static_cast<long>(s) * half;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < n; i += static_cast<long>(gridDim.x) * blockDim.x) {
    const int j = static_cast<int>(i % half), t = static_cast<int>(i / half);
    const double theta = pow(static_cast<double>(base), -2.0 * j / dh);
    double sn, cs;
    sincos(t * theta, &sn, &cs);
    tab[i] = make_float2(static_cast<float>(cs), static_cast<float>(sn));
  }
}
// bf16 RoPE from the table: one CTA per token row (blockIdx.y), thread = (head, 8 consecutive j):
// q and k halves as 16-byte vectors, no per-element division or double-precision math.
__global__ void rope_v8_k(__nv_bfloat16* qkv, const float2* __restrict__ tab, int s, int nh, int dh, int inverse) {
  const int half = dh / 2, h8 = half / 8;
  const int tid = blockIdx.x * blockDim.x + threadIdx.x;
  if (tid >= nh * h8) return;
  const int head = tid / h8, j0 = (tid - head * h8) * 8;
  const long r = blockIdx.y;
  const int t = static_cast<int>(r % s);
  const int h = nh * dh;
  const float sgn = inverse ? -1.f : 1.f;
  float c[8], sn[8];
  const float4* tp = reinterpret_cast<const float4*>(tab + static_cast<long>(t) * half + j0);
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    const float4 v = tp[e];
    c[2 * e] = v.x; sn[2 * e] = sgn * v.y; c[2 * e + 1] = v.z; sn[2 * e + 1] = sgn * v.w;
  }
#pragma unroll
  for (int part = 0; part < 2; ++part) {   // q, then k
    __nv_bfloat16* p = qkv + r * 3 * h + part * h + head * dh;
    uint4 u1 = *reinterpret_cast<const uint4*>(p + j0), u2 = *reinterpret_cast<const uint4*>(p + j0 + half);
    const __nv_bfloat16* x1 = reinterpret_cast<const __nv_bfloat16*>(&u1);
    const __nv_bfloat16* x2 = reinterpret_cast<const __nv_bfloat16*>(&u2);
    uint4 o1, o2;
    __nv_bfloat16* y1 = reinterpret_cast<__nv_bfloat16*>(&o1);
    __nv_bfloat16* y2 = reinterpret_cast<__nv_bfloat16*>(&o2);
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      const float a = __bfloat162float(x1[e]), b = __bfloat162float(x2[e]);
      y1[e] = __float2bfloat16_rn(a * c[e] - b * sn[e]);
      y2[e] = __float2bfloat16_rn(a * sn[e] + b * c[e]);
    }
    *reinterpret_cast<uint4*>(p + j0) = o1;
    *reinterpret_cast<uint4*>(p + j0 + half) = o2;
  }
}

// --------------------------------------------------------------------- SwiGLU
template <class T>
__global__ void swiglu_fwd_k(const T* GU, T* M, int rows, int f) {
  const long n = static_cast<long>(rows) * f;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < n; i += static_cast<long>(gridDim.x) * blockDim.x) {
    const long r = i / f;
    const int j = static_cast<int>(i % f);
    const float g = ldf(GU + r * 2 * f + j), u = ldf(GU + r * 2 * f + f + j);
    stf(M + i, g / (1.f + __expf(-g)) * u);
  }
}
template <class T>
__global__ void swiglu_bwd_k(const T* GU, const T* dM, T* dGU, int rows, int f) {
  const long n = static_cast<long>(rows) * f;
  for (long i = blockIdx.x * static_cast<long>(blockDim.x) + threadIdx.x; i < n; i += static_cast<long>(gridDim.x) * blockDim.x) {
    const long r = i / f;
    const int j = static_cast<int>(i % f);
    const float g = ldf(GU + r * 2 * f + j), u = ldf(GU + r * 2 * f + f + j), dm = ldf(dM + i);
    const float sg = 1.f / (1.f + __expf(-g));
    stf(dGU + r * 2 * f + j, dm * u * sg * (1.f + g * (1.f - sg)));
    stf(dGU + r * 2 * f + f + j, dm * g * sg);
  }
}

template <class T>
__global__ void gelu_fwd_k(const T* Z, T* G, size_t n) {
  const float c = 0.7978845608028654f;
  for (size_t i = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; i < n; i += static_cast<size_t>(gridDim.x) * blockDim.x) {
    const float z = ldf(Z + i);
    float t;
    if constexpr (std::is_same<T, __nv_bfloat16>::value) asm("tanh.approx.f32 %0, %1;" : "=f"(t) : "f"(c * (z + 0.044715f * z * z * z)));
    else t = tanhf(c * (z + 0.044715f * z * z * z));
    stf(G + i, 0.5f * z * (1.f + t));
  }
}

// bf16, 16-byte vectors (8 elements per thread-iteration); widths % 8 == 0
__device__ __forceinline__ float tanh_fast(float x) {
  float t;
  asm("tanh.approx.f32 %0, %1;" : "=f"(t) : "f"(x));
  return t;
}
__global__ void gelu_fwd_v8_k(const uint4* Z, uint4* G, size_t n8) {
  const float c = 0.7978845608028654f;
  for (size_t i = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; i < n8; i += static_cast<size_t>(gridDim.x) * blockDim.x) {
    const uint4 u = Z[i];
    const __nv_bfloat16* hz = reinterpret_cast<const __nv_bfloat16*>(&u);
    uint4 o;
    __nv_bfloat16* ho = reinterpret_cast<__nv_bfloat16*>(&o);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float z = __bfloat162float(hz[j]);
      ho[j] = __float2bfloat16_rn(0.5f * z * (1.f + tanh_fast(c * (z + 0.044715f * z * z * z))));
    }
    G[i] = o;
  }
}
// GU row = [gate (f) | up (f)]; M = silu(gate) * up
// 2-D grid (x: 16-byte column vectors, y: rows): no per-vector row division
__global__ void swiglu_fwd_v8_k(const __nv_bfloat16* GU, __nv_bfloat16* M, int rows, int f) {
  const int f8 = f / 8;
  {
    const long r = blockIdx.y;
    const int jv = blockIdx.x * blockDim.x + threadIdx.x;
    if (jv >= f8 || r >= rows) return;
    const long i = r * f8 + jv;
    const int j8 = jv * 8;
    const uint4 ug = *reinterpret_cast<const uint4*>(GU + r * 2 * f + j8);
    const uint4 uu = *reinterpret_cast<const uint4*>(GU + r * 2 * f + f + j8);
    const __nv_bfloat16* hg = reinterpret_cast<const __nv_bfloat16*>(&ug);
    const __nv_bfloat16* hu = reinterpret_cast<const __nv_bfloat16*>(&uu);
    uint4 o;
    __nv_bfloat16* ho = reinterpret_cast<__nv_bfloat16*>(&o);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float g = __bfloat162float(hg[j]);
      ho[j] = __float2bfloat16_rn(g / (1.f + __expf(-g)) * __bfloat162float(hu[j]));
    }
    *reinterpret_cast<uint4*>(M + i * 8) = o;
  }
}
__global__ void swiglu_bwd_v8_k(const __nv_bfloat16* GU, const __nv_bfloat16* dM, __nv_bfloat16* dGU, int rows, int f) {
  const int f8 = f / 8;
  {
    const long r = blockIdx.y;
    const int jv = blockIdx.x * blockDim.x + threadIdx.x;
    if (jv >= f8 || r >= rows) return;
    const long i = r * f8 + jv;
    const int j8 = jv * 8;
    const uint4 ug = *reinterpret_cast<const uint4*>(GU + r * 2 * f + j8);
    const uint4 uu = *reinterpret_cast<const uint4*>(GU + r * 2 * f + f + j8);
    const uint4 ud = *reinterpret_cast<const uint4*>(dM + i * 8);
    const __nv_bfloat16* hg = reinterpret_cast<const __nv_bfloat16*>(&ug);
    const __nv_bfloat16* hu = reinterpret_cast<const __nv_bfloat16*>(&uu);
    const __nv_bfloat16* hd = reinterpret_cast<const __nv_bfloat16*>(&ud);
    uint4 og, ou;
    __nv_bfloat16* hog = reinterpret_cast<__nv_bfloat16*>(&og);
    __nv_bfloat16* hou = reinterpret_cast<__nv_bfloat16*>(&ou);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float g = __bfloat162float(hg[j]), u = __bfloat162float(hu[j]), dm = __bfloat162float(hd[j]);
      const float sg = 1.f / (1.f + __expf(-g));
      hog[j] = __float2bfloat16_rn(dm * u * sg * (1.f + g * (1.f - sg)));
      hou[j] = __float2bfloat16_rn(dm * g * sg);
    }
    *reinterpret_cast<uint4*>(dGU + r * 2 * f + j8) = og;
    *reinterpret_cast<uint4*>(dGU + r * 2 * f + f + j8) = ou;
  }
}

// ---------------------------------------------------------------- softmax-CE
template <class T>
__global__ void softmax_ce_k(const float* logits, const int32_t* tok, int ld_tok, int s, int V, float inv_ntok,
                             T* dlogits, float* row_loss, long row0) {
  __shared__ float sm[32], sl[32];
  const long r = blockIdx.x;
  const float* z = logits + r * V;
  float m = -INFINITY, l = 0.f;
  for (int c = threadIdx.x; c < V; c += blockDim.x) {
    const float v = z[c];
    if (v > m) { l = l * __expf(m - v) + 1.f; m = v; } else { l += __expf(v - m); }
  }
  // combine (m, l) pairs: warp then block, fixed order
  for (int o = 16; o > 0; o >>= 1) {
    const float m2 = __shfl_xor_sync(0xffffffffu, m, o), l2 = __shfl_xor_sync(0xffffffffu, l, o);
    const float mn = fmaxf(m, m2);
    l = (mn == -INFINITY) ? 0.f : l * __expf(m - mn) + l2 * __expf(m2 - mn);
    m = mn;
  }
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32, nw = blockDim.x / 32;
  if (lane == 0) { sm[w] = m; sl[w] = l; }
  __syncthreads();
  if (threadIdx.x == 0) {
    float M = sm[0], Ls = sl[0];
    for (int i = 1; i < nw; ++i) {
      const float mn = fmaxf(M, sm[i]);
      Ls = Ls * __expf(M - mn) + sl[i] * __expf(sm[i] - mn);
      M = mn;
    }
    sm[0] = M; sl[0] = Ls;
  }
  __syncthreads();
  const float lse = sm[0] + logf(sl[0]);
  const int b = static_cast<int>((row0 + r) / s), t = static_cast<int>((row0 + r) % s);
  const int y = tok[static_cast<long>(b) * ld_tok + t + 1];
  for (int c = threadIdx.x; c < V; c += blockDim.x) {
    const float p = __expf(z[c] - lse);
    stf(dlogits + r * V + c, (p - (c == y ? 1.f : 0.f)) * inv_ntok);
  }
  if (threadIdx.x == 0) row_loss[r] = lse - z[y];
}

__global__ void loss_reduce_k(const float* row_loss, int rows, double* out) {
  __shared__ double sh[1024];
  double acc = 0.0;
  for (int i = threadIdx.x; i < rows; i += blockDim.x) acc += row_loss[i];
  sh[threadIdx.x] = acc;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) out[0] = sh[0];
}

__global__ void cast_k(const float* x, __nv_bfloat16* y, size_t n) {
  for (size_t i = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; i < n; i += static_cast<size_t>(gridDim.x) * blockDim.x)
    y[i] = __float2bfloat16_rn(x[i]);
}
// 8 elements per thread-iteration: two 16-byte loads, one 16-byte store
__global__ void cast_v8_k(const float4* x, uint4* y, size_t n8) {
  for (size_t i = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; i < n8; i += static_cast<size_t>(gridDim.x) * blockDim.x) {
    const float4 a = x[2 * i], b = x[2 * i + 1];
    uint4 u;
    __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&u);
    h[0] = __floats2bfloat162_rn(a.x, a.y); h[1] = __floats2bfloat162_rn(a.z, a.w);
    h[2] = __floats2bfloat162_rn(b.x, b.y); h[3] = __floats2bfloat162_rn(b.z, b.w);
    y[i] = u;
  }
}
__global__ void add_k(float* a, const float* b, size_t n) {
  for (size_t i = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; i < n; i += static_cast<size_t>(gridDim.x) * blockDim.x)
    a[i] += b[i];
}
__global__ void copy_k(float* a, const float* b, size_t n) {
  for (size_t i = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; i < n; i += static_cast<size_t>(gridDim.x) * blockDim.x)
    a[i] = b[i];
}

int grid_for(long n, int threads = 256) { long g = (n + threads - 1) / threads; return static_cast<int>(g < 148 * 16 ? (g < 1 ? 1 : g) : 148 * 16); }

}  // namespace

template <class T>
void embed_fwd(const int32_t* tok, int ld_tok, int B, int s, const T* wte, const T* wpe, T* H, int h, cudaStream_t st) {
  KScope ks_(K_EMBED, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    const long n8 = static_cast<long>(B) * s * (h / 8);
    if (h % 8 == 0 && n8 < (1L << 31) && (reinterpret_cast<uintptr_t>(wte) & 15) == 0 &&
        (!wpe || (reinterpret_cast<uintptr_t>(wpe) & 15) == 0) && (reinterpret_cast<uintptr_t>(H) & 15) == 0) {
      embed_fwd_v8_k<<<grid_for(n8), 256, 0, st>>>(tok, ld_tok, s, wte, wpe, H, h / 8, static_cast<int>(n8));
      note_launch();
      return;
    }
  }
  embed_fwd_k<T><<<grid_for(static_cast<long>(B) * s * h), 256, 0, st>>>(tok, ld_tok, B, s, wte, wpe, H, h);
  note_launch();
}

template <class T>
void embed_bwd(const int32_t* tok, int ld_tok, int B, int s, const T* dH, int h, float* dwte, float* dwpe,
               void* scratch, cudaStream_t st) {
  KScope ks_(K_EMBED, st);
  const int Ttok = B * s;
  int np2 = 1;
  while (np2 < Ttok) np2 <<= 1;
  long long* keys = static_cast<long long*>(scratch);   // scratch holds 2 * Ttok keys (layout.cpp)
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(embed_sort_k, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    cudaFuncSetAttribute(embed_sort_chunk_k, cudaFuncAttributeMaxDynamicSharedMemorySize, kSortChunk * 8);
    attr = true;
  }
  if (np2 <= kSortChunk) {
    embed_sort_k<<<1, 1024, static_cast<size_t>(np2) * sizeof(long long), st>>>(tok, ld_tok, B, s, keys, np2);
    note_launch();
  } else {
    long long* buf[2] = {keys, keys + Ttok};
    int cur = 0;
    embed_sort_chunk_k<<<cdiv(Ttok, kSortChunk), 1024, kSortChunk * 8, st>>>(tok, ld_tok, s, Ttok, buf[0]);
    note_launch();
    for (int w = kSortChunk; w < Ttok; w *= 2) {
      embed_merge_k<<<cdiv(Ttok, 256), 256, 0, st>>>(buf[cur], buf[cur ^ 1], Ttok, w);
      note_launch();
      cur ^= 1;
    }
    keys = buf[cur];
  }
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (h % 8 == 0 && (reinterpret_cast<uintptr_t>(dH) & 15) == 0 && (reinterpret_cast<uintptr_t>(dwte) & 15) == 0) {
      embed_segsum_v8_k<<<cdiv(static_cast<long>(Ttok) * 32, 256), 256, 0, st>>>(keys, Ttok, dH, h, dwte);
      note_launch();
    } else {
      embed_segsum_k<T><<<cdiv(static_cast<long>(Ttok) * 32, 256), 256, 0, st>>>(keys, Ttok, dH, h, dwte);
      note_launch();
    }
  } else {
    if (h % 4 == 0 && (reinterpret_cast<uintptr_t>(dH) & 15) == 0 && (reinterpret_cast<uintptr_t>(dwte) & 15) == 0)
      embed_segsum_f4_k<<<cdiv(static_cast<long>(Ttok) * 32, 256), 256, 0, st>>>(keys, Ttok, dH, h, dwte);
    else
      embed_segsum_k<T><<<cdiv(static_cast<long>(Ttok) * 32, 256), 256, 0, st>>>(keys, Ttok, dH, h, dwte);
    note_launch();
  }
  if (dwpe) {
    bool done = false;
    if constexpr (std::is_same<T, __nv_bfloat16>::value) {
      if (h % 8 == 0 && (reinterpret_cast<uintptr_t>(dH) & 15) == 0 && (reinterpret_cast<uintptr_t>(dwpe) & 15) == 0) {
        embed_pos_bwd_v8_k<<<grid_for(static_cast<long>(s) * (h / 8)), 256, 0, st>>>(dH, B, s, h / 8, dwpe);
        done = true;
      }
    }
    if (!done) embed_pos_bwd_k<T><<<grid_for(static_cast<long>(s) * h), 256, 0, st>>>(dH, B, s, h, dwpe);
    note_launch();
  }
}

bool norm_apply(const __nv_bfloat16* x, const float* g, const float* b, const float* stats, __nv_bfloat16* y, int rows,
                int n, cudaStream_t st);   // rowpipe.cu
template <class T>
void norm_recompute(const T* x, const float* g, const float* b, T* y, float* stats, int rows, int n, float eps, int rms,
                    cudaStream_t st) {
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    KScope ks_(K_NORM, st);
    if (norm_apply(x, g, rms ? nullptr : b, stats, y, rows, n, st)) return;
  }
  if (rms) rmsnorm_fwd<T>(x, g, y, stats, rows, n, eps, st);
  else layernorm_fwd<T>(x, g, b, y, stats, rows, n, eps, st);
}

template <class T>
void layernorm_fwd(const T* x, const float* g, const float* b, T* y, float* stats, int rows, int n, float eps, cudaStream_t st) {
  KScope ks_(K_NORM, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (g_norm_tile == 3 && n <= 4096 && norm_fwd_warp(x, g, b, y, stats, rows, n, eps, 0, st)) return;
    if (g_norm_tile >= 2 && norm_fwd_pipe(x, g, b, y, stats, rows, n, eps, 0, st)) return;
    if (n % 8 == 0) {
      if (n <= 1024) norm_fwd_reg_k<false, 4><<<cdiv(rows, 8), 256, 0, st>>>(x, g, b, y, stats, rows, n, eps);
      else if (n <= 2048) norm_fwd_reg_k<false, 8><<<cdiv(rows, 8), 256, 0, st>>>(x, g, b, y, stats, rows, n, eps);
      else if (n <= 4096) norm_fwd_reg_k<false, 16><<<cdiv(rows, 8), 256, 0, st>>>(x, g, b, y, stats, rows, n, eps);
      else if (n <= 5120) norm_fwd_reg_k<false, 20><<<cdiv(rows, 8), 256, 0, st>>>(x, g, b, y, stats, rows, n, eps);
      else norm_fwd_v8_k<false><<<cdiv(rows, 8), 256, 0, st>>>(x, g, b, y, stats, rows, n, eps);
      note_launch();
      return;
    }
  }
  norm_fwd_k<T, false><<<cdiv(rows, 8), 256, 0, st>>>(x, g, b, y, stats, rows, n, eps);
  note_launch();
}
template <class T>
void rmsnorm_fwd(const T* x, const float* g, T* y, float* stats, int rows, int n, float eps, cudaStream_t st) {
  KScope ks_(K_NORM, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (g_norm_tile == 3 && n <= 4096 && norm_fwd_warp(x, g, nullptr, y, stats, rows, n, eps, 1, st)) return;
    if (g_norm_tile >= 2 && norm_fwd_pipe(x, g, nullptr, y, stats, rows, n, eps, 1, st)) return;
    if (n % 8 == 0) {
      if (n <= 1024) norm_fwd_reg_k<true, 4><<<cdiv(rows, 8), 256, 0, st>>>(x, g, nullptr, y, stats, rows, n, eps);
      else if (n <= 2048) norm_fwd_reg_k<true, 8><<<cdiv(rows, 8), 256, 0, st>>>(x, g, nullptr, y, stats, rows, n, eps);
      else if (n <= 4096) norm_fwd_reg_k<true, 16><<<cdiv(rows, 8), 256, 0, st>>>(x, g, nullptr, y, stats, rows, n, eps);
      else if (n <= 5120) norm_fwd_reg_k<true, 20><<<cdiv(rows, 8), 256, 0, st>>>(x, g, nullptr, y, stats, rows, n, eps);
      else norm_fwd_v8_k<true><<<cdiv(rows, 8), 256, 0, st>>>(x, g, nullptr, y, stats, rows, n, eps);
      note_launch();
      return;
    }
  }
  norm_fwd_k<T, true><<<cdiv(rows, 8), 256, 0, st>>>(x, g, nullptr, y, stats, rows, n, eps);
  note_launch();
}
template <class T>
void norm_bwd_dx(const T* dy, const T* x, const float* stats, const float* g, const T* dres, T* dx, int rows, int n,
                 int rms, cudaStream_t st) {
  KScope ks_(K_NORM, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (g_norm_tile >= 2 && norm_bwd_pipe(dy, x, stats, g, dres, dx, rows, n, rms, nullptr, nullptr, nullptr, nullptr, 0, st))
      return;
    if (g_norm_tile && norm_bwd_tile(dy, x, stats, g, dres, dx, rows, n, rms, nullptr, nullptr, nullptr, nullptr, 0, st))
      return;
    if (n % 8 == 0) {
      if (n <= 1024) norm_bwd_dx_reg_k<4><<<cdiv(rows, 8), 256, 0, st>>>(dy, x, stats, g, dres, dx, rows, n, rms);
      else if (n <= 2048) norm_bwd_dx_reg_k<8><<<cdiv(rows, 8), 256, 0, st>>>(dy, x, stats, g, dres, dx, rows, n, rms);
      else norm_bwd_dx_v8_k<<<cdiv(rows, 8), 256, 0, st>>>(dy, x, stats, g, dres, dx, rows, n, rms);
      note_launch();
      return;
    }
  }
  norm_bwd_dx_k<T><<<cdiv(rows, 8), 256, 0, st>>>(dy, x, stats, g, dres, dx, rows, n, rms);
  note_launch();
}
void colsum_reduce(const float* partial, int nblk, int n, float* out0, float* out1, float* out2, cudaStream_t st) {
  const int arrays = out2 ? 3 : (out1 ? 2 : 1);
  // (a 32-warp variant with every row load issued first measured no faster in whole steps:
  // profiles/r02/colsum_reduce_ab.txt)
  colsum_reduce_k<<<dim3(cdiv(n, 32), arrays), 512, 0, st>>>(partial, nblk, n, out0, out1, out2);
  note_launch();
}
void colsum_finish(const float* partial, int nblk, int n, float* out, cudaStream_t st) {
  KScope ks_(K_COLSUM, st);
  colsum_reduce(partial, nblk, n, out, nullptr, nullptr, st);
}

template <class T>
void colsum(const T* a, const T* x, const float* stats, int rows, int n, int lda, int mode, float* out0, float* out1,
            float* partial, cudaStream_t st) {
  KScope ks_(K_COLSUM, st);
  int nblk = rows < 128 ? rows : 128;
  if (nblk < 1) return;
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (n % 8 == 0 && lda % 8 == 0) {
      const int cb = cdiv(n, 256);
      // ~8 CTAs (64 warps) per SM so enough 16-byte loads are in flight; the partial stays small
      int rb = (8 * device_sms() + cb - 1) / cb;
      rb = rb < 1 ? 1 : (rb > 128 ? 128 : rb);
      rb = rb > rows ? rows : rb;
      nblk = rb;
      dim3 grid(cb, nblk);
      colsum_partial_v2_k<<<grid, 256, 0, st>>>(a, x, stats, rows, n, lda, mode == 2 ? 1 : mode, partial, nblk);
      note_launch();
      colsum_reduce(partial, nblk, n, out0, mode == 1 ? out1 : nullptr, nullptr, st);
      return;
    }
  }
  dim3 grid(cdiv(n, 256), nblk);
  colsum_partial_k<T><<<grid, 256, 0, st>>>(a, x, stats, rows, n, lda, mode == 2 ? 1 : mode, partial, nblk);
  note_launch();
  colsum_reduce(partial, nblk, n, out0, mode == 1 ? out1 : nullptr, nullptr, st);
}

template <class T>
void norm_bwd(const T* dy, const T* x, const float* stats, const float* g, const T* dres, T* dx, int rows, int n,
              int rms, float* dg, float* db, float* dsum, float* partial, size_t partial_floats, cudaStream_t st) {
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (g_norm_tile) {
      KScope ks_(K_NORM, st);
      if (g_norm_tile >= 2 &&
          norm_bwd_pipe(dy, x, stats, g, dres, dx, rows, n, rms, dg, db, dsum, partial, partial_floats, st))
        return;
      if (norm_bwd_tile(dy, x, stats, g, dres, dx, rows, n, rms, dg, db, dsum, partial, partial_floats, st)) return;
    }
  }
  norm_bwd_dx<T>(dy, x, stats, g, dres, dx, rows, n, rms, st);
  colsum<T>(dy, x, stats, rows, n, n, rms ? 2 : 1, dg, db, partial, st);
  if (dsum) colsum<T>(dx, nullptr, nullptr, rows, n, n, 0, dsum, nullptr, partial, st);
}

void norm_bwd_mixed(const __nv_bfloat16* dy, const __nv_bfloat16* x, const float* stats, const float* g,
                    const __nv_bfloat16* dres, const float* dres32, __nv_bfloat16* dx, float* dx32, int rows, int n,
                    int rms, float* dg, float* db, float* dsum, float* partial, size_t partial_floats, cudaStream_t st) {
  KScope ks_(K_NORM, st);
  if (norm_bwd_pipe_mixed(dy, x, stats, g, dres, dres32, dx, dx32, rows, n, rms, dg, db, dsum, partial, partial_floats,
                          st))
    return;
  norm_bwd_mixed_k<<<cdiv(rows, 8), 256, 0, st>>>(dy, x, stats, g, dres, dres32, dx, dx32, rows, n, rms);
  note_launch();
  colsum<__nv_bfloat16>(dy, x, stats, rows, n, n, rms ? 2 : 1, dg, db, partial, st);
  if (dsum) {
    if (dx32) colsum<float>(dx32, nullptr, nullptr, rows, n, n, 0, dsum, nullptr, partial, st);
    else colsum<__nv_bfloat16>(dx, nullptr, nullptr, rows, n, n, 0, dsum, nullptr, partial, st);
  }
}

template <class T>
void attn_fwd(const T* qkv, T* O, float* lse, int B, int s, int nh, int dh, cudaStream_t st, void* pad_ws) {
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (flash_attn_supported(dh)) { flash_attn_fwd(qkv, O, lse, B, s, nh, dh, st, pad_ws); return; }
  }
  (void)pad_ws;
  attn_fwd_k<T><<<cdiv(static_cast<long>(B) * s * nh, 8), 256, 0, st>>>(qkv, O, lse, B, s, nh, dh);
  note_launch();
}
template <class T>
void attn_bwd(const T* qkv, const T* O, const T* dO, const float* lse, T* dqkv, float* Dsc, int B, int s, int nh,
              int dh, cudaStream_t st, void* ds_ws, size_t ds_ws_bytes, void* pad_ws, float* bpart, bool* bpart_done) {
  if (bpart_done) *bpart_done = false;
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (flash_attn_supported(dh)) {
      flash_attn_bwd(qkv, O, dO, lse, dqkv, Dsc, B, s, nh, dh, st, ds_ws, ds_ws_bytes, pad_ws, bpart, bpart_done);
      return;
    }
  }
  (void)bpart;
  (void)ds_ws; (void)ds_ws_bytes; (void)pad_ws;
  const int grid = cdiv(static_cast<long>(B) * s * nh, 8);
  attn_bwd_dq_k<T><<<grid, 256, 0, st>>>(qkv, O, dO, lse, dqkv, Dsc, B, s, nh, dh);
  note_launch();
  attn_bwd_dkdv_k<T><<<grid, 256, 0, st>>>(qkv, dO, lse, Dsc, dqkv, B, s, nh, dh);
  note_launch();
}

void rope_table(float2* tab, int s, int dh, float base, cudaStream_t st) {
  KScope ks_(K_ELEMWISE, st);
  rope_table_k<<<grid_for(static_cast<long>(s) * (dh / 2)), 256, 0, st>>>(tab, s, dh, base);
  note_launch();
}
template <class T>
void rope(T* qkv, int B, int s, int nh, int dh, float base, int inverse, cudaStream_t st, const float2* tab) {
  KScope ks_(K_ELEMWISE, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    const int h8 = dh / 16;
    if (tab && dh % 16 == 0 && static_cast<long>(B) * s <= 65535 &&
        (reinterpret_cast<uintptr_t>(qkv) & 15) == 0) {
      const int nthr = nh * h8, bx = nthr < 256 ? ((nthr + 31) / 32) * 32 : 256;
      dim3 grid((nthr + bx - 1) / bx, static_cast<unsigned>(static_cast<long>(B) * s));
      rope_v8_k<<<grid, bx, 0, st>>>(qkv, tab, s, nh, dh, inverse);
      note_launch();
      return;
    }
  }
  (void)tab;
  rope_k<T><<<grid_for(static_cast<long>(B) * s * nh * (dh / 2)), 256, 0, st>>>(qkv, B, s, nh, dh, base, inverse);
  note_launch();
}
template <class T>
void swiglu_fwd(const T* GU, T* M, int rows, int f, cudaStream_t st) {
  KScope ks_(K_ELEMWISE, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (f % 8 == 0) {
      swiglu_fwd_v8_k<<<dim3(cdiv(f / 8, 256), rows), 256, 0, st>>>(GU, M, rows, f);
      note_launch();
      return;
    }
  }
  swiglu_fwd_k<T><<<grid_for(static_cast<long>(rows) * f), 256, 0, st>>>(GU, M, rows, f);
  note_launch();
}
template <class T>
void swiglu_bwd(const T* GU, const T* dM, T* dGU, int rows, int f, cudaStream_t st) {
  KScope ks_(K_ELEMWISE, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (f % 8 == 0) {
      swiglu_bwd_v8_k<<<dim3(cdiv(f / 8, 256), rows), 256, 0, st>>>(GU, dM, dGU, rows, f);
      note_launch();
      return;
    }
  }
  swiglu_bwd_k<T><<<grid_for(static_cast<long>(rows) * f), 256, 0, st>>>(GU, dM, dGU, rows, f);
  note_launch();
}
template <class T>
void softmax_ce(const float* logits, const int32_t* tok, int ld_tok, int s, int rows, int V, float inv_ntok,
                T* dlogits, float* row_loss, cudaStream_t st, long row0) {
  KScope ks_(K_CE, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (softmax_ce_fast(logits, tok, ld_tok, s, rows, V, inv_ntok, dlogits, row_loss, st, row0)) return;
  }
  softmax_ce_k<T><<<rows, 512, 0, st>>>(logits, tok, ld_tok, s, V, inv_ntok, dlogits, row_loss, row0);
  note_launch();
}
template <class T>
void gelu_fwd(const T* Z, T* G, size_t n, cudaStream_t st) {
  KScope ks_(K_ELEMWISE, st);
  if constexpr (std::is_same<T, __nv_bfloat16>::value) {
    if (n % 8 == 0 && reinterpret_cast<uintptr_t>(Z) % 16 == 0 && reinterpret_cast<uintptr_t>(G) % 16 == 0) {
      gelu_fwd_v8_k<<<grid_for(static_cast<long>(n / 8)), 256, 0, st>>>(reinterpret_cast<const uint4*>(Z),
                                                                        reinterpret_cast<uint4*>(G), n / 8);
      note_launch();
      return;
    }
  }
  gelu_fwd_k<T><<<grid_for(static_cast<long>(n)), 256, 0, st>>>(Z, G, n);
  note_launch();
}
void loss_reduce(const float* row_loss, int rows, double* out, cudaStream_t st) {
  KScope ks_(K_CE, st);
  loss_reduce_k<<<1, 1024, 0, st>>>(row_loss, rows, out);
  note_launch();
}
void cast_f32_bf16(const float* x, __nv_bfloat16* y, size_t n, cudaStream_t st) {
  KScope ks_(K_ELEMWISE, st);
  if (n % 8 == 0 && (reinterpret_cast<uintptr_t>(x) & 15) == 0 && (reinterpret_cast<uintptr_t>(y) & 15) == 0) {
    cast_v8_k<<<grid_for(static_cast<long>(n / 8)), 256, 0, st>>>(reinterpret_cast<const float4*>(x),
                                                                  reinterpret_cast<uint4*>(y), n / 8);
  } else {
    cast_k<<<grid_for(static_cast<long>(n)), 256, 0, st>>>(x, y, n);
  }
  note_launch();
}
void add_f32(float* a, const float* b, size_t n, cudaStream_t st) { add_k<<<grid_for(static_cast<long>(n)), 256, 0, st>>>(a, b, n); note_launch(); }
void copy_f32(float* a, const float* b, size_t n, cudaStream_t st) { copy_k<<<grid_for(static_cast<long>(n)), 256, 0, st>>>(a, b, n); note_launch(); }

// dst[i] = ((src0[i] + src1[i]) + src2[i]) + ...: the copies of one parameter summed in copy order
// (the loopback's acc = c0; acc += c1; ... association). Every source is read before dst is
// written, so dst may be one of the sources; sources may live in another rank's memory.
__global__ void sum_copies_k(float* dst, CopySrcs s, size_t n) {
  for (size_t i = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; i < n;
       i += static_cast<size_t>(gridDim.x) * blockDim.x) {
    float acc = s.p[0][i];
    for (int c = 1; c < s.n; ++c) acc += s.p[c][i];
    dst[i] = acc;
  }
}
void sum_copies_f32(float* dst, const CopySrcs& srcs, size_t n, cudaStream_t st) {
  sum_copies_k<<<grid_for(static_cast<long>(n)), 256, 0, st>>>(dst, srcs, n);
  note_launch();
}

#define INST(T)                                                                                                     \
  template void embed_fwd<T>(const int32_t*, int, int, int, const T*, const T*, T*, int, cudaStream_t);              \
  template void embed_bwd<T>(const int32_t*, int, int, int, const T*, int, float*, float*, void*, cudaStream_t);     \
  template void layernorm_fwd<T>(const T*, const float*, const float*, T*, float*, int, int, float, cudaStream_t);  \
  template void rmsnorm_fwd<T>(const T*, const float*, T*, float*, int, int, float, cudaStream_t);                   \
  template void norm_bwd_dx<T>(const T*, const T*, const float*, const float*, const T*, T*, int, int, int,          \
                               cudaStream_t);                                                                      \
  template void norm_recompute<T>(const T*, const float*, const float*, T*, float*, int, int, float, int,          \
                                  cudaStream_t);                                                                 \
  template void colsum<T>(const T*, const T*, const float*, int, int, int, int, float*, float*, float*, cudaStream_t); \
  template void norm_bwd<T>(const T*, const T*, const float*, const float*, const T*, T*, int, int, int, float*,      \
                            float*, float*, float*, size_t, cudaStream_t);                                           \
  template void attn_fwd<T>(const T*, T*, float*, int, int, int, int, cudaStream_t, void*);                                 \
  template void attn_bwd<T>(const T*, const T*, const T*, const float*, T*, float*, int, int, int, int, cudaStream_t, \
                            void*, size_t, void*, float*, bool*);                                                  \
  template void rope<T>(T*, int, int, int, int, float, int, cudaStream_t, const float2*);                             \
  template void swiglu_fwd<T>(const T*, T*, int, int, cudaStream_t);                                                 \
  template void swiglu_bwd<T>(const T*, const T*, T*, int, int, cudaStream_t);                                       \
  template void softmax_ce<T>(const float*, const int32_t*, int, int, int, int, float, T*, float*, cudaStream_t,    \
                              long);                                                                                \
  template void gelu_fwd<T>(const T*, T*, size_t, cudaStream_t);
INST(float)
INST(__nv_bfloat16)

}  // namespace mario
