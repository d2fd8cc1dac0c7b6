// SPOS CNN kernels (configs[1]): NHWC activations, fp32 BatchNorm statistics and masters,
// CUDA cores for everything that is not a dense contraction (the 1x1 convs and the frozen
// head's 1x1 conv run on the tcgen05 GEMM, gemm.cu).
//
// Storage (A28): forward tensors (conv outputs z, BN/ReLU outputs y, block
// outputs) are bf16x2 -- two bf16 planes, hi = bf16(v) and lo = bf16(v - hi), lo plane at
// `plane` elements after hi -- i.e. a 16-bit mantissa, because BatchNorm + ReLU turn any
// 2^-9 perturbation of the forward activations into ReLU-mask flips that decorrelate the
// weight gradient; backward tensors (dy, dz, dx) are plain bf16.
//
// Block internals follow SURVEY §8c "C2 SPOS candidate" (readings A16, A27):
// every conv is bias-free and followed by training-mode BatchNorm (batch statistics over
// N*H*W, biased variance, eps 1e-5).  Per conv -> BN [-> ReLU] unit the forward is
//   conv -> z;  bn_stats(z) -> per-row-block partials (sum, sum of squares), the last CTA
//   reduces them to mean, rstd;  bn_apply -> y = relu?(g * ((z - mean) * rstd) + b)
// and the backward (dy = grad of y; s1 = sum dy', s2 = sum dy' * xh over the batch, dy' = dy
// masked by the ReLU):
//   bn_bwd_reduce -> partials of s1, s2, the last CTA reduces them and applies the WRITE of
//   g, b (dg = s2, db = s1; the pre-update g, b are kept for the input gradient);
//   bn_bwd_apply -> dz = rstd * g * (dy' - s1/P - xh * s2/P)  (bf16).
// Every reduction has a fixed order (per-thread sequential, then a fixed cross-thread order,
// then a fixed order over row blocks), never floating-point atomics: bitwise reproducible.
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>

#include "common.h"
#include "kernels.h"
#include "launch.h"
#include "bnfuse.cuh"
#include "fixpoint.cuh"
#include "ptx.cuh"

namespace naspipe {
namespace {

constexpr int TPB = 256;          // threads per block of the row-block kernels
// target CTAs of the row-block reductions: fewer, longer row blocks keep the partial count
// (and so the fixed-order finalize) short; NASPIPE_RED_CTAS overrides it for tuning.
static int red_ctas() {
  static const int v = [] {  // thread-safe one-time init
    const char* e = getenv("NASPIPE_RED_CTAS");
    return e ? std::max(16, atoi(e)) : 296;
  }();
  return v;
}
// target CTAs of the depthwise weight-gradient partials (NASPIPE_DW_RED_CTAS, default: the
// BatchNorm target above)
static int dw_red_ctas() {
  static const int v = [] {  // thread-safe one-time init
    const char* e = getenv("NASPIPE_DW_RED_CTAS");
    return e ? std::max(16, atoi(e)) : red_ctas();
  }();
  return v;
}
constexpr float BN_EPS = 1e-5f;

// Row blocking of the per-channel reductions: a function of (P, C) only (deterministic),
// about RED_CTAS blocks, each a multiple of the kernel's row lanes RP = TPB / (C/8).
// Each row lane handles at least NASPIPE_RED_MIN_ITERS rows (default 8; measured 1 / 4 / 8 / 16 /
// 32: 6.47 / 6.35 / 6.33 / 6.59 / 7.06 ms per configs[1] step): small tensors
// (the 7x7 / 14x14 stages, P = 3136 / 12544) otherwise spread a few rows over ~700 CTAs, each
// paying the shared-memory reduction and 2C fixed-point atomics on the same 2C addresses.
static int red_min_iters() {
  static const int v = [] {
    const char* e = getenv("NASPIPE_RED_MIN_ITERS");
    return e ? std::max(1, atoi(e)) : 8;
  }();
  return v;
}
inline int red_rows(int P, int C, int vec = 8, int target = 0) {
  const int rp = TPB / (C / vec);
  if (target <= 0) target = red_ctas();
  int rows = (P + target - 1) / target;
  rows = std::max(rows, rp * red_min_iters());
  rows = ((rows + rp - 1) / rp) * rp;
  return rows < rp ? rp : rows;
}

inline void check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}
inline int grid_for(size_t items, int per_block = TPB) {
  const size_t g = (items + per_block - 1) / per_block;
  return (int)std::min<size_t>(std::max<size_t>(g, 1), (size_t)num_sms() * 16);
}

__device__ __forceinline__ void load8(const bf16* p, float (&v)[8]) {
  const uint4 q = *reinterpret_cast<const uint4*>(p);
  const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    v[2 * i] = __uint_as_float(w[i] << 16);
    v[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
  }
}
__device__ __forceinline__ void store8(bf16* p, const float (&v)[8]) {
  uint4 q;
  q.x = ptx::pack_bf16(v[0], v[1]);
  q.y = ptx::pack_bf16(v[2], v[3]);
  q.z = ptx::pack_bf16(v[4], v[5]);
  q.w = ptx::pack_bf16(v[6], v[7]);
  *reinterpret_cast<uint4*>(p) = q;
}
// bf16x2: v = hi + lo (exact in fp32); store: hi = RNE(v), lo = RNE(v - hi)
__device__ __forceinline__ void load8x2(const bf16* p, size_t plane, float (&v)[8]) {
  float lo[8];
  load8(p, v);
  load8(p + plane, lo);
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] += lo[i];
}
__device__ __forceinline__ void store8x2(bf16* p, size_t plane, const float (&v)[8]) {
  float lo[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) lo[i] = v[i] - __bfloat162float(__float2bfloat16_rn(v[i]));
  store8(p, v);
  store8(p + plane, lo);
}
__device__ __forceinline__ void load8f(const float* p, float (&v)[8]) {
  const float4 a = reinterpret_cast<const float4*>(p)[0], b = reinterpret_cast<const float4*>(p)[1];
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}

// ---------------------------------------------------------------- frozen stem (conv3x3 s2)
// x fp32 NHWC [B,H,H,3], w fp32 [C0][3][3][3] ([out, kh, kw, in]), pad 1 -> z bf16 [B,H/2,H/2,C0]
__global__ void stem_conv_kernel(const float* __restrict__ x, const float* __restrict__ w, bf16* __restrict__ z,
                                 int B, int H, int C0) {
  extern __shared__ float ws[];
  ptx::pdl_wait();
  for (int i = threadIdx.x; i < C0 * 27; i += blockDim.x) ws[i] = w[i];
  __syncthreads();
  const int Ho = H / 2;
  const size_t P = (size_t)B * Ho * Ho;
  for (size_t p = blockIdx.x * (size_t)blockDim.x + threadIdx.x; p < P; p += (size_t)gridDim.x * blockDim.x) {
    const int b = (int)(p / ((size_t)Ho * Ho));
    const int rem = (int)(p % ((size_t)Ho * Ho));
    const int oh = rem / Ho, ow = rem % Ho;
    float in[27];
#pragma unroll
    for (int u = 0; u < 3; ++u)
#pragma unroll
      for (int v = 0; v < 3; ++v) {
        const int ih = 2 * oh + u - 1, iw = 2 * ow + v - 1;
        const bool ok = ih >= 0 && ih < H && iw >= 0 && iw < H;
        const float* src = x + (((size_t)b * H + (ok ? ih : 0)) * H + (ok ? iw : 0)) * 3;
#pragma unroll
        for (int ci = 0; ci < 3; ++ci) in[(u * 3 + v) * 3 + ci] = ok ? src[ci] : 0.f;
      }
    for (int c0 = 0; c0 < C0; c0 += 8) {
      float acc[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        float a = 0.f;
        const float* wc = ws + (c0 + i) * 27;
#pragma unroll
        for (int t = 0; t < 27; ++t) a = __fmaf_rn(in[t], wc[t], a);
        acc[i] = a;
      }
      store8x2(z + p * C0 + c0, P * C0, acc);
    }
  }
}

// ---------------------------------------------------------------- BatchNorm forward
// Per-channel reductions over P rows without a finalize launch and without float atomics:
// each CTA reduces its row block in a fixed order (per-thread sequential, then the RP lane
// sums in lane order) to fp32 partials, converts them to 64-bit FIXED POINT and adds them
// with integer atomics into acc[2C].  Integer addition is associative, so the totals --
// and everything computed from them -- are bitwise independent of the CTA arrival order.
// The consumer kernel (bn_apply / bn_bwd_apply) reads the totals; its last CTA (arrival
// ticket) publishes the per-channel results and zeroes acc and the ticket for the next use.
//
// Fixed-point scales, fix_add / fix_get and the overflow flag acc[2C]: fixpoint.cuh.

// arrival ticket: true in every thread of the CTA that arrives last (all others are done)
__device__ __forceinline__ bool last_cta(int* ticket) {
  __shared__ int last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(ticket, 1) == (int)(gridDim.x * gridDim.y) - 1;
  }
  __syncthreads();
  if (last) __threadfence();
  return last;
}

// mean = s1 / P, rstd = 1/sqrt(s2 / P - mean^2 + eps) (biased variance), from the totals
__device__ __forceinline__ void bn_moments(const unsigned long long* acc, int C, int c, int P, float& mu, float& rs) {
  const double m = fix_get(acc, c, FIX_S1) / P;
  const double var = fmax(fix_get(acc, C + c, FIX_S2) / P - m * m, 0.0);
  mu = (float)m;
  rs = (float)(1.0 / sqrt(var + (double)BN_EPS));
}

// Thread (r, g): rows r, r + RP, ... of its block, channels [8g, 8g+8); RP = TPB / G row
// lanes; the RP lane sums are combined in lane order, then added to acc (fixed point).
__global__ void bn_stats_kernel(const bf16* __restrict__ z, int P, int C, int rows, unsigned long long* acc) {
  extern __shared__ float red[];  // [RP][2C]
  ptx::pdl_wait();
  const int G = C / 8, RP = TPB / G;
  const int r = threadIdx.x / G, g = threadIdx.x % G;
  const int row0 = blockIdx.x * rows, row1 = min(P, row0 + rows);
  const size_t plane = (size_t)P * C;
  if (r < RP) {
    float s[8] = {}, q[8] = {};
    int row = row0 + r;
    for (; row + 3 * RP < row1; row += 4 * RP) {
      float v[4][8];
#pragma unroll
      for (int u = 0; u < 4; ++u) load8x2(z + (size_t)(row + u * RP) * C + 8 * g, plane, v[u]);
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          s[i] += v[u][i];
          q[i] = __fmaf_rn(v[u][i], v[u][i], q[i]);
        }
    }
    for (; row < row1; row += RP) {
      float v[8];
      load8x2(z + (size_t)row * C + 8 * g, plane, v);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        s[i] += v[i];
        q[i] = __fmaf_rn(v[i], v[i], q[i]);
      }
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      red[r * 2 * C + 8 * g + i] = s[i];
      red[r * 2 * C + C + 8 * g + i] = q[i];
    }
  }
  __syncthreads();
  for (int e = threadIdx.x; e < 2 * C; e += TPB) {
    float a = 0.f;
    for (int k = 0; k < RP; ++k) a += red[k * 2 * C + e];
    fix_add(acc, e, acc + 2 * C, a, e < C ? FIX_S1 : FIX_S2);
  }
}

// Elementwise kernels over [P rows][C]: thread (pixel lane, channel group g) keeps its
// group's per-channel parameters in registers and strides over pixels.
__device__ __forceinline__ int ew_lanes(int C) { return TPB / (C / 8); }

template <int U>  // pixels in flight per thread
__device__ __forceinline__ void bn_apply_body(const bf16* __restrict__ z, int P, int C, const unsigned long long* acc,
                                              const float* __restrict__ gam, const float* __restrict__ bet, int relu,
                                              bf16* __restrict__ y, int ldy, size_t yplane, float* mean = nullptr,
                                              float* rstd = nullptr, unsigned long long* clear = nullptr,
                                              int clear_n = 0) {
  // the CTA derives every channel's moments once (fp64, from the fixed-point totals)
  __shared__ float smu[2048], srs[2048];  // C <= 8 TPB = 2048 (host check)
  for (int cc = threadIdx.x; cc < C; cc += blockDim.x) {
    bn_moments(acc, C, cc, P, smu[cc], srs[cc]);
    if (mean != nullptr && blockIdx.x == 0) {  // ring mode: CTA 0 publishes (same values in every CTA)
      mean[cc] = smu[cc];
      rstd[cc] = srs[cc];
    }
  }
  if (clear != nullptr && blockIdx.x == 0)
    for (int e = threadIdx.x; e < clear_n; e += blockDim.x) clear[e] = 0ull;
  __syncthreads();
  const int G = C / 8, lanes = ew_lanes(C);
  const int pl = threadIdx.x / G, c = (threadIdx.x % G) * 8;
  if (pl >= lanes) return;
  float mu[8], rs[8], g8[8], b8[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    mu[i] = smu[c + i];
    rs[i] = srs[c + i];
  }
  load8f(gam + c, g8);
  load8f(bet + c, b8);
  const size_t zplane = (size_t)P * C;
  const int step = gridDim.x * lanes;
  int p = blockIdx.x * lanes + pl;
  for (; p + (U - 1) * step < P; p += U * step) {  // U pixels in flight
    float v[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) load8x2(z + (size_t)(p + u * step) * C + c, zplane, v[u]);
#pragma unroll
    for (int u = 0; u < U; ++u) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const float o = bn_y(v[u][i], mu[i], rs[i], g8[i], b8[i]);
        v[u][i] = relu ? fmaxf(o, 0.f) : o;
      }
      store8x2(y + (size_t)(p + u * step) * ldy + c, yplane, v[u]);
    }
  }
  for (; p < P; p += step) {
    float v[8];
    load8x2(z + (size_t)p * C + c, zplane, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const float o = bn_y(v[i], mu[i], rs[i], g8[i], b8[i]);
      v[i] = relu ? fmaxf(o, 0.f) : o;
    }
    store8x2(y + (size_t)p * ldy + c, yplane, v);
  }
}

template <int U>
__global__ void bn_apply_kernel(const bf16* __restrict__ z, int P, int C, unsigned long long* acc, int* ticket,
                                float* __restrict__ mean, float* __restrict__ rstd, const float* __restrict__ gam,
                                const float* __restrict__ bet, int relu, bf16* __restrict__ y, int ldy,
                                size_t yplane, unsigned long long* clear, int clear_n) {
  ptx::pdl_wait();
  if (ticket == nullptr) {  // ring mode (kernels.h BnWrite note): no ticket, no fence, no serial tail
    bn_apply_body<U>(z, P, C, acc, gam, bet, relu, y, ldy, yplane, mean, rstd, clear, clear_n);
    return;
  }
  bn_apply_body<U>(z, P, C, acc, gam, bet, relu, y, ldy, yplane);
  if (last_cta(ticket)) {  // every CTA has read the totals: publish mean / rstd, clear
    for (int c = threadIdx.x; c < C; c += blockDim.x) {
      float mu, rs;
      bn_moments(acc, C, c, P, mu, rs);
      mean[c] = mu;
      rstd[c] = rs;
    }
    __syncthreads();
    for (int e = threadIdx.x; e < 2 * C; e += blockDim.x) acc[e] = 0ull;
    if (threadIdx.x == 0) *ticket = 0;
  }
}

// ---------------------------------------------------------------- BatchNorm backward
// 4 channels per thread (BV): the per-channel constants (mean, rstd, g, b, s1, s2) of 8
// channels held 92-96 registers (2 CTAs/SM, 25 % occupancy, ~2 TB/s measured by ncu);
// 4 channels halve them.
constexpr int BV = 4;
__device__ __forceinline__ void load4(const bf16* p, float (&v)[4]) {
  const uint2 q = *reinterpret_cast<const uint2*>(p);
  v[0] = __uint_as_float(q.x << 16);
  v[1] = __uint_as_float(q.x & 0xffff0000u);
  v[2] = __uint_as_float(q.y << 16);
  v[3] = __uint_as_float(q.y & 0xffff0000u);
}
__device__ __forceinline__ void load4x2(const bf16* p, size_t plane, float (&v)[4]) {
  float lo[4];
  load4(p, v);
  load4(p + plane, lo);
#pragma unroll
  for (int i = 0; i < 4; ++i) v[i] += lo[i];
}
__device__ __forceinline__ void store4(bf16* p, const float (&v)[4]) {
  *reinterpret_cast<uint2*>(p) = make_uint2(ptx::pack_bf16(v[0], v[1]), ptx::pack_bf16(v[2], v[3]));
}
__device__ __forceinline__ void load4f(const float* p, float (&v)[4]) {
  const float4 a = *reinterpret_cast<const float4*>(p);
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
}

__device__ __forceinline__ void bn_bwd_item(const bf16* dy, const bf16* z, size_t zplane, const float (&mu)[BV],
                                            const float (&rs)[BV], const float (&g8)[BV], const float (&b8)[BV],
                                            int relu, float (&d)[BV], float (&xh)[BV]) {
  float zz[BV];
  load4(dy, d);
  load4x2(z, zplane, zz);
#pragma unroll
  for (int i = 0; i < BV; ++i) bn_bwd_elem(d[i], zz[i], mu[i], rs[i], g8[i], b8[i], relu, xh[i]);
}

// s1 = sum dy', s2 = sum dy' xh (dy' = dy masked by the ReLU): fixed-order row-block
// partials added to acc[2C] in fixed point (see bn_stats_kernel).  Thread (r, g): rows r,
// r + RP, ... of its block, channels [4g, 4g+4); RP = TPB / (C/4).
template <int UR>  // rows in flight per lane (the sums stay in row order whatever UR)
__global__ void bn_bwd_reduce_kernel(const bf16* __restrict__ dy, int lddy, const bf16* __restrict__ z, int P, int C,
                                     const float* __restrict__ mean, const float* __restrict__ rstd,
                                     const float* __restrict__ gam, const float* __restrict__ bet, int relu,
                                     int rows, unsigned long long* acc) {
  extern __shared__ float red[];  // [RP][2C]
  ptx::pdl_wait();
  const int G = C / BV, RP = TPB / G;
  const int r = threadIdx.x / G, g = threadIdx.x % G;
  const int row0 = blockIdx.x * rows, row1 = min(P, row0 + rows);
  const size_t zplane = (size_t)P * C;
  if (r < RP) {
    float mu[BV], rs[BV], g8[BV], b8[BV];
    load4f(mean + BV * g, mu);
    load4f(rstd + BV * g, rs);
    load4f(gam + BV * g, g8);
    load4f(bet + BV * g, b8);
    float s1[BV] = {}, s2[BV] = {};
    int row = row0 + r;
    for (; row + (UR - 1) * RP < row1; row += UR * RP) {  // UR rows in flight
      float d[UR][BV], xh[UR][BV];
#pragma unroll
      for (int u = 0; u < UR; ++u)
        bn_bwd_item(dy + (size_t)(row + u * RP) * lddy + BV * g, z + (size_t)(row + u * RP) * C + BV * g, zplane, mu,
                    rs, g8, b8, relu, d[u], xh[u]);
#pragma unroll
      for (int u = 0; u < UR; ++u)
#pragma unroll
        for (int i = 0; i < BV; ++i) {
          s1[i] += d[u][i];
          s2[i] = __fmaf_rn(d[u][i], xh[u][i], s2[i]);
        }
    }
    for (; row < row1; row += RP) {
      float d[BV], xh[BV];
      bn_bwd_item(dy + (size_t)row * lddy + BV * g, z + (size_t)row * C + BV * g, zplane, mu, rs, g8, b8, relu, d, xh);
#pragma unroll
      for (int i = 0; i < BV; ++i) {
        s1[i] += d[i];
        s2[i] = __fmaf_rn(d[i], xh[i], s2[i]);
      }
    }
#pragma unroll
    for (int i = 0; i < BV; ++i) {
      red[r * 2 * C + BV * g + i] = s1[i];
      red[r * 2 * C + C + BV * g + i] = s2[i];
    }
  }
  __syncthreads();
  for (int e = threadIdx.x; e < 2 * C; e += TPB) {
    float a = 0.f;
    for (int k = 0; k < RP; ++k) a += red[k * 2 * C + e];
    fix_add(acc, e, acc + 2 * C, a, FIX_B);
  }
}

template <int U>  // pixels in flight per thread
__device__ __forceinline__ void bn_bwd_apply_body(const bf16* __restrict__ dy, int lddy, const bf16* __restrict__ z,
                                                  int P, int C, const float* __restrict__ mean,
                                                  const float* __restrict__ rstd, const float* __restrict__ gam,
                                                  const float* __restrict__ bet, const unsigned long long* acc, int relu,
                                                  bf16* __restrict__ dz) {
  __shared__ float sm1[1024], sm2[1024];  // the CTA converts the fixed-point totals once (C <= 4 TPB)
  for (int cc = threadIdx.x; cc < C; cc += blockDim.x) {
    sm1[cc] = (float)fix_get(acc, cc, FIX_B);
    sm2[cc] = (float)fix_get(acc, C + cc, FIX_B);
  }
  __syncthreads();
  const int G = C / BV, lanes = TPB / G;
  const int pl = threadIdx.x / G, c = (threadIdx.x % G) * BV;
  if (pl >= lanes) return;
  const float invP = 1.0f / (float)P;
  float mu[BV], rs[BV], g8[BV], b8[BV], m1[BV], m2[BV];
  load4f(mean + c, mu);
  load4f(rstd + c, rs);
  load4f(gam + c, g8);
  load4f(bet + c, b8);
#pragma unroll
  for (int i = 0; i < BV; ++i) {
    m1[i] = sm1[c + i] * invP;
    m2[i] = sm2[c + i] * invP;
  }
  const size_t zplane = (size_t)P * C;
  const int step = gridDim.x * lanes;
  int p = blockIdx.x * lanes + pl;
  for (; p + (U - 1) * step < P; p += U * step) {  // U pixels in flight
    float d[U][BV], xh[U][BV];
#pragma unroll
    for (int u = 0; u < U; ++u)
      bn_bwd_item(dy + (size_t)(p + u * step) * lddy + c, z + (size_t)(p + u * step) * C + c, zplane, mu, rs, g8, b8,
                  relu, d[u], xh[u]);
#pragma unroll
    for (int u = 0; u < U; ++u) {
#pragma unroll
      for (int i = 0; i < BV; ++i) d[u][i] = rs[i] * g8[i] * (d[u][i] - m1[i] - xh[u][i] * m2[i]);
      store4(dz + (size_t)(p + u * step) * C + c, d[u]);
    }
  }
  for (; p < P; p += step) {
    float d[BV], xh[BV];
    bn_bwd_item(dy + (size_t)p * lddy + c, z + (size_t)p * C + c, zplane, mu, rs, g8, b8, relu, d, xh);
#pragma unroll
    for (int i = 0; i < BV; ++i) d[i] = rs[i] * g8[i] * (d[i] - m1[i] - xh[i] * m2[i]);
    store4(dz + (size_t)p * C + c, d);
  }
}

// dz = rstd g (dy' - s1/P - xh s2/P) with the PRE-update g, b (reading A4: the input
// gradient uses the weights before the WRITE); the last CTA -- after every CTA has read
// g, b -- applies the WRITE g -= lr s2, b -= lr s1 (into gu/bu: g/b in place, the bulk
// accumulator under BSP) and clears acc and the ticket.
// the deferred WRITE of a previous use (ring mode): g -= lr s2, b -= lr s1, then zero its sums
__device__ __forceinline__ void bn_write(const BnWrite& w) {
  if (w.acc == nullptr) return;
  if (w.update)
    for (int c = threadIdx.x; c < w.C; c += blockDim.x) {
      const float f1 = (float)fix_get(w.acc, c, FIX_B), f2 = (float)fix_get(w.acc, w.C + c, FIX_B);
      w.gu[c] = (w.gu == w.g ? w.g[c] : w.gu[c]) - w.lr * f2;
      w.bu[c] = (w.bu == w.b ? w.b[c] : w.bu[c]) - w.lr * f1;
    }
  __syncthreads();  // every thread has read the sums
  for (int e = threadIdx.x; e < 2 * w.C; e += blockDim.x) w.acc[e] = 0ull;
}

__global__ void bn_write_kernel(const BnWrite w) {
  ptx::pdl_wait();
  bn_write(w);
}

template <int U>
__global__ void bn_bwd_apply_kernel(const bf16* __restrict__ dy, int lddy, const bf16* __restrict__ z, int P, int C,
                                    const float* __restrict__ mean, const float* __restrict__ rstd, const float* gam,
                                    const float* bet, float* gamu, float* betu, float lr, int update,
                                    unsigned long long* acc, int* ticket, int relu, bf16* __restrict__ dz,
                                    const BnWrite prev) {
  ptx::pdl_wait();
  if (ticket == nullptr) {  // ring mode: CTA 0 first performs the previous use's deferred WRITE
    if (blockIdx.x == 0) bn_write(prev);
    bn_bwd_apply_body<U>(dy, lddy, z, P, C, mean, rstd, gam, bet, acc, relu, dz);
    return;
  }
  bn_bwd_apply_body<U>(dy, lddy, z, P, C, mean, rstd, gam, bet, acc, relu, dz);
  if (last_cta(ticket)) {
    if (update)
      for (int c = threadIdx.x; c < C; c += blockDim.x) {
        const float f1 = (float)fix_get(acc, c, FIX_B), f2 = (float)fix_get(acc, C + c, FIX_B);
        gamu[c] = (gamu == gam ? gam[c] : gamu[c]) - lr * f2;
        betu[c] = (betu == bet ? bet[c] : betu[c]) - lr * f1;
      }
    __syncthreads();
    for (int e = threadIdx.x; e < 2 * C; e += blockDim.x) acc[e] = 0ull;
    if (threadIdx.x == 0) *ticket = 0;
  }
}

// ---------------------------------------------------------------- depthwise conv (pad K/2): stride-2 input gradient
// weights fp32 [C][K][K]; staged in shared memory as [K*K][C]
template <int K>
__device__ __forceinline__ void stage_dw_weights(float* ws, const float* w, int C) {
  for (int i = threadIdx.x; i < C * K * K; i += blockDim.x) {
    const int c = i / (K * K), t = i % (K * K);
    ws[t * C + c] = w[i];
  }
  __syncthreads();
}

// ---------------------------------------------------------------- depthwise conv, shared-memory tiles
// Correlation out[b,oh,ow,c] = sum_{u,v} in[b, oh*S+u*DIL-PAD, ow*S+v*DIL-PAD, c] w'[c,u,v] (+ add),
// PAD = DIL*(K/2), KE = DIL*(K-1)+1 the dilated extent,
// w' = w (forward) or w flipped in u and v (FLIP: the stride-1 input gradient).  A CTA owns
// a tile of DT_H output rows x TW columns x CPG groups of 8 channels: the input halo is
// staged in shared memory once (16-byte loads, fp32), each thread keeps one channel's k x k
// weights in registers and computes a DT_H-row strip of one column from shared memory (each
// staged value feeds up to DT_H outputs).  X2: bf16x2 input/output (forward), else bf16.
// Fused reductions (fixed order per CTA, fixed point across CTAs): X2 with `stats` adds the
// BatchNorm sums of the stored output (bn_stats); FLIP with bnb.acc adds the BatchNorm-backward
// sums of the unit whose output gradient the stored dx is (bn_bwd_reduce, BnBwdFuse).
constexpr int DT_H = 8;

// XBN (forward, X2): the input is y = relu?(BN(z)) of a unit whose bn_apply was folded in
// here (BnApplyIn): the halo loads z and applies BN [+ ReLU] with the CTA's per-channel
// moments from the fixed-point sums, rounding y to bf16x2 as bn_apply stores it; the last
// CTA publishes mean / rstd and the g / b used, and clears the sums (bn_apply's duties).
constexpr int XBN_CH = TPB / 8;  // channels of a CTA: CPG * 8 <= 32

// per-channel BN parameters of channels [c0, c0 + n) in shared memory: forward = moments
// from the fixed-point sums and the live g, b; backward = the published mean / rstd and the
// forward's g, b snapshots
__device__ __forceinline__ void xbn_stage(const BnApplyIn& xb, bool fwd, int c0, int n, int C, float* mu, float* rs,
                                          float* g, float* b) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    const int c = c0 + i;
    if (c >= C) continue;
    if (fwd) {
      bn_moments(xb.acc, C, c, xb.P, mu[i], rs[i]);
      g[i] = xb.g[c];
      b[i] = xb.b[c];
    } else {
      mu[i] = xb.mean[c];
      rs[i] = xb.rstd[c];
      g[i] = xb.gsnap[c];
      b[i] = xb.bsnap[c];
    }
  }
  __syncthreads();
}
// y of 8 channels (smem parameter index j0) from z, rounded to bf16x2 (hi + lo) or, HI_ONLY,
// to its hi plane
template <bool HI_ONLY>
__device__ __forceinline__ void xbn_y8(float (&v)[8], const float* mu, const float* rs, const float* g, const float* b,
                                       int j0, int relu) {
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    float y = bn_y(v[j], mu[j0 + j], rs[j0 + j], g[j0 + j], b[j0 + j]);
    y = relu ? fmaxf(y, 0.f) : y;
    const float hi = __bfloat162float(__float2bfloat16_rn(y));
    v[j] = HI_ONLY ? hi : hi + __bfloat162float(__float2bfloat16_rn(y - hi));
  }
}

template <int K, int S, int DIL, bool X2, bool FLIP, bool XBN = false, int DH = DT_H>
__global__ void __launch_bounds__(TPB) dw_tile_kernel(const bf16* __restrict__ in, const float* __restrict__ w,
                                                    const bf16* __restrict__ add, bf16* __restrict__ out, int B,
                                                    int H, int C, int TW, int strips, unsigned long long* stats,
                                                    const BnBwdFuse bnb, const BnApplyIn xbn) {
  static_assert(!XBN || (X2 && !FLIP), "BN-on-load is a forward (bf16x2) mode");
  constexpr int PAD = DIL * (K / 2), KE = DIL * (K - 1) + 1, IH = (DH - 1) * S + KE;
  extern __shared__ float tile[];  // [CPG][IH][IW][8]
  ptx::pdl_wait();
  const int Ho = (H + 2 * PAD - KE) / S + 1;
  const int CPG = TPB / (8 * TW), IW = (TW - 1) * S + KE;
  const int RH = DH * strips;  // output rows of the CTA: `strips` strips of DH rows
  const int tiles_h = (Ho + RH - 1) / RH, tiles_w = (Ho + TW - 1) / TW;
  int t = blockIdx.x;
  const int tw = t % tiles_w;
  t /= tiles_w;
  const int th = t % tiles_h;
  t /= tiles_h;
  const int b = t;
  const int cg0 = blockIdx.y * CPG;  // first channel group of the CTA
  const size_t iplane = (size_t)B * H * H * C, oplane = (size_t)B * Ho * Ho * C;
  __shared__ float xmu[XBN ? XBN_CH : 1], xrs[XBN ? XBN_CH : 1], xg[XBN ? XBN_CH : 1], xb[XBN ? XBN_CH : 1];
  if constexpr (XBN) xbn_stage(xbn, true, cg0 * 8, CPG * 8, C, xmu, xrs, xg, xb);
  const int ch = threadIdx.x % 8, col = (threadIdx.x / 8) % TW, cgi = threadIdx.x / (8 * TW);
  const int c = (cg0 + cgi) * 8 + ch;
  float wr[K][K];
#pragma unroll
  for (int u = 0; u < K; ++u)
#pragma unroll
    for (int v = 0; v < K; ++v)
      wr[u][v] = c < C ? w[c * K * K + (FLIP ? (K - 1 - u) * K + (K - 1 - v) : u * K + v)] : 0.f;
  const int ow = tw * TW + col;
  const bool valid = c < C && ow < Ho;
  // fused sums over the CTA's strips: (sum, sum of squares) of the stored z (X2), or
  // (sum dy', sum dy' xh) (FLIP with bnb)
  const bool fuse_b = !X2 && FLIP && bnb.acc != nullptr;
  float ss = 0.f, sq = 0.f;
  float bmu = 0.f, brs = 0.f, bg = 0.f, bb = 0.f;
  if (fuse_b && valid) {
    bmu = bnb.mean[c];
    brs = bnb.rstd[c];
    bg = bnb.g[c];
    bb = bnb.b[c];
  }
  const float* tb = tile + (cgi * IH * IW + col * S) * 8 + ch;
  const int iw0 = tw * TW * S - PAD;
  for (int st = 0; st < strips; ++st) {
    const int oh0 = th * RH + st * DH;
    if (oh0 >= Ho) break;  // CTA-uniform
    const int ih0 = oh0 * S - PAD;
    __syncthreads();  // the previous strip's halo has been consumed
    // stage the halo: CPG x IH x IW pixels of 8 channels (XBN: y = BN(z) [+ ReLU] on load;
    // the zero padding stays zero)
    for (int i = threadIdx.x; i < CPG * IH * IW; i += TPB) {
      const int cl = i % IW, row = (i / IW) % IH, cg = i / (IW * IH);
      const int ih = ih0 + row, iw = iw0 + cl, c8 = (cg0 + cg) * 8;
      float v[8] = {};
      if (ih >= 0 && ih < H && iw >= 0 && iw < H && c8 < C) {
        const bf16* p = (XBN ? xbn.z : in) + (((size_t)b * H + ih) * H + iw) * C + c8;
        if (X2) load8x2(p, XBN ? xbn.zplane : iplane, v);
        else load8(p, v);
        if constexpr (XBN) xbn_y8<false>(v, xmu, xrs, xg, xb, cg * 8, xbn.relu);
      }
      float4* d = reinterpret_cast<float4*>(tile + i * 8);
      d[0] = make_float4(v[0], v[1], v[2], v[3]);
      d[1] = make_float4(v[4], v[5], v[6], v[7]);
    }
    __syncthreads();
    float acc[DH];
#pragma unroll
    for (int r = 0; r < DH; ++r) acc[r] = 0.f;
#pragma unroll
    for (int ir = 0; ir < IH; ++ir) {
      const float* rowp = tb + ir * IW * 8;
#pragma unroll
      for (int v = 0; v < K; ++v) {
        const float x = rowp[v * DIL * 8];
#pragma unroll
        for (int r = 0; r < DH; ++r) {
          const int tt = ir - r * S;  // = u * DIL (compile-time after unrolling)
          if (tt >= 0 && tt % DIL == 0 && tt / DIL < K) acc[r] = __fmaf_rn(x, wr[tt / DIL][v], acc[r]);
        }
      }
    }
    if (valid) {
      const size_t o0 = (((size_t)b * Ho + oh0) * Ho + ow) * C + c, rstride = (size_t)Ho * C;
      const int nr = min(DH, Ho - oh0);
#pragma unroll
      for (int r = 0; r < DH; ++r) {
        if (r >= nr) break;
        const size_t o = o0 + r * rstride;
        if (X2) {
          const bf16 hi = __float2bfloat16_rn(acc[r]);
          const bf16 lo = __float2bfloat16_rn(acc[r] - __bfloat162float(hi));
          out[o] = hi;
          out[o + oplane] = lo;
          const float v = __bfloat162float(hi) + __bfloat162float(lo);
          ss += v;
          sq = __fmaf_rn(v, v, sq);
        } else {
          const bf16 ob = __float2bfloat16_rn(add ? acc[r] + __bfloat162float(add[o]) : acc[r]);
          out[o] = ob;
          if (fuse_b) {  // bn_bwd_reduce's terms of the stored dy
            float d = __bfloat162float(ob), xh;
            const float zz = __bfloat162float(bnb.z[o]) + __bfloat162float(bnb.z[o + bnb.zplane]);
            bn_bwd_elem(d, zz, bmu, brs, bg, bb, bnb.relu, xh);
            ss += d;
            sq = __fmaf_rn(d, xh, sq);
          }
        }
      }
    }
  }
  unsigned long long* sacc = X2 ? stats : (fuse_b ? bnb.acc : nullptr);
  if (sacc != nullptr) {
    // per channel over the CTA's TW columns, fixed order: xor tree over the 4 columns of a
    // warp (lanes ch + 8 col), then the warps of the channel group in warp order
    __shared__ float wsum[TPB / 32][2][8];
#pragma unroll
    for (int o = 8; o < 32; o <<= 1) {
      ss += __shfl_xor_sync(0xffffffffu, ss, o);
      sq += __shfl_xor_sync(0xffffffffu, sq, o);
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane < 8) {
      wsum[warp][0][lane] = ss;
      wsum[warp][1][lane] = sq;
    }
    __syncthreads();
    const int wpg = TW / 4;  // warps per channel group
    if (threadIdx.x < CPG * 16) {
      const int g = threadIdx.x / 16, which = (threadIdx.x / 8) & 1, chn = threadIdx.x & 7;
      const int cc = (cg0 + g) * 8 + chn;
      float a = 0.f;
      for (int k = 0; k < wpg; ++k) a += wsum[g * wpg + k][which][chn];
      if (cc < C) fix_add(sacc, (which ? C : 0) + cc, sacc + 2 * C, a, X2 ? (which ? FIX_S2 : FIX_S1) : FIX_B);
    }
  }
  if constexpr (XBN) {
    if (last_cta(xbn.ticket)) {  // every CTA has read the input sums: publish, clear
      for (int cc = threadIdx.x; cc < C; cc += TPB) {
        float mu, rs;
        bn_moments(xbn.acc, C, cc, xbn.P, mu, rs);
        xbn.mean[cc] = mu;
        xbn.rstd[cc] = rs;
        xbn.gsnap[cc] = xbn.g[cc];
        xbn.bsnap[cc] = xbn.b[cc];
      }
      __syncthreads();
      for (int e = threadIdx.x; e < 2 * C; e += TPB) xbn.acc[e] = 0ull;
      if (threadIdx.x == 0) *xbn.ticket = 0;
    }
  }
}

// Input gradient of a STRIDE-2 depthwise conv, tiled (replaces round 2's grid-stride gather,
// which took 32 / 75 / 182 us per k = 3 / 5 / 7 launch at configs[1]'s 112x112 inputs):
//   dx[b,ih,iw,c] = sum_{u,v} dz[b,oh,ow,c] w[c,u,v] over oh*2 + u*DIL - PAD = ih,
//   ow*2 + v*DIL - PAD = iw (+ add), PAD = DIL*(K/2).
// A CTA owns DT_H rows x TW columns x CPG channel groups of dx; the dz window they read
// (DT_H/2 + ~K*DIL/2 rows x TW/2 + ~K*DIL/2 columns) is staged in shared memory once.  Row
// parity is compile-time (ih0 is even); the column parity picks the valid v taps, so the
// threads are permuted so that each warp's 4 columns share one parity (no divergence).
// BnBwdFuse: as dw_tile_kernel's FLIP mode (bn_bwd_reduce fused, fixed order per CTA).
constexpr int S2_STRIPS = 4;  // DT_H-row strips per CTA (the weights and the grid's fixed costs amortised over them)

// One thread's DT_H outputs of a strip from the staged dz window (column parity class Q,
// compile-time): with EP = (PAD - (K-1) DIL) & 1, output row r takes tap u iff
// EP + (K-1-u) DIL + r is even, from staged row (EP + (K-1-u) DIL + r) / 2; column tap v iff
// Q + (K-1-v) DIL is even, at staged column cb + (Q + (K-1-v) DIL) / 2.  All offsets but the
// row pitch are compile-time: ~1 FFMA + 1 LDS per tap (the generic gather spent ~15 integer
// instructions per tap).
template <int K, int DIL, int Q>
__device__ __forceinline__ void s2_strip(const float* base, int ow8, const float (&wr)[K][K], float (&acc)[DT_H]) {
  constexpr int PAD = DIL * (K / 2), EP = (PAD - (K - 1) * DIL) & 1;
#pragma unroll
  for (int r = 0; r < DT_H; ++r) {
    float a = 0.f;
#pragma unroll
    for (int u = 0; u < K; ++u) {
      if (((EP + (K - 1 - u) * DIL + r) & 1) != 0) continue;
      const float* row = base + ((EP + (K - 1 - u) * DIL + r) >> 1) * ow8;
#pragma unroll
      for (int v = 0; v < K; ++v) {
        if (((Q + (K - 1 - v) * DIL) & 1) != 0) continue;
        a = __fmaf_rn(row[((Q + (K - 1 - v) * DIL) >> 1) * 8], wr[u][v], a);
      }
    }
    acc[r] = a;
  }
}

template <int K, int DIL>
__global__ void __launch_bounds__(TPB) dw_dgrad_s2_kernel(const bf16* __restrict__ dz, const float* __restrict__ w,
                                                        const bf16* __restrict__ add, bf16* __restrict__ dx, int B,
                                                        int H, int C, int TW, const BnBwdFuse bnb) {
  constexpr int PAD = DIL * (K / 2), KE = DIL * (K - 1) + 1, OH = DT_H / 2 + (KE + 1) / 2 + 1;
  constexpr int RH = DT_H * S2_STRIPS, EP = (PAD - (K - 1) * DIL) & 1;
  extern __shared__ float tile[];  // [CPG][OH][OW][8]
  ptx::pdl_wait();
  const int Ho = (H + 2 * PAD - KE) / 2 + 1;
  const int CPG = TPB / (8 * TW), OW = TW / 2 + (KE + 1) / 2 + 1;
  const int tiles_h = (H + RH - 1) / RH, tiles_w = (H + TW - 1) / TW;
  int t = blockIdx.x;
  const int tw = t % tiles_w;
  t /= tiles_w;
  const int th = t % tiles_h;
  const int b = t / tiles_h;
  const int cg0 = blockIdx.y * CPG;
  const int iw0 = tw * TW;  // even
  const int ow0 = (iw0 + PAD - (K - 1) * DIL) >> 1;  // first dz column the tile reads (floor; may be < 0)
  // thread -> (channel, column, channel group); columns permuted so a warp's 4 share a parity
  const int ch = threadIdx.x % 8, ci = (threadIdx.x / 8) % TW, cgi = threadIdx.x / (8 * TW);
  const int col = (ci & ~7) + 2 * (ci & 3) + ((ci >> 2) & 1);
  const int c = (cg0 + cgi) * 8 + ch;
  float wr[K][K];
#pragma unroll
  for (int u = 0; u < K; ++u)
#pragma unroll
    for (int v = 0; v < K; ++v) wr[u][v] = c < C ? w[c * K * K + u * K + v] : 0.f;
  const int iw = iw0 + col;
  const int cc = EP + col;  // staged column of tap v: (cc + (K-1-v) DIL) / 2
  const float* base = tile + (cgi * OH * OW + (cc >> 1)) * 8 + ch;
  const int ow8 = OW * 8;
  const bool fuse_b = bnb.acc != nullptr;
  const bool valid = c < C && iw < H;
  float ss = 0.f, sq = 0.f, bmu = 0.f, brs = 0.f, bg = 0.f, bb = 0.f;
  if (fuse_b && valid) {
    bmu = bnb.mean[c];
    brs = bnb.rstd[c];
    bg = bnb.g[c];
    bb = bnb.b[c];
  }
  const size_t rstride = (size_t)H * C;
  for (int st = 0; st < S2_STRIPS; ++st) {
    const int ih0 = th * RH + st * DT_H;  // even
    if (ih0 >= H) break;  // CTA-uniform
    const int oh0 = (ih0 + PAD - (K - 1) * DIL) >> 1;  // first dz row the strip reads (floor)
    __syncthreads();  // the previous strip's window has been consumed
    for (int i = threadIdx.x; i < CPG * OH * OW; i += TPB) {
      const int cl = i % OW, row = (i / OW) % OH, cg = i / (OW * OH);
      const int oh = oh0 + row, ow = ow0 + cl, c8 = (cg0 + cg) * 8;
      float v[8] = {};
      if (oh >= 0 && oh < Ho && ow >= 0 && ow < Ho && c8 < C) load8(dz + (((size_t)b * Ho + oh) * Ho + ow) * C + c8, v);
      float4* d = reinterpret_cast<float4*>(tile + i * 8);
      d[0] = make_float4(v[0], v[1], v[2], v[3]);
      d[1] = make_float4(v[4], v[5], v[6], v[7]);
    }
    __syncthreads();
    float acc[DT_H];
    if (cc & 1) s2_strip<K, DIL, 1>(base, ow8, wr, acc);  // warp-uniform
    else s2_strip<K, DIL, 0>(base, ow8, wr, acc);
    if (valid) {
      const size_t o0 = (((size_t)b * H + ih0) * H + iw) * C + c;
      const int nr = min(DT_H, H - ih0);
#pragma unroll
      for (int r = 0; r < DT_H; ++r) {
        if (r >= nr) break;
        const size_t o = o0 + r * rstride;
        const bf16 ob = __float2bfloat16_rn(add ? acc[r] + __bfloat162float(add[o]) : acc[r]);
        dx[o] = ob;
        if (fuse_b) {
          float d = __bfloat162float(ob), xh;
          const float zz = __bfloat162float(bnb.z[o]) + __bfloat162float(bnb.z[o + bnb.zplane]);
          bn_bwd_elem(d, zz, bmu, brs, bg, bb, bnb.relu, xh);
          ss += d;
          sq = __fmaf_rn(d, xh, sq);
        }
      }
    }
  }
  if (fuse_b) {  // per channel: xor tree over the warp's 4 columns, then its warps in warp order
    __shared__ float wsum[TPB / 32][2][8];
#pragma unroll
    for (int o = 8; o < 32; o <<= 1) {
      ss += __shfl_xor_sync(0xffffffffu, ss, o);
      sq += __shfl_xor_sync(0xffffffffu, sq, o);
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane < 8) {
      wsum[warp][0][lane] = ss;
      wsum[warp][1][lane] = sq;
    }
    __syncthreads();
    const int wpg = TW / 4;
    if (threadIdx.x < CPG * 16) {
      const int g = threadIdx.x / 16, which = (threadIdx.x / 8) & 1, chn = threadIdx.x & 7;
      const int c2 = (cg0 + g) * 8 + chn;
      float a = 0.f;
      for (int k = 0; k < wpg; ++k) a += wsum[g * wpg + k][which][chn];
      if (c2 < C) fix_add(bnb.acc, (which ? C : 0) + c2, bnb.acc + 2 * C, a, FIX_B);
    }
  }
}

// Weight gradient partials, tiled like the forward (dw_tile_kernel): CTA (tile column tw,
// part p; channel-group block blockIdx.y) loops over the (image, DT_H-row strip) tiles
// q = p, p + NP, ... < B * tiles_h; per tile it stages the input halo in shared memory and
// thread (ch, col, cg) — output column tw*TW + col, channel c — holds its DT_H values of dz
// in registers and accumulates all K x K taps, reading each staged input once per tile
// (K*K FMAs per DT_H*K*K / (IH*K) reads instead of one load per FMA).  The TW column sums
// are then added in column order and, in 64-bit fixed point, into acc[c][u][v] (the weight's
// layout; fixpoint.cuh: bitwise independent of the CTA order).  The last CTA (ticket) applies
// the SGD WRITE w -= lr * total (w = the master, or the bulk accumulator under BSP) and clears
// acc: one launch instead of partials + a fixed-order summing SGD kernel.
// XBN: x = the hi plane of relu?(BN(z)) recomputed on load from the published mean / rstd
// and the forward's g / b snapshots (BnApplyIn; bn_apply was folded into the forward conv).
template <int K, int S, int DIL, bool XBN = false>
__global__ void __launch_bounds__(TPB) dw_wgrad_kernel(const bf16* __restrict__ dz, const bf16* __restrict__ x,
                                                       unsigned long long* gacc, int* ticket, float* w, float lr,
                                                       int B, int H, int C, int TW, int NP, const BnApplyIn xbn) {
  constexpr int PAD = DIL * (K / 2), KE = DIL * (K - 1) + 1, IH = (DT_H - 1) * S + KE, K2 = K * K;
  extern __shared__ float tile[];  // [CPG][IH][IW][8]; later [TPB][K2] for the column sums
  ptx::pdl_wait();
  const int Ho = (H + 2 * PAD - KE) / S + 1;
  const int CPG = TPB / (8 * TW), IW = (TW - 1) * S + KE;
  const int tiles_h = (Ho + DT_H - 1) / DT_H, tiles_w = (Ho + TW - 1) / TW;
  const int tw = blockIdx.x % tiles_w, p = blockIdx.x / tiles_w;
  const int cg0 = blockIdx.y * CPG;
  const int ch = threadIdx.x % 8, col = (threadIdx.x / 8) % TW, cgi = threadIdx.x / (8 * TW);
  const int c = (cg0 + cgi) * 8 + ch, ow = tw * TW + col;
  __shared__ float xmu[XBN ? XBN_CH : 1], xrs[XBN ? XBN_CH : 1], xg[XBN ? XBN_CH : 1], xb[XBN ? XBN_CH : 1];
  if constexpr (XBN) xbn_stage(xbn, false, cg0 * 8, CPG * 8, C, xmu, xrs, xg, xb);
  float acc[K][K];
#pragma unroll
  for (int u = 0; u < K; ++u)
#pragma unroll
    for (int v = 0; v < K; ++v) acc[u][v] = 0.f;
  for (int q = p; q < B * tiles_h; q += NP) {
    const int b = q / tiles_h, th = q % tiles_h;
    const int ih0 = th * DT_H * S - PAD, iw0 = tw * TW * S - PAD;
    __syncthreads();  // the previous tile has been consumed
    for (int i = threadIdx.x; i < CPG * IH * IW; i += TPB) {
      const int cl = i % IW, row = (i / IW) % IH, cg = i / (IW * IH);
      const int ih = ih0 + row, iw = iw0 + cl, cc = (cg0 + cg) * 8;
      float v[8] = {};
      if (ih >= 0 && ih < H && iw >= 0 && iw < H && cc < C) {
        const size_t o = (((size_t)b * H + ih) * H + iw) * C + cc;
        if constexpr (XBN) {
          load8x2(xbn.z + o, xbn.zplane, v);
          xbn_y8<true>(v, xmu, xrs, xg, xb, cg * 8, xbn.relu);
        } else {
          load8(x + o, v);
        }
      }
      float4* d = reinterpret_cast<float4*>(tile + (size_t)i * 8);
      d[0] = make_float4(v[0], v[1], v[2], v[3]);
      d[1] = make_float4(v[4], v[5], v[6], v[7]);
    }
    float g[DT_H];
#pragma unroll
    for (int r = 0; r < DT_H; ++r) {
      const int oh = th * DT_H + r;
      g[r] = (c < C && ow < Ho && oh < Ho) ? __bfloat162float(dz[(((size_t)b * Ho + oh) * Ho + ow) * C + c]) : 0.f;
    }
    __syncthreads();
    const float* tb = tile + ((size_t)cgi * IH * IW + col * S) * 8 + ch;
#pragma unroll
    for (int ir = 0; ir < IH; ++ir) {
#pragma unroll
      for (int v = 0; v < K; ++v) {
        const float xv = tb[((size_t)ir * IW + v * DIL) * 8];
#pragma unroll
        for (int r = 0; r < DT_H; ++r) {
          const int t = ir - r * S;  // = u * DIL
          if (t >= 0 && t % DIL == 0 && t / DIL < K) acc[t / DIL][v] = __fmaf_rn(g[r], xv, acc[t / DIL][v]);
        }
      }
    }
  }
  __syncthreads();
  float* red = tile;  // [TPB][K2]
#pragma unroll
  for (int u = 0; u < K; ++u)
#pragma unroll
    for (int v = 0; v < K; ++v) red[(size_t)threadIdx.x * K2 + u * K + v] = acc[u][v];
  __syncthreads();
  for (int e = threadIdx.x; e < CPG * 8 * K2; e += TPB) {
    const int tap = e % K2, cc = e / K2, cgl = cc / 8, chl = cc % 8;
    const int cglob = (cg0 + cgl) * 8 + chl;
    if (cglob >= C) continue;
    float sum = 0.f;
    for (int cl = 0; cl < TW; ++cl) sum += red[(size_t)((cgl * TW + cl) * 8 + chl) * K2 + tap];
    fix_add(gacc, cglob * K2 + tap, gacc + (size_t)C * K2, sum, FIX_B);
  }
  if (last_cta(ticket)) {  // every CTA's partial is in: the WRITE, then clear for the next use
    for (int i = threadIdx.x; i < C * K2; i += TPB) {
      w[i] -= lr * (float)fix_get(gacc, i, FIX_B);
      gacc[i] = 0ull;
    }
    if (threadIdx.x == 0) *ticket = 0;
  }
}


// ---------------------------------------------------------------- dense k x k conv: columns
// thread = (output pixel, tap, 8-channel group): one 16-byte hi and lo copy (exact)
__global__ void im2col_x2_kernel(const bf16* __restrict__ x, size_t xplane, int B, int H, int C, int k, int S,
                                 bf16* __restrict__ cols, size_t cplane) {
  ptx::pdl_wait();
  const int Ho = (H - 1) / S + 1, pad = k / 2, G = C / 8, K = k * k * C;
  const size_t items = (size_t)B * Ho * Ho * k * k * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const int g = (int)(it % G);
    const int tap = (int)((it / G) % (k * k));
    const size_t po = it / ((size_t)G * k * k);
    const int ow = (int)(po % Ho), oh = (int)((po / Ho) % Ho), b = (int)(po / ((size_t)Ho * Ho));
    const int ih = oh * S + tap / k - pad, iw = ow * S + tap % k - pad;
    uint4 hi = make_uint4(0u, 0u, 0u, 0u), lo = hi;
    if (ih >= 0 && ih < H && iw >= 0 && iw < H) {
      const size_t o = (((size_t)b * H + ih) * H + iw) * C + 8 * g;
      hi = *reinterpret_cast<const uint4*>(x + o);
      lo = *reinterpret_cast<const uint4*>(x + xplane + o);
    }
    const size_t d = po * K + (size_t)tap * C + 8 * g;
    *reinterpret_cast<uint4*>(cols + d) = hi;
    *reinterpret_cast<uint4*>(cols + cplane + d) = lo;
  }
}

// thread = (input pixel, 8-channel group): the taps that read it, in (u, v) order, fp32
__global__ void col2im_kernel(const float* __restrict__ dcols, int B, int H, int C, int k, int S,
                              const bf16* __restrict__ add, bf16* __restrict__ dx) {
  ptx::pdl_wait();
  const int Ho = (H - 1) / S + 1, pad = k / 2, G = C / 8, K = k * k * C;
  const size_t items = (size_t)B * H * H * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const int g = (int)(it % G);
    const size_t pi = it / G;
    const int iw = (int)(pi % H), ih = (int)((pi / H) % H), b = (int)(pi / ((size_t)H * H));
    float acc[8] = {};
    for (int u = 0; u < k; ++u) {
      const int t = ih + pad - u;
      if (t < 0 || t % S) continue;
      const int oh = t / S;
      if (oh >= Ho) continue;
      for (int v = 0; v < k; ++v) {
        const int q = iw + pad - v;
        if (q < 0 || q % S) continue;
        const int ow = q / S;
        if (ow >= Ho) continue;
        float dv[8];
        load8f(dcols + (((size_t)b * Ho + oh) * Ho + ow) * K + (size_t)(u * k + v) * C + 8 * g, dv);
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] += dv[i];
      }
    }
    if (add) {
      float a[8];
      load8(add + pi * C + 8 * g, a);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += a[i];
    }
    store8(dx + pi * C + 8 * g, acc);
  }
}

// ---------------------------------------------------------------- channel split / merge
// stride-1 block input x [P, 2Ch]: out[:, i] = x[:, 2i] (passed through, ld ldo), xm[:, i] = x[:, 2i+1]
// (all three bf16x2; x and xm planes P*2Ch and P*Ch apart, out's planes oplane apart)
__global__ void chan_split_kernel(const bf16* __restrict__ x, int P, int Ch, bf16* __restrict__ out, int ldo,
                                  size_t oplane, bf16* __restrict__ xm) {
  ptx::pdl_wait();
  const int G = Ch / 8;
  const size_t items = (size_t)P * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const size_t p = it / G;
    const int g = (int)(it % G);
    const size_t xplane = (size_t)P * 2 * Ch, mplane = (size_t)P * Ch;
#pragma unroll
    for (int pl = 0; pl < 2; ++pl) {  // the hi and lo planes move unchanged (exact copies)
      float a[8], b[8], ev[8], od[8];
      load8(x + pl * xplane + p * 2 * Ch + 16 * g, a);
      load8(x + pl * xplane + p * 2 * Ch + 16 * g + 8, b);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        ev[i] = a[2 * i];
        od[i] = a[2 * i + 1];
        ev[4 + i] = b[2 * i];
        od[4 + i] = b[2 * i + 1];
      }
      store8(out + pl * oplane + p * ldo + 8 * g, ev);
      store8(xm + pl * mplane + p * Ch + 8 * g, od);
    }
  }
}

// dx[:, 2i] = dproj[:, i] (ld ldp), dx[:, 2i+1] = dm[:, i]
__global__ void chan_merge_kernel(const bf16* __restrict__ dproj, int ldp, const bf16* __restrict__ dm, int P, int Ch,
                                  bf16* __restrict__ dx) {
  ptx::pdl_wait();
  const int G = Ch / 8;
  const size_t items = (size_t)P * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const size_t p = it / G;
    const int g = (int)(it % G);
    float a[8], b[8], lo[8], hi[8];
    load8(dproj + p * ldp + 8 * g, a);
    load8(dm + p * Ch + 8 * g, b);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      lo[2 * i] = a[i];
      lo[2 * i + 1] = b[i];
      hi[2 * i] = a[4 + i];
      hi[2 * i + 1] = b[4 + i];
    }
    store8(dx + p * 2 * Ch + 16 * g, lo);
    store8(dx + p * 2 * Ch + 16 * g + 8, hi);
  }
}

// ---------------------------------------------------------------- frozen head
// gap[b, c] = (sum_{hw} r[b, hw, c]) / HW, in hw order
__global__ void gap_kernel(const bf16* __restrict__ r, int B, int HW, int C, float* __restrict__ gap) {
  ptx::pdl_wait();
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= B * C) return;
  const int b = i / C, c = i % C;
  float s = 0.f;
  const size_t plane = (size_t)B * HW * C;
  for (int k = 0; k < HW; ++k) {
    const size_t o = ((size_t)b * HW + k) * C + c;
    s += __bfloat162float(r[o]) + __bfloat162float(r[o + plane]);
  }
  gap[i] = s / (float)HW;
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int s = 16; s >= 1; s >>= 1) v += __shfl_xor_sync(0xffffffffu, v, s);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int s = 16; s >= 1; s >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, s));
  return v;
}

// One block per 32 classes: logits[b][j] = sum_c gap[b][c] W_fc[j][c] (fp32, c ascending),
// gap / W tiles of 32 columns staged in shared memory; thread (j, sample group).
// logits[b, j] = sum_c gap[b, c] wf[j, c]: CTA = 8 samples x 32 classes (grid 32 x B/8 on
// configs[1]); c in chunks of FC_KC through shared memory (a few long coalesced load phases
// instead of many short latency-bound ones); each output is one sequential fp32 FMA chain
// over c = 0..C-1 (fixed order, bitwise reproducible).
constexpr int FC_KC = 256;
__global__ void fc_logits_kernel(const float* __restrict__ gap, const float* __restrict__ wf, int B, int C, int ncls,
                                 float* __restrict__ logits) {
  extern __shared__ float fsm[];
  float* ws = fsm;                     // [32][FC_KC + 1]
  float* gs = fsm + 32 * (FC_KC + 1);  // [8][FC_KC]
  ptx::pdl_wait();
  const int jl = threadIdx.x % 32, bl = threadIdx.x / 32, j = blockIdx.x * 32 + jl, b = blockIdx.y * 8 + bl;
  float acc = 0.f;
  for (int c0 = 0; c0 < C; c0 += FC_KC) {
    for (int i = threadIdx.x; i < 32 * FC_KC; i += TPB) {
      const int r = i / FC_KC, c = c0 + i % FC_KC, jj = blockIdx.x * 32 + r;
      ws[r * (FC_KC + 1) + i % FC_KC] = (jj < ncls && c < C) ? wf[(size_t)jj * C + c] : 0.f;
    }
    for (int i = threadIdx.x; i < 8 * FC_KC; i += TPB) {
      const int r = i / FC_KC, c = c0 + i % FC_KC, bb = blockIdx.y * 8 + r;
      gs[i] = (bb < B && c < C) ? gap[(size_t)bb * C + c] : 0.f;
    }
    __syncthreads();
#pragma unroll 8
    for (int cc = 0; cc < FC_KC; ++cc) acc = __fmaf_rn(gs[bl * FC_KC + cc], ws[jl * (FC_KC + 1) + cc], acc);
    __syncthreads();
  }
  if (b < B && j < ncls) logits[(size_t)b * ncls + j] = acc;
}

// One block per sample: softmax cross-entropy of its logits, dlogits = (p - onehot) / B.
__global__ void ce_kernel(const float* __restrict__ logits, const int* __restrict__ labels, int B, int ncls,
                          float* __restrict__ dlogits, float* __restrict__ loss_per) {
  __shared__ float red[TPB / 32];
  __shared__ float bc;
  ptx::pdl_wait();
  const int b = blockIdx.x, warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = TPB / 32;
  const float* lg = logits + (size_t)b * ncls;
  float mx = -INFINITY;
  for (int j = threadIdx.x; j < ncls; j += TPB) mx = fmaxf(mx, lg[j]);
  mx = warp_max(mx);
  if (lane == 0) red[warp] = mx;
  __syncthreads();
  if (threadIdx.x == 0) {
    float m = red[0];
    for (int k = 1; k < nw; ++k) m = fmaxf(m, red[k]);
    bc = m;
  }
  __syncthreads();
  mx = bc;
  float se = 0.f;
  for (int j = threadIdx.x; j < ncls; j += TPB) se += expf(lg[j] - mx);
  se = warp_sum(se);
  __syncthreads();
  if (lane == 0) red[warp] = se;
  __syncthreads();
  if (threadIdx.x == 0) {
    float s = 0.f;
    for (int k = 0; k < nw; ++k) s += red[k];
    bc = mx + logf(s);
  }
  __syncthreads();
  const float lse = bc;
  const int lab = labels[b];
  const bool ok = lab >= 0 && lab < ncls;
  for (int j = threadIdx.x; j < ncls; j += TPB)
    dlogits[(size_t)b * ncls + j] = (expf(lg[j] - lse) - (j == lab ? 1.f : 0.f)) / (float)B;
  if (threadIdx.x == 0) loss_per[b] = ok ? lse - lg[lab] : __int_as_float(0x7fc00000);  // NaN flags a bad label
}

__global__ void ce_mean_kernel(const float* __restrict__ loss_per, int B, float* __restrict__ loss) {
  ptx::pdl_wait();
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    float s = 0.f;
    for (int b = 0; b < B; ++b) s += loss_per[b];
    *loss = s / (float)B;
  }
}

// One block per 32 channels: dgap[b][c] = sum_j dlogits[b][j] W_fc[j][c] (fp32, j ascending).
// dgap[b, c] = sum_j dlogits[b, j] wf[j, c]: CTA = 8 samples x 32 channels (grid C/32 x B/8),
// j in chunks of FC_KC through shared memory; one sequential FMA chain over j per output.
__global__ void fc_dgap_kernel(const float* __restrict__ dlogits, const float* __restrict__ wf, int B, int C, int ncls,
                               float* __restrict__ dgap) {
  extern __shared__ float fsm[];
  float* ws = fsm;                // [FC_KC][32]
  float* ds = fsm + FC_KC * 32;   // [8][FC_KC]
  ptx::pdl_wait();
  const int cl = threadIdx.x % 32, bl = threadIdx.x / 32, c = blockIdx.x * 32 + cl, b = blockIdx.y * 8 + bl;
  float acc = 0.f;
  for (int j0 = 0; j0 < ncls; j0 += FC_KC) {
    for (int i = threadIdx.x; i < FC_KC * 32; i += TPB) {
      const int r = i / 32, cc = blockIdx.x * 32 + i % 32, j = j0 + r;
      ws[i] = (j < ncls && cc < C) ? wf[(size_t)j * C + cc] : 0.f;
    }
    for (int i = threadIdx.x; i < 8 * FC_KC; i += TPB) {
      const int r = i / FC_KC, j = j0 + i % FC_KC, bb = blockIdx.y * 8 + r;
      ds[i] = (bb < B && j < ncls) ? dlogits[(size_t)bb * ncls + j] : 0.f;
    }
    __syncthreads();
#pragma unroll 8
    for (int jj = 0; jj < FC_KC; ++jj) acc = __fmaf_rn(ds[bl * FC_KC + jj], ws[jj * 32 + cl], acc);
    __syncthreads();
  }
  if (b < B && c < C) dgap[(size_t)b * C + c] = acc;
}

// dr[b, hw, c] = dgap[b, c] / HW
__global__ void head_bcast_kernel(const float* __restrict__ dgap, int B, int HW, int C, bf16* __restrict__ dr) {
  ptx::pdl_wait();
  const int G = C / 8;
  const size_t items = (size_t)B * HW * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const size_t p = it / G;
    const int c = (int)(it % G) * 8;
    const int b = (int)(p / HW);
    float v[8];
    load8f(dgap + (size_t)b * C + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = v[i] / (float)HW;
    store8(dr + p * C + c, v);
  }
}

__global__ void synth_labels_kernel(int* __restrict__ labels, int B, int ncls, uint64_t seed) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= B) return;
  uint64_t z = seed * 0x9E3779B97F4A7C15ull + (uint64_t)i + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  z ^= z >> 31;
  labels[i] = (int)(z % (uint64_t)ncls);
}

template <typename Kern>
void set_smem(Kern k, size_t bytes) {
  if (bytes > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
}

__global__ void f2x2_kernel(const float* __restrict__ a, bf16* __restrict__ hi, bf16* __restrict__ lo, size_t n) {
  ptx::pdl_wait();
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    const float v = a[i];
    const bf16 h = __float2bfloat16_rn(v);
    hi[i] = h;
    lo[i] = __float2bfloat16_rn(v - __bfloat162float(h));
  }
}

}  // namespace

// ================================================================ host launchers
void f32_to_bf16x2(cudaStream_t s, const float* w32, bf16* hi, bf16* lo, size_t n) {
  launch_pdl(f2x2_kernel, dim3(grid_for(n)), dim3(TPB), 0, s, w32, hi, lo, n);
  check_launch("f32_to_bf16x2");
}

void spos_stem_conv(cudaStream_t s, const float* x, const float* w, bf16* z, int B, int H, int C0) {
  NP_REQUIRE(C0 % 8 == 0 && H % 2 == 0, NASPIPE_EINVAL, "stem C0=%d H=%d", C0, H);
  const size_t P = (size_t)B * (H / 2) * (H / 2);
  launch_pdl(stem_conv_kernel, dim3(grid_for(P)), dim3(TPB), C0 * 27 * sizeof(float), s, x, w, z, B, H, C0);
  check_launch("stem_conv");
}

// grid of the pixel-strided elementwise kernels: a whole number of waves of the kernel's
// resident CTAs (occ per SM, from the occupancy calculator), so the grid-stride loop gives
// every SM the same work -- a fixed 8 CTAs/SM left a 2/3-full third wave for a 3-CTA/SM
// kernel.  NASPIPE_EW_WAVES (default 1: measured best, 7.15 -> 7.01 ms per configs[1] step) overrides the wave count for tuning.
static int ew_waves() {
  static const int v = [] {  // thread-safe one-time init
    const char* e = getenv("NASPIPE_EW_WAVES");
    return e ? std::max(1, atoi(e)) : 1;
  }();
  return v;
}
// NASPIPE_MAX_CTAS_PER_SM (tuning): cap the resident-CTA count used for the grid sizes below
// resident CTAs per SM of `kern` at `smem` dynamic bytes, cached per (kernel address, smem)
// -- a static per template instantiation was shared by kernels of the same type (e.g. the
// dw_tile_kernel<K> of different K); guarded: engines may be created from
// several host threads
template <typename Kern>
static int occupancy(Kern kern, size_t smem) {
  static std::mutex mu;
  static std::map<std::pair<const void*, size_t>, int> cache;
  static const int cap = [] {
    const char* e = getenv("NASPIPE_MAX_CTAS_PER_SM");
    return e ? std::max(1, atoi(e)) : 0;
  }();
  std::lock_guard<std::mutex> lk(mu);
  const auto key = std::make_pair(reinterpret_cast<const void*>(kern), smem);
  auto it = cache.find(key);
  if (it != cache.end()) return it->second;
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, TPB, smem) != cudaSuccess || n < 1) n = 1;
  n = cap ? std::min(n, cap) : n;
  cache[key] = n;
  return n;
}
// grid-stride kernels over `items` threads of work: capped at NASPIPE_GS_WAVES (default 1:
// measured best, 7.01 -> 6.95 ms per configs[1] step) waves of resident CTAs; 0 = grid_for's
// fixed 16 CTAs/SM
static int gs_waves() {
  static const int v = [] {  // thread-safe one-time init
    const char* e = getenv("NASPIPE_GS_WAVES");
    return e ? std::max(0, atoi(e)) : 1;
  }();
  return v;
}
template <typename Kern>
static int gs_grid(Kern kern, size_t items, size_t smem = 0) {
  if (!gs_waves()) return grid_for(items);
  const int occ = occupancy(kern, smem);
  const size_t g = (items + TPB - 1) / TPB;
  return (int)std::min<size_t>(std::max<size_t>(g, 1), (size_t)num_sms() * occ * gs_waves());
}
// minimum pixels per thread of the BatchNorm elementwise kernels (NASPIPE_EW_MIN_PIX, default
// 1 = one wave whatever the size): every CTA derives all C channels' moments first, so a
// full wave of CTAs over a 7x7 tensor mostly repeats that prologue
static int ew_min_pix() {
  static const int v = [] {
    const char* e = getenv("NASPIPE_EW_MIN_PIX");
    return e ? std::max(1, atoi(e)) : 1;
  }();
  return v;
}
template <typename Kern>
static int ew_grid(Kern kern, int P, int C, int vec = 8) {
  const int occ = occupancy(kern, 0);
  const int lanes = TPB / (C / vec), per = lanes * ew_min_pix();
  return std::max(1, std::min((P + per - 1) / per, num_sms() * occ * ew_waves()));
}

static size_t red_smem(int C, int vec = 8) { return (size_t)(TPB / (C / vec)) * 2 * C * sizeof(float); }
static int red_blocks(int P, int C, int vec = 8, int target = 0) {
  const int r = red_rows(P, C, vec, target);
  return (P + r - 1) / r;
}

// pixels in flight per thread in the BatchNorm apply kernels: NASPIPE_BN_UNROLL (2 or 4)
static int bn_unroll() {
  static const int v = [] {
    const char* e = getenv("NASPIPE_BN_UNROLL");
    return (e && atoi(e) == 2) ? 2 : 4;  // 4 measured best on the final code (6.235 vs 6.28-6.35 ms)
  }();
  return v;
}

void bn_stats(cudaStream_t s, const bf16* z, int P, int C, unsigned long long* acc) {
  NP_REQUIRE(C % 8 == 0 && C / 8 <= TPB, NASPIPE_EINVAL, "bn_stats C=%d", C);
  const size_t sm = red_smem(C);
  set_smem(bn_stats_kernel, sm);
  launch_pdl(bn_stats_kernel, dim3(red_blocks(P, C)), dim3(TPB), sm, s, z, P, C, red_rows(P, C), acc);
  check_launch("bn_stats");
}

void bn_apply(cudaStream_t s, const bf16* z, int P, int C, unsigned long long* acc, int* ticket, float* mean,
              float* rstd, const float* g, const float* b, int relu, bf16* y, int ldy, size_t yplane,
              unsigned long long* clear, int clear_n) {
  NP_REQUIRE(C % 8 == 0 && C / 8 <= TPB, NASPIPE_EINVAL, "bn_apply C=%d", C);
  if (bn_unroll() == 4)
    launch_pdl(bn_apply_kernel<4>, dim3(ew_grid(bn_apply_kernel<4>, P, C)), dim3(TPB), 0, s, z, P, C, acc, ticket, mean,
               rstd, g, b, relu, y, ldy, yplane, clear, clear_n);
  else
    launch_pdl(bn_apply_kernel<2>, dim3(ew_grid(bn_apply_kernel<2>, P, C)), dim3(TPB), 0, s, z, P, C, acc, ticket, mean,
               rstd, g, b, relu, y, ldy, yplane, clear, clear_n);
  check_launch("bn_apply");
}

void bn_bwd_reduce(cudaStream_t s, const bf16* dy, int lddy, const bf16* z, int P, int C, const float* mean,
                   const float* rstd, const float* g, const float* b, int relu, unsigned long long* acc) {
  NP_REQUIRE(C % 8 == 0 && C / BV <= TPB, NASPIPE_EINVAL, "bn_bwd C=%d", C);
  const size_t sm = red_smem(C, BV);
  // rows in flight per lane: NASPIPE_BNR_UNROLL (4 or 8; the sums are bitwise the same)
  static const int ur = [] {
    const char* e = getenv("NASPIPE_BNR_UNROLL");
    return (e && atoi(e) == 8) ? 8 : 4;
  }();
  auto kern = ur == 8 ? bn_bwd_reduce_kernel<8> : bn_bwd_reduce_kernel<4>;
  set_smem(kern, sm);
  // one wave of resident CTAs (the fixed-point totals do not depend on the row blocking's
  // summation order only through the partials, which are a function of (P, C) and this
  // occupancy-derived target, itself fixed per build and device)
  const int target = num_sms() * occupancy(bn_bwd_reduce_kernel<4>, sm);
  launch_pdl(kern, dim3(red_blocks(P, C, BV, target)), dim3(TPB), sm, s, dy, lddy, z, P, C, mean, rstd, g, b, relu,
             red_rows(P, C, BV, target), acc);
  check_launch("bn_bwd_reduce");
}

void bn_bwd_apply(cudaStream_t s, const bf16* dy, int lddy, const bf16* z, int P, int C, const float* mean,
                  const float* rstd, const float* g, const float* b, float* gu, float* bu, float lr, int update,
                  unsigned long long* acc, int* ticket, int relu, bf16* dz, const BnWrite& prev) {
  NP_REQUIRE(C % 8 == 0 && C / BV <= TPB, NASPIPE_EINVAL, "bn_bwd_apply C=%d", C);
  if (bn_unroll() == 4)
    launch_pdl(bn_bwd_apply_kernel<4>, dim3(ew_grid(bn_bwd_apply_kernel<4>, P, C, BV)), dim3(TPB), 0, s, dy, lddy, z, P,
               C, mean, rstd, g, b, gu, bu, lr, update, acc, ticket, relu, dz, prev);
  else
    launch_pdl(bn_bwd_apply_kernel<2>, dim3(ew_grid(bn_bwd_apply_kernel<2>, P, C, BV)), dim3(TPB), 0, s, dy, lddy, z, P,
               C, mean, rstd, g, b, gu, bu, lr, update, acc, ticket, relu, dz, prev);
  check_launch("bn_bwd_apply");
}

void bn_write_flush(cudaStream_t s, const BnWrite& w) {
  if (w.acc == nullptr) return;
  launch_pdl(bn_write_kernel, dim3(1), dim3(TPB), 0, s, w);
  check_launch("bn_write_flush");
}

bool bn_fix_overflow(const unsigned long long* acc, int C) {
  unsigned long long v = 0;
  cudaMemcpy(&v, acc + 2 * (size_t)C, sizeof v, cudaMemcpyDeviceToHost);
  return v != 0;
}

// (kernel size, dilation) -> constexpr KK, DD
#define DW_DISPATCH(K, D, EXPR)                                                        \
  switch ((K) * 4 + (D)) {                                                             \
    case 13: { constexpr int KK = 3, DD = 1; EXPR; break; }                            \
    case 21: { constexpr int KK = 5, DD = 1; EXPR; break; }                            \
    case 29: { constexpr int KK = 7, DD = 1; EXPR; break; }                            \
    case 14: { constexpr int KK = 3, DD = 2; EXPR; break; }                            \
    case 22: { constexpr int KK = 5, DD = 2; EXPR; break; }                            \
    case 30: { constexpr int KK = 7, DD = 2; EXPR; break; }                            \
    default: NP_REQUIRE(false, NASPIPE_EINVAL, "depthwise kernel %d dilation %d", K, D); \
  }

// DT_H-row strips per depthwise CTA: NASPIPE_DW_STRIPS (1 / 2 / 4; default 0 = by grid size)
static int dw_strips() {
  static const int v = [] {
    const char* e = getenv("NASPIPE_DW_STRIPS");
    return e ? std::max(0, std::min(4, atoi(e))) : 0;
  }();
  return v;
}

// tile width: the smallest of 8 / 16 / 32 columns covering min(Ho, 32)
// NASPIPE_DW_TW (8 / 16 / 32; 0 = by size): tile width of the depthwise kernels.  A CTA covers
// TW columns x (256 / (8 TW)) groups of 8 channels, so narrower tiles read more of each
// pixel's channels (whole 32-byte sectors) at the cost of more halo columns.
static int dw_tw_knob() {
  static const int v = [] {
    const char* e = getenv("NASPIPE_DW_TW");
    const int t = e ? atoi(e) : 0;
    return (t == 8 || t == 16 || t == 32) ? t : 0;
  }();
  return v;
}
// default: 8 columns up to Ho = 8, else 16 (measured on configs[1]: 16-wide tiles 6.284 ms
// per step, 32-wide (for Ho > 16) 6.322, 8-wide 6.356; profiles/r2_ab2/README.md)
static int dw_tw(int Ho) {
  const int t = Ho <= 8 ? 8 : 16;
  return dw_tw_knob() ? std::min(dw_tw_knob(), Ho <= 8 ? 8 : (Ho <= 16 ? 16 : 32)) : t;
}

// rows per depthwise strip of dw_tile: NASPIPE_DW_DH (8 or 16; default 8)
static int dw_dh() {
  static const int v = [] {
    const char* e = getenv("NASPIPE_DW_DH");
    return (e && atoi(e) == 16) ? 16 : 8;
  }();
  return v;
}

template <int K, int S, int DIL, bool X2, bool FLIP, bool XBN, int DH>
static void dw_tile_dh(cudaStream_t s, const bf16* in, const float* w, const bf16* add, bf16* out, int B, int H, int C,
                       unsigned long long* stats, const BnBwdFuse& bnb, const BnApplyIn& xbn) {
  constexpr int KE = DIL * (K - 1) + 1;
  const int Ho = (H - 1) / S + 1, TW = dw_tw(Ho), CPG = TPB / (8 * TW);
  const int IH = (DH - 1) * S + KE, IW = (TW - 1) * S + KE;
  const size_t sm = (size_t)CPG * IH * IW * 8 * sizeof(float);
  auto kern = dw_tile_kernel<K, S, DIL, X2, FLIP, XBN, DH>;
  set_smem(kern, sm);
  // strips of DH rows per CTA: as many (<= 4) as keep >= 2 waves of resident CTAs (the
  // weights, the halo setup and the reductions amortised over more outputs per CTA)
  const int tiles_w = (Ho + TW - 1) / TW, gy = (C / 8 + CPG - 1) / CPG, rows = (Ho + DH - 1) / DH;
  int strips = dw_strips();
  if (strips <= 0) {
    const long wave = (long)num_sms() * occupancy(kern, sm);
    strips = 1;
    while (strips < 4 && (long)B * ((rows + 2 * strips - 1) / (2 * strips)) * tiles_w * gy >= 2 * wave) strips *= 2;
  }
  const int gx = B * ((Ho + DH * strips - 1) / (DH * strips)) * tiles_w;
  launch_pdl(kern, dim3(gx, gy), dim3(TPB), sm, s, in, w, add, out, B, H, C, TW, strips, stats, bnb, xbn);
}

template <int K, int S, int DIL, bool X2, bool FLIP, bool XBN = false>
static void dw_tile(cudaStream_t s, const bf16* in, const float* w, const bf16* add, bf16* out, int B, int H, int C,
                    unsigned long long* stats = nullptr, const BnBwdFuse& bnb = BnBwdFuse(),
                    const BnApplyIn& xbn = BnApplyIn()) {
  if (dw_dh() == 16) dw_tile_dh<K, S, DIL, X2, FLIP, XBN, 16>(s, in, w, add, out, B, H, C, stats, bnb, xbn);
  else dw_tile_dh<K, S, DIL, X2, FLIP, XBN, DT_H>(s, in, w, add, out, B, H, C, stats, bnb, xbn);
}

void dw_fwd(cudaStream_t s, const bf16* x, const float* w, bf16* z, int B, int H, int C, int k, int S, int dil,
            unsigned long long* stats) {
  NP_REQUIRE(C % 8 == 0 && (S == 1 || S == 2), NASPIPE_EINVAL, "dw_fwd C=%d S=%d", C, S);
  if (S == 1) { DW_DISPATCH(k, dil, (dw_tile<KK, 1, DD, true, false>(s, x, w, nullptr, z, B, H, C, stats))); }
  else { DW_DISPATCH(k, dil, (dw_tile<KK, 2, DD, true, false>(s, x, w, nullptr, z, B, H, C, stats))); }
  check_launch("dw_fwd");
}

void dw_fwd_bn(cudaStream_t s, const BnApplyIn& xin, const float* w, bf16* z, int B, int H, int C, int k, int S,
               int dil, unsigned long long* stats) {
  NP_REQUIRE(C % 8 == 0 && (S == 1 || S == 2) && xin.P == B * H * H && xin.acc && xin.ticket && xin.mean &&
                 xin.gsnap && stats != xin.acc,
             NASPIPE_EINVAL, "dw_fwd_bn C=%d S=%d P=%d", C, S, xin.P);
  if (S == 1) { DW_DISPATCH(k, dil, (dw_tile<KK, 1, DD, true, false, true>(s, nullptr, w, nullptr, z, B, H, C, stats, BnBwdFuse(), xin))); }
  else { DW_DISPATCH(k, dil, (dw_tile<KK, 2, DD, true, false, true>(s, nullptr, w, nullptr, z, B, H, C, stats, BnBwdFuse(), xin))); }
  check_launch("dw_fwd_bn");
}

template <int K, int DIL>
static void dw_dgrad_s2(cudaStream_t s, const bf16* dz, const float* w, const bf16* add, bf16* dx, int B, int H, int C,
                        const BnBwdFuse& bnb) {
  constexpr int KE = DIL * (K - 1) + 1, OH = DT_H / 2 + (KE + 1) / 2 + 1;
  const int TW = dw_tw(H), CPG = TPB / (8 * TW);
  const int RH = DT_H * S2_STRIPS;
  const int gx = B * ((H + RH - 1) / RH) * ((H + TW - 1) / TW), gy = (C / 8 + CPG - 1) / CPG;
  const size_t sm = (size_t)CPG * OH * (TW / 2 + (KE + 1) / 2 + 1) * 8 * sizeof(float);
  set_smem(dw_dgrad_s2_kernel<K, DIL>, sm);
  launch_pdl(dw_dgrad_s2_kernel<K, DIL>, dim3(gx, gy), dim3(TPB), sm, s, dz, w, add, dx, B, H, C, TW, bnb);
}

void dw_dgrad(cudaStream_t s, const bf16* dz, const float* w, const bf16* add, bf16* dx, int B, int H, int C, int k,
              int S, int dil, const BnBwdFuse& bnb) {
  NP_REQUIRE(C % 8 == 0 && (S == 1 || S == 2), NASPIPE_EINVAL, "dw_dgrad C=%d S=%d", C, S);
  if (S == 1) {  // the input gradient of a stride-1 conv is the correlation with the flipped kernel
    DW_DISPATCH(k, dil, (dw_tile<KK, 1, DD, false, true>(s, dz, w, add, dx, B, H, C, nullptr, bnb)));
  } else {
    DW_DISPATCH(k, dil, (dw_dgrad_s2<KK, DD>(s, dz, w, add, dx, B, H, C, bnb)));
  }
  check_launch("dw_dgrad");
}

// weight-gradient grid: tiles_w tile columns x NP parts x channel-group blocks, about
// dw_red_ctas() CTAs; partial blocks = tiles_w * NP (a function of the shape only).
static void dw_wgrad_grid(int B, int H, int C, int k, int S, int& TW, int& NP, int& gy, int& tiles_w) {
  const int Ho = (H - 1) / S + 1;
  TW = dw_tw(Ho);
  const int CPG = TPB / (8 * TW);
  tiles_w = (Ho + TW - 1) / TW;
  gy = (C / 8 + CPG - 1) / CPG;
  const int tiles = B * ((Ho + DT_H - 1) / DT_H);
  NP = std::max(1, std::min(tiles, dw_red_ctas() / std::max(1, tiles_w * gy)));
  (void)k;
}
int dw_wgrad_blocks(int B, int H, int C, int k, int S) {  // grid size (diagnostics)
  int TW, NP, gy, tw;
  dw_wgrad_grid(B, H, C, k, S, TW, NP, gy, tw);
  return tw * NP;
}

void dw_wgrad_sgd(cudaStream_t s, const bf16* dz, const bf16* x, unsigned long long* acc, int* ticket, float* w,
                  float lr, int B, int H, int C, int k, int S, int dil, const BnApplyIn* xin) {
  NP_REQUIRE(C % 8 == 0 && C / 8 <= TPB, NASPIPE_EINVAL, "dw_wgrad C=%d", C);
  NP_REQUIRE(S == 1 || S == 2, NASPIPE_EINVAL, "dw_wgrad stride %d", S);
  int TW, NP, gy, tiles_w;
  dw_wgrad_grid(B, H, C, k, S, TW, NP, gy, tiles_w);
  const int CPG = TPB / (8 * TW);
  auto smem = [&](int K, int D) {
    const int KE = D * (K - 1) + 1, IH = (DT_H - 1) * S + KE, IW = (TW - 1) * S + KE;
    return std::max((size_t)CPG * IH * IW * 8, (size_t)TPB * K * K) * sizeof(float);
  };
  const dim3 grid(tiles_w * NP, gy);
  const BnApplyIn xb = xin ? *xin : BnApplyIn();
#define DW_WG1(KK, SS, DD, XB)                                                                                     \
  {                                                                                                              \
    set_smem(dw_wgrad_kernel<KK, SS, DD, XB>, smem(KK, DD));                                                     \
    launch_pdl(dw_wgrad_kernel<KK, SS, DD, XB>, grid, dim3(TPB), smem(KK, DD), s, dz, x, acc, ticket, w, lr, B, H, C, \
               TW, NP, xb);                                                                                      \
  }
#define DW_WG(KK, SS, DD) \
  if (xin) DW_WG1(KK, SS, DD, true) else DW_WG1(KK, SS, DD, false)
  if (S == 1) {
    DW_DISPATCH(k, dil, DW_WG(KK, 1, DD));
  } else {
    DW_DISPATCH(k, dil, DW_WG(KK, 2, DD));
  }
#undef DW_WG
#undef DW_WG1
  check_launch("dw_wgrad");
}

void im2col_x2(cudaStream_t s, const bf16* x, size_t xplane, int B, int H, int C, int k, int S, bf16* cols,
               size_t cplane) {
  NP_REQUIRE(C % 8 == 0 && (S == 1 || S == 2) && (k % 2) == 1, NASPIPE_EINVAL, "im2col C=%d k=%d S=%d", C, k, S);
  const int Ho = (H - 1) / S + 1;
  const size_t items = (size_t)B * Ho * Ho * k * k * (C / 8);
  launch_pdl(im2col_x2_kernel, dim3(gs_grid(im2col_x2_kernel, items)), dim3(TPB), 0, s, x, xplane, B, H, C, k, S, cols,
             cplane);
  check_launch("im2col_x2");
}

void col2im(cudaStream_t s, const float* dcols, int B, int H, int C, int k, int S, const bf16* add, bf16* dx) {
  NP_REQUIRE(C % 8 == 0 && (S == 1 || S == 2) && (k % 2) == 1, NASPIPE_EINVAL, "col2im C=%d k=%d S=%d", C, k, S);
  const size_t items = (size_t)B * H * H * (C / 8);
  launch_pdl(col2im_kernel, dim3(gs_grid(col2im_kernel, items)), dim3(TPB), 0, s, dcols, B, H, C, k, S, add, dx);
  check_launch("col2im");
}

void chan_split(cudaStream_t s, const bf16* x, int P, int Ch, bf16* out, int ldo, size_t oplane, bf16* xm) {
  launch_pdl(chan_split_kernel, dim3(gs_grid(chan_split_kernel, (size_t)P * (Ch / 8))), dim3(TPB), 0, s, x, P, Ch, out, ldo, oplane,
             xm);
  check_launch("chan_split");
}

void chan_merge(cudaStream_t s, const bf16* dproj, int ldp, const bf16* dm, int P, int Ch, bf16* dx) {
  launch_pdl(chan_merge_kernel, dim3(gs_grid(chan_merge_kernel, (size_t)P * (Ch / 8))), dim3(TPB), 0, s, dproj, ldp, dm, P, Ch, dx);
  check_launch("chan_merge");
}

void gap_pool(cudaStream_t s, const bf16* r, int B, int HW, int C, float* gap) {
  launch_pdl(gap_kernel, dim3((B * C + TPB - 1) / TPB), dim3(TPB), 0, s, r, B, HW, C, gap);
  check_launch("gap");
}

void fc_ce(cudaStream_t s, const float* gap, const float* wf, const int* labels, int B, int C, int ncls,
           float* logits, float* dlogits, float* loss_per) {
  const size_t sm = (32 * (FC_KC + 1) + 8 * FC_KC) * sizeof(float);
  set_smem(fc_logits_kernel, sm);
  launch_pdl(fc_logits_kernel, dim3((ncls + 31) / 32, (B + 7) / 8), dim3(TPB), sm, s, gap, wf, B, C, ncls, logits);
  launch_pdl(ce_kernel, dim3(B), dim3(TPB), 0, s, logits, labels, B, ncls, dlogits, loss_per);
  check_launch("fc_ce");
}

void ce_mean(cudaStream_t s, const float* loss_per, int B, float* loss) {
  launch_pdl(ce_mean_kernel, dim3(1), dim3(32), 0, s, loss_per, B, loss);
  check_launch("ce_mean");
}

void fc_dgap(cudaStream_t s, const float* dlogits, const float* wf, int B, int C, int ncls, float* dgap) {
  const size_t sm = (FC_KC * 32 + 8 * FC_KC) * sizeof(float);
  set_smem(fc_dgap_kernel, sm);
  launch_pdl(fc_dgap_kernel, dim3((C + 31) / 32, (B + 7) / 8), dim3(TPB), sm, s, dlogits, wf, B, C, ncls, dgap);
  check_launch("fc_dgap");
}

void head_bcast(cudaStream_t s, const float* dgap, int B, int HW, int C, bf16* dr) {
  launch_pdl(head_bcast_kernel, dim3(grid_for((size_t)B * HW * (C / 8))), dim3(TPB), 0, s, dgap, B, HW, C, dr);
  check_launch("head_bcast");
}

void synth_labels(cudaStream_t s, int* labels, int B, int ncls, uint64_t seed) {
  synth_labels_kernel<<<(B + 127) / 128, 128, 0, s>>>(labels, B, ncls, seed);
  check_launch("synth_labels");
}

}  // namespace naspipe
