// Non-causal multi-head attention for S <= 128 (reading A17), the mma.sync kernels used for
// the shapes the tcgen05 kernels (attention_tc.cu: S = 128, head dim 64 / 128) do not cover
// (NASPIPE_ATTN_MMA_SYNC=1 forces these everywhere): one CTA per (batch, head)
// holds the whole S x S score tile, so forward and backward need no atomics and are
// bitwise deterministic.  Tensor-core math via mma.sync m16n8k16 (bf16 in, fp32 acc);
// each of the 8 warps owns 16 query rows (forward, dQ) and 16 key rows (dK, dV).
// Attention is ~2.5% of the transformer block's FLOPs; the GEMMs carry the
// tcgen05 path.
#include "common.h"
#include "kernels.h"
#include "launch.h"
#include "ptx.cuh"

namespace naspipe {
namespace {

constexpr int SMAX = 128;
constexpr int NWARP = 8;

template <int HD>
struct AttnCfg {
  static constexpr int LDH = HD + 8;       // padded row (bf16) -> conflict-free ldmatrix
  static constexpr int LDS = SMAX + 8;
};

// cooperative asynchronous copy (cp.async, 16 B per request, all requests in flight) of S
// rows x HD cols (bf16) from global (row pitch ld) into smem (pitch LDH); completes at
// cp_async_wait_all() + __syncthreads()
template <int HD>
__device__ __forceinline__ void load_tile(bf16* dst, const bf16* src, int S, int ld) {
  constexpr int CH = HD / 8;  // 16-byte chunks per row
  for (int i = threadIdx.x; i < S * CH; i += blockDim.x) {
    const int r = i / CH, c = i % CH;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(
                     ptx::smem_u32(dst + r * AttnCfg<HD>::LDH + c * 8)),
                 "l"(src + (size_t)r * ld + c * 8)
                 : "memory");
  }
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
}

// A fragment (16x16) at rows r0, cols k0 of a row-major smem tile with pitch ld
__device__ __forceinline__ void lds_a(const bf16* base, int ld, int r0, int k0, uint32_t (&a)[4]) {
  const int lane = threadIdx.x & 31, mi = lane >> 3;
  const bf16* p = base + (r0 + (mi & 1) * 8 + (lane & 7)) * ld + k0 + (mi >> 1) * 8;
  ptx::ldsm_x4(ptx::smem_u32(p), a[0], a[1], a[2], a[3]);
}
// A fragment of X^T (16x16): rows (m) = columns m0.. of X, cols (k) = rows k0.. of X
__device__ __forceinline__ void lds_a_t(const bf16* base, int ld, int m0, int k0, uint32_t (&a)[4]) {
  const int lane = threadIdx.x & 31, mi = lane >> 3;
  const bf16* p = base + (k0 + (mi >> 1) * 8 + (lane & 7)) * ld + m0 + (mi & 1) * 8;
  ptx::ldsm_x4_t(ptx::smem_u32(p), a[0], a[1], a[2], a[3]);
}
// B fragments for two n-blocks (n0, n0+8) at k-block k0 where B[k][n] = X[n][k] (X row-major,
// k contiguous): b[0],b[1] -> n-block n0; b[2],b[3] -> n-block n0+8
__device__ __forceinline__ void lds_b_nk(const bf16* base, int ld, int n0, int k0, uint32_t (&b)[4]) {
  const int lane = threadIdx.x & 31, mi = lane >> 3;
  const bf16* p = base + (n0 + (mi >> 1) * 8 + (lane & 7)) * ld + k0 + (mi & 1) * 8;
  ptx::ldsm_x4(ptx::smem_u32(p), b[0], b[1], b[2], b[3]);
}
// B fragments where B[k][n] = X[k][n] (X row-major, n contiguous)
__device__ __forceinline__ void lds_b_kn(const bf16* base, int ld, int k0, int n0, uint32_t (&b)[4]) {
  const int lane = threadIdx.x & 31, mi = lane >> 3;
  const bf16* p = base + (k0 + (mi & 1) * 8 + (lane & 7)) * ld + n0 + (mi >> 1) * 8;
  ptx::ldsm_x4_t(ptx::smem_u32(p), b[0], b[1], b[2], b[3]);
}

// S = Q K^T for this warp's 16 rows: acc[nb][4] for key n-blocks nb < S/8
template <int HD>
__device__ __forceinline__ void scores(const bf16* Qs, const bf16* Ks, int r0, int S, float (&acc)[SMAX / 8][4]) {
  constexpr int LD = AttnCfg<HD>::LDH;
#pragma unroll
  for (int nb = 0; nb < SMAX / 8; ++nb) acc[nb][0] = acc[nb][1] = acc[nb][2] = acc[nb][3] = 0.f;
#pragma unroll
  for (int kk = 0; kk < HD / 16; ++kk) {
    uint32_t a[4];
    lds_a(Qs, LD, r0, kk * 16, a);
#pragma unroll
    for (int np = 0; np < SMAX / 16; ++np) {
      if (np * 16 < S) {
        uint32_t b[4];
        lds_b_nk(Ks, LD, np * 16, kk * 16, b);
        ptx::mma_bf16_16816(acc[2 * np], a, b[0], b[1]);
        ptx::mma_bf16_16816(acc[2 * np + 1], a, b[2], b[3]);
      }
    }
  }
}

template <int HD>
__global__ void __launch_bounds__(256) attn_fwd_kernel(const bf16* __restrict__ qkv, bf16* __restrict__ o,
                                                       float* __restrict__ lse, int S, int d, int h) {
  using C = AttnCfg<HD>;
  extern __shared__ __align__(16) uint8_t sm[];
  bf16* Qs = reinterpret_cast<bf16*>(sm);
  bf16* Ks = Qs + SMAX * C::LDH;
  bf16* Vs = Ks + SMAX * C::LDH;
  const int bh = blockIdx.x, b = bh / h, hh = bh % h;
  const size_t ld = 3 * (size_t)d;
  const bf16* base = qkv + (size_t)b * S * ld + hh * HD;
  ptx::pdl_wait();
  load_tile<HD>(Qs, base, S, (int)ld);
  load_tile<HD>(Ks, base + d, S, (int)ld);
  load_tile<HD>(Vs, base + 2 * d, S, (int)ld);
  cp_async_wait_all();
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int r0 = warp * 16;
  if (r0 >= S) return;
  const float scale_log2 = 1.4426950408889634f / sqrtf((float)HD);
  float acc[SMAX / 8][4];
  scores<HD>(Qs, Ks, r0, S, acc);
  float mx0 = -INFINITY, mx1 = -INFINITY;
#pragma unroll
  for (int nb = 0; nb < SMAX / 8; ++nb)
    if (nb * 8 < S) {
      mx0 = fmaxf(mx0, fmaxf(acc[nb][0], acc[nb][1]));
      mx1 = fmaxf(mx1, fmaxf(acc[nb][2], acc[nb][3]));
    }
#pragma unroll
  for (int s = 1; s <= 2; s <<= 1) {
    mx0 = fmaxf(mx0, __shfl_xor_sync(0xffffffffu, mx0, s));
    mx1 = fmaxf(mx1, __shfl_xor_sync(0xffffffffu, mx1, s));
  }
  float sum0 = 0.f, sum1 = 0.f;
#pragma unroll
  for (int nb = 0; nb < SMAX / 8; ++nb)
    if (nb * 8 < S) {
      acc[nb][0] = exp2f((acc[nb][0] - mx0) * scale_log2);
      acc[nb][1] = exp2f((acc[nb][1] - mx0) * scale_log2);
      acc[nb][2] = exp2f((acc[nb][2] - mx1) * scale_log2);
      acc[nb][3] = exp2f((acc[nb][3] - mx1) * scale_log2);
      sum0 += acc[nb][0] + acc[nb][1];
      sum1 += acc[nb][2] + acc[nb][3];
    }
#pragma unroll
  for (int s = 1; s <= 2; s <<= 1) {
    sum0 += __shfl_xor_sync(0xffffffffu, sum0, s);
    sum1 += __shfl_xor_sync(0xffffffffu, sum1, s);
  }
  float oacc[HD / 8][4];
#pragma unroll
  for (int nb = 0; nb < HD / 8; ++nb) oacc[nb][0] = oacc[nb][1] = oacc[nb][2] = oacc[nb][3] = 0.f;
#pragma unroll
  for (int kk = 0; kk < SMAX / 16; ++kk) {
    if (kk * 16 < S) {
      uint32_t a[4];
      a[0] = ptx::pack_bf16(acc[2 * kk][0], acc[2 * kk][1]);
      a[1] = ptx::pack_bf16(acc[2 * kk][2], acc[2 * kk][3]);
      a[2] = ptx::pack_bf16(acc[2 * kk + 1][0], acc[2 * kk + 1][1]);
      a[3] = ptx::pack_bf16(acc[2 * kk + 1][2], acc[2 * kk + 1][3]);
#pragma unroll
      for (int np = 0; np < HD / 16; ++np) {
        uint32_t bb[4];
        lds_b_kn(Vs, C::LDH, kk * 16, np * 16, bb);
        ptx::mma_bf16_16816(oacc[2 * np], a, bb[0], bb[1]);
        ptx::mma_bf16_16816(oacc[2 * np + 1], a, bb[2], bb[3]);
      }
    }
  }
  const float inv0 = 1.f / sum0, inv1 = 1.f / sum1;
  bf16* orow0 = o + ((size_t)b * S + r0 + g) * d + hh * HD;
  bf16* orow1 = orow0 + 8 * (size_t)d;
#pragma unroll
  for (int nb = 0; nb < HD / 8; ++nb) {
    *reinterpret_cast<uint32_t*>(orow0 + nb * 8 + 2 * t) = ptx::pack_bf16(oacc[nb][0] * inv0, oacc[nb][1] * inv0);
    *reinterpret_cast<uint32_t*>(orow1 + nb * 8 + 2 * t) = ptx::pack_bf16(oacc[nb][2] * inv1, oacc[nb][3] * inv1);
  }
  if (t == 0) {
    const float ln2 = 0.6931471805599453f;
    float* l = lse + (size_t)bh * S + r0 + g;
    l[0] = mx0 * scale_log2 * ln2 + logf(sum0);
    l[8] = mx1 * scale_log2 * ln2 + logf(sum1);
  }
}

// Backward.  HD <= 64 keeps ONE S x S bf16 buffer (P, then dS) so that two CTAs fit per SM
// (108 KB of shared memory instead of 143 KB; the configs[2] h=16 blocks launch B*h = 512
// CTAs): P is written, dV = P^T dO is formed, then dS (kept in registers) replaces it and
// dK = dS^T Q follows.  HD > 64 keeps both buffers (one CTA per SM either way).
template <int HD>
__global__ void __launch_bounds__(256, (HD <= 64 ? 2 : 1)) attn_bwd_kernel(const bf16* __restrict__ qkv, const bf16* __restrict__ o,
                                                       const float* __restrict__ lse, const bf16* __restrict__ dout,
                                                       bf16* __restrict__ dqkv, int S, int d, int h) {
  using C = AttnCfg<HD>;
  constexpr bool ONEBUF = HD <= 64;
  extern __shared__ __align__(16) uint8_t sm[];
  bf16* Qs = reinterpret_cast<bf16*>(sm);
  bf16* Ks = Qs + SMAX * C::LDH;
  bf16* Vs = Ks + SMAX * C::LDH;
  bf16* dOs = Vs + SMAX * C::LDH;
  bf16* Ps = dOs + SMAX * C::LDH;
  bf16* dSs = ONEBUF ? Ps : Ps + SMAX * C::LDS;
  float* Di = reinterpret_cast<float*>(Ps + (ONEBUF ? 1 : 2) * SMAX * C::LDS);
  const int bh = blockIdx.x, b = bh / h, hh = bh % h;
  const size_t ld = 3 * (size_t)d;
  const bf16* base = qkv + (size_t)b * S * ld + hh * HD;
  ptx::pdl_wait();
  load_tile<HD>(Qs, base, S, (int)ld);
  load_tile<HD>(Ks, base + d, S, (int)ld);
  load_tile<HD>(Vs, base + 2 * d, S, (int)ld);
  load_tile<HD>(dOs, dout + (size_t)b * S * d + hh * HD, S, d);
  bf16* Os = Ps;  // O is staged in the P buffer (free until phase 1 writes P)
  static_assert(C::LDS >= C::LDH, "O staging must fit the P rows");
  {
    constexpr int CH = HD / 8;
    const bf16* osrc = o + (size_t)b * S * d + hh * HD;
    for (int i = threadIdx.x; i < S * CH; i += blockDim.x) {
      const int r = i / CH, c = i % CH;
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(ptx::smem_u32(Os + r * C::LDS + c * 8)),
                   "l"(osrc + (size_t)r * d + c * 8)
                   : "memory");
    }
  }
  cp_async_wait_all();
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  // Di = rowsum(dO * O) (fp32), one warp per row, fixed lane order
  for (int r = warp; r < S; r += NWARP) {
    const bf16* orow = Os + r * C::LDS;
    const bf16* drow = dOs + r * C::LDH;
    float acc = 0.f;
    for (int c = 2 * lane; c < HD; c += 64) {
      const float2 ov = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(orow + c));
      const float2 dv = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(drow + c));
      acc += ov.x * dv.x + ov.y * dv.y;
    }
#pragma unroll
    for (int s = 16; s >= 1; s >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, s);
    if (lane == 0) Di[r] = acc;
  }
  __syncthreads();
  const float scale = 1.f / sqrtf((float)HD);
  const float scale_log2 = 1.4426950408889634f * scale;
  const int r0 = warp * 16;
  const bool active = r0 < S;
  float dp[SMAX / 8][4];  // dS rows of this warp (kept for the one-buffer path)
  if (active) {
    float sacc[SMAX / 8][4];
    scores<HD>(Qs, Ks, r0, S, sacc);
    const float l0 = lse[(size_t)bh * S + r0 + g] * 1.4426950408889634f;
    const float l1 = lse[(size_t)bh * S + r0 + g + 8] * 1.4426950408889634f;
#pragma unroll
    for (int nb = 0; nb < SMAX / 8; ++nb) {
      sacc[nb][0] = exp2f(sacc[nb][0] * scale_log2 - l0);
      sacc[nb][1] = exp2f(sacc[nb][1] * scale_log2 - l0);
      sacc[nb][2] = exp2f(sacc[nb][2] * scale_log2 - l1);
      sacc[nb][3] = exp2f(sacc[nb][3] * scale_log2 - l1);
    }
    // dP = dO V^T
    scores<HD>(dOs, Vs, r0, S, dp);
    const float d0 = Di[r0 + g], d1 = Di[r0 + g + 8];
#pragma unroll
    for (int nb = 0; nb < SMAX / 8; ++nb) {
      if (nb * 8 < S) {
        const int col = nb * 8 + 2 * t;
        // dS = P * (dP - Di)
        dp[nb][0] = sacc[nb][0] * (dp[nb][0] - d0);
        dp[nb][1] = sacc[nb][1] * (dp[nb][1] - d0);
        dp[nb][2] = sacc[nb][2] * (dp[nb][2] - d1);
        dp[nb][3] = sacc[nb][3] * (dp[nb][3] - d1);
        *reinterpret_cast<uint32_t*>(Ps + (r0 + g) * C::LDS + col) = ptx::pack_bf16(sacc[nb][0], sacc[nb][1]);
        *reinterpret_cast<uint32_t*>(Ps + (r0 + g + 8) * C::LDS + col) = ptx::pack_bf16(sacc[nb][2], sacc[nb][3]);
        if (!ONEBUF) {
          *reinterpret_cast<uint32_t*>(dSs + (r0 + g) * C::LDS + col) = ptx::pack_bf16(dp[nb][0], dp[nb][1]);
          *reinterpret_cast<uint32_t*>(dSs + (r0 + g + 8) * C::LDS + col) = ptx::pack_bf16(dp[nb][2], dp[nb][3]);
        }
      }
    }
    // dQ = dS K * scale
    float acc[HD / 8][4];
#pragma unroll
    for (int nb = 0; nb < HD / 8; ++nb) acc[nb][0] = acc[nb][1] = acc[nb][2] = acc[nb][3] = 0.f;
#pragma unroll
    for (int kk = 0; kk < SMAX / 16; ++kk) {
      if (kk * 16 < S) {
        uint32_t a[4];
        a[0] = ptx::pack_bf16(dp[2 * kk][0], dp[2 * kk][1]);
        a[1] = ptx::pack_bf16(dp[2 * kk][2], dp[2 * kk][3]);
        a[2] = ptx::pack_bf16(dp[2 * kk + 1][0], dp[2 * kk + 1][1]);
        a[3] = ptx::pack_bf16(dp[2 * kk + 1][2], dp[2 * kk + 1][3]);
#pragma unroll
        for (int np = 0; np < HD / 16; ++np) {
          uint32_t bb[4];
          lds_b_kn(Ks, C::LDH, kk * 16, np * 16, bb);
          ptx::mma_bf16_16816(acc[2 * np], a, bb[0], bb[1]);
          ptx::mma_bf16_16816(acc[2 * np + 1], a, bb[2], bb[3]);
        }
      }
    }
    bf16* q0 = dqkv + ((size_t)b * S + r0 + g) * ld + hh * HD;
    bf16* q1 = q0 + 8 * ld;
#pragma unroll
    for (int nb = 0; nb < HD / 8; ++nb) {
      *reinterpret_cast<uint32_t*>(q0 + nb * 8 + 2 * t) = ptx::pack_bf16(acc[nb][0] * scale, acc[nb][1] * scale);
      *reinterpret_cast<uint32_t*>(q1 + nb * 8 + 2 * t) = ptx::pack_bf16(acc[nb][2] * scale, acc[nb][3] * scale);
    }
  }
  __syncthreads();
  bf16* k0p = dqkv + ((size_t)b * S + r0 + g) * ld + d + hh * HD;
  bf16* k1p = k0p + 8 * ld;
  bf16* v0p = k0p + d;
  bf16* v1p = k1p + d;
  if (ONEBUF) {
    // dV = P^T dO (this warp: key rows r0..r0+15), then dS replaces P and dK = dS^T Q * scale
    if (active) {
      float dv[HD / 8][4];
#pragma unroll
      for (int nb = 0; nb < HD / 8; ++nb) dv[nb][0] = dv[nb][1] = dv[nb][2] = dv[nb][3] = 0.f;
#pragma unroll
      for (int kk = 0; kk < SMAX / 16; ++kk) {
        if (kk * 16 < S) {
          uint32_t ap[4];
          lds_a_t(Ps, C::LDS, r0, kk * 16, ap);
#pragma unroll
          for (int np = 0; np < HD / 16; ++np) {
            uint32_t bo[4];
            lds_b_kn(dOs, C::LDH, kk * 16, np * 16, bo);
            ptx::mma_bf16_16816(dv[2 * np], ap, bo[0], bo[1]);
            ptx::mma_bf16_16816(dv[2 * np + 1], ap, bo[2], bo[3]);
          }
        }
      }
#pragma unroll
      for (int nb = 0; nb < HD / 8; ++nb) {
        *reinterpret_cast<uint32_t*>(v0p + nb * 8 + 2 * t) = ptx::pack_bf16(dv[nb][0], dv[nb][1]);
        *reinterpret_cast<uint32_t*>(v1p + nb * 8 + 2 * t) = ptx::pack_bf16(dv[nb][2], dv[nb][3]);
      }
    }
    __syncthreads();  // every warp has read P
    if (active) {
#pragma unroll
      for (int nb = 0; nb < SMAX / 8; ++nb) {
        if (nb * 8 < S) {
          const int col = nb * 8 + 2 * t;
          *reinterpret_cast<uint32_t*>(dSs + (r0 + g) * C::LDS + col) = ptx::pack_bf16(dp[nb][0], dp[nb][1]);
          *reinterpret_cast<uint32_t*>(dSs + (r0 + g + 8) * C::LDS + col) = ptx::pack_bf16(dp[nb][2], dp[nb][3]);
        }
      }
    }
    __syncthreads();
    if (!active) return;
    float dk[HD / 8][4];
#pragma unroll
    for (int nb = 0; nb < HD / 8; ++nb) dk[nb][0] = dk[nb][1] = dk[nb][2] = dk[nb][3] = 0.f;
#pragma unroll
    for (int kk = 0; kk < SMAX / 16; ++kk) {
      if (kk * 16 < S) {
        uint32_t as[4];
        lds_a_t(dSs, C::LDS, r0, kk * 16, as);
#pragma unroll
        for (int np = 0; np < HD / 16; ++np) {
          uint32_t bq[4];
          lds_b_kn(Qs, C::LDH, kk * 16, np * 16, bq);
          ptx::mma_bf16_16816(dk[2 * np], as, bq[0], bq[1]);
          ptx::mma_bf16_16816(dk[2 * np + 1], as, bq[2], bq[3]);
        }
      }
    }
#pragma unroll
    for (int nb = 0; nb < HD / 8; ++nb) {
      *reinterpret_cast<uint32_t*>(k0p + nb * 8 + 2 * t) = ptx::pack_bf16(dk[nb][0] * scale, dk[nb][1] * scale);
      *reinterpret_cast<uint32_t*>(k1p + nb * 8 + 2 * t) = ptx::pack_bf16(dk[nb][2] * scale, dk[nb][3] * scale);
    }
    return;
  }
  if (!active) return;
  // dK = dS^T Q * scale ; dV = P^T dO   (this warp: key rows r0..r0+15)
  float dk[HD / 8][4], dv[HD / 8][4];
#pragma unroll
  for (int nb = 0; nb < HD / 8; ++nb) {
    dk[nb][0] = dk[nb][1] = dk[nb][2] = dk[nb][3] = 0.f;
    dv[nb][0] = dv[nb][1] = dv[nb][2] = dv[nb][3] = 0.f;
  }
#pragma unroll
  for (int kk = 0; kk < SMAX / 16; ++kk) {
    if (kk * 16 < S) {
      uint32_t as[4], ap[4];
      lds_a_t(dSs, C::LDS, r0, kk * 16, as);
      lds_a_t(Ps, C::LDS, r0, kk * 16, ap);
#pragma unroll
      for (int np = 0; np < HD / 16; ++np) {
        uint32_t bq[4], bo[4];
        lds_b_kn(Qs, C::LDH, kk * 16, np * 16, bq);
        lds_b_kn(dOs, C::LDH, kk * 16, np * 16, bo);
        ptx::mma_bf16_16816(dk[2 * np], as, bq[0], bq[1]);
        ptx::mma_bf16_16816(dk[2 * np + 1], as, bq[2], bq[3]);
        ptx::mma_bf16_16816(dv[2 * np], ap, bo[0], bo[1]);
        ptx::mma_bf16_16816(dv[2 * np + 1], ap, bo[2], bo[3]);
      }
    }
  }
#pragma unroll
  for (int nb = 0; nb < HD / 8; ++nb) {
    *reinterpret_cast<uint32_t*>(k0p + nb * 8 + 2 * t) = ptx::pack_bf16(dk[nb][0] * scale, dk[nb][1] * scale);
    *reinterpret_cast<uint32_t*>(k1p + nb * 8 + 2 * t) = ptx::pack_bf16(dk[nb][2] * scale, dk[nb][3] * scale);
    *reinterpret_cast<uint32_t*>(v0p + nb * 8 + 2 * t) = ptx::pack_bf16(dv[nb][0], dv[nb][1]);
    *reinterpret_cast<uint32_t*>(v1p + nb * 8 + 2 * t) = ptx::pack_bf16(dv[nb][2], dv[nb][3]);
  }
}

template <int HD>
void fwd_launch(cudaStream_t s, const bf16* qkv, bf16* o, float* lse, int B, int S, int d, int h) {
  const int smem = 3 * SMAX * AttnCfg<HD>::LDH * 2;
  cudaFuncSetAttribute(attn_fwd_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  launch_pdl(attn_fwd_kernel<HD>, dim3(B * h), dim3(256), smem, s, qkv, o, lse, S, d, h);
}
template <int HD>
void bwd_launch(cudaStream_t s, const bf16* qkv, const bf16* o, const float* lse, const bf16* dout, bf16* dqkv,
                int B, int S, int d, int h) {
  const int smem = 4 * SMAX * AttnCfg<HD>::LDH * 2 + (HD <= 64 ? 1 : 2) * SMAX * AttnCfg<HD>::LDS * 2 + SMAX * 4;
  cudaFuncSetAttribute(attn_bwd_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  launch_pdl(attn_bwd_kernel<HD>, dim3(B * h), dim3(256), smem, s, qkv, o, lse, dout, dqkv, S, d, h);
}

#define NP_HD_DISPATCH(HDV, CALL) \
  switch (HDV) {                  \
    case 16: CALL(16); break;     \
    case 32: CALL(32); break;     \
    case 48: CALL(48); break;     \
    case 64: CALL(64); break;     \
    case 80: CALL(80); break;     \
    case 96: CALL(96); break;     \
    case 112: CALL(112); break;   \
    case 128: CALL(128); break;   \
    default: NP_REQUIRE(false, NASPIPE_EINVAL, "head dim %d unsupported", HDV); \
  }

}  // namespace

void attn_fwd(cudaStream_t s, const bf16* qkv, bf16* o, float* lse, int B, int S, int d, int h) {
  NP_REQUIRE(S % 16 == 0 && S <= SMAX, NASPIPE_EINVAL, "attention needs S %% 16 == 0 and S <= 128 (S=%d)", S);
  if (attn_tc_supported(S, d, h)) return attn_fwd_tc(s, qkv, o, lse, B, S, d, h);  // tcgen05 (attention_tc.cu)
  const int hd = d / h;
#define CALLF(X) fwd_launch<X>(s, qkv, o, lse, B, S, d, h)
  NP_HD_DISPATCH(hd, CALLF)
#undef CALLF
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "attn_fwd: %s", cudaGetErrorString(e));
}

void attn_bwd(cudaStream_t s, const bf16* qkv, const bf16* o, const float* lse, const bf16* dout, bf16* dqkv,
              int B, int S, int d, int h) {
  NP_REQUIRE(S % 16 == 0 && S <= SMAX, NASPIPE_EINVAL, "attention needs S %% 16 == 0 and S <= 128 (S=%d)", S);
  if (attn_tc_supported(S, d, h)) return attn_bwd_tc(s, qkv, o, lse, dout, dqkv, B, S, d, h);
  const int hd = d / h;
#define CALLB(X) bwd_launch<X>(s, qkv, o, lse, dout, dqkv, B, S, d, h)
  NP_HD_DISPATCH(hd, CALLB)
#undef CALLB
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "attn_bwd: %s", cudaGetErrorString(e));
}

}  // namespace naspipe
