// Sequence convolutions of the NLP op families (Table 5: Conv 3x1, Sep Conv 7x1,
// Light Conv 5x1; reading A38, oracle/transformer.py): activations [T = B*S, d] row-major,
// convolutions run along the sequence axis with zero padding inside each sequence of S rows.
//
//  * seqconv_fwd      y[t,i] = sum_u w'[i,u] x[t+u-P, i]      (depthwise, P = K/2)
//                     w' = the taps (Sep Conv), or softmax(Wl[i / (d/H), :]) computed in the
//                     kernel (Light Conv; H weight-sharing heads), flipped in u for the
//                     input gradient (the transpose of a "same" correlation).
//  * seqconv_wgrad_sgd  g[i,u] = sum_t dy[t,i] x[t+u-P, i]: fp32 CTA partials over 128-row
//                     blocks in a fixed order, added in 64-bit fixed point (fixpoint.cuh,
//                     reading A33: bitwise independent of the CTA order); the last CTA
//                     (ticket) applies the SGD WRITE (Light Conv: through the softmax Jacobian,
//                     summed over each head's channels in channel order) and clears.
//  * conv3_cols / conv3_cols_bwd   im2col of Conv 3x1 ([T, 3d], column u*d + i = x[t+u-1, i])
//                     and its adjoint (sum of the three shifted column blocks).
// HBM-bound elementwise work: 16-byte loads of 8 channels per thread, rows in registers.
#include <algorithm>
#include <cmath>

#include "common.h"
#include "kernels.h"
#include "launch.h"
#include "fixpoint.cuh"
#include "ptx.cuh"

namespace naspipe {
namespace {

constexpr int SC_TPB = 256;
constexpr int SC_R = 8;        // output rows per thread (forward / input gradient)
constexpr int WG_STRIPS = 8;   // weight gradient: row strips per CTA
constexpr int WG_RS = 16;      // rows per strip -> 128 rows per CTA
constexpr int WG_ROWS = WG_STRIPS * WG_RS;
constexpr int WG_CG = SC_TPB / WG_STRIPS;  // 32 channel groups of 8 = 256 channels per CTA

__device__ __forceinline__ void ld8(const bf16* p, float (&v)[8]) {
  const uint4 q = *reinterpret_cast<const uint4*>(p);
  const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    v[2 * i] = __uint_as_float(w[i] << 16);
    v[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
  }
}
__device__ __forceinline__ void st8(bf16* p, const float (&v)[8]) {
  uint4 q;
  q.x = ptx::pack_bf16(v[0], v[1]);
  q.y = ptx::pack_bf16(v[2], v[3]);
  q.z = ptx::pack_bf16(v[4], v[5]);
  q.w = ptx::pack_bf16(v[6], v[7]);
  *reinterpret_cast<uint4*>(p) = q;
}

// taps of channel i: direct w[i][u] (H == 0) or softmax over u of Wl[i / (d/H)][u]
template <int K>
__device__ __forceinline__ void channel_taps(const float* __restrict__ w, int H, int d, int i, float (&t)[K]) {
  if (H == 0) {
#pragma unroll
    for (int u = 0; u < K; ++u) t[u] = w[(size_t)i * K + u];
    return;
  }
  const float* r = w + (size_t)(i / (d / H)) * K;
  float mx = r[0];
#pragma unroll
  for (int u = 1; u < K; ++u) mx = fmaxf(mx, r[u]);
  float s = 0.f;
#pragma unroll
  for (int u = 0; u < K; ++u) {
    t[u] = expf(r[u] - mx);
    s += t[u];
  }
  const float inv = 1.0f / s;
#pragma unroll
  for (int u = 0; u < K; ++u) t[u] *= inv;
}

// thread = (8-channel group, SC_R-row strip inside one sequence)
template <int K, bool FLIP, bool OUTF32>
__global__ void __launch_bounds__(SC_TPB) seqconv_kernel(const bf16* __restrict__ x, const float* __restrict__ w,
                                                         int H, void* __restrict__ out, int T, int S, int d) {
  constexpr int P = K / 2;
  ptx::pdl_wait();
  const int G = d / 8, strips = (S + SC_R - 1) / SC_R;
  const size_t items = (size_t)(T / S) * strips * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const int g = (int)(it % G);
    const size_t q = it / G;
    const int st = (int)(q % strips), b = (int)(q / strips);
    const int c0 = 8 * g, t0 = st * SC_R;
    float tp[8][K];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      float tj[K];
      channel_taps<K>(w, H, d, c0 + j, tj);
#pragma unroll
      for (int u = 0; u < K; ++u) tp[j][u] = FLIP ? tj[K - 1 - u] : tj[u];
    }
    float acc[SC_R][8];
#pragma unroll
    for (int r = 0; r < SC_R; ++r)
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[r][j] = 0.f;
    const bf16* xb = x + (size_t)b * S * d + c0;
#pragma unroll
    for (int ri = 0; ri < SC_R + K - 1; ++ri) {  // input row t0 + ri - P feeds outputs r = ri - u
      const int t = t0 + ri - P;
      if (t < 0 || t >= S) continue;
      float v[8];
      ld8(xb + (size_t)t * d, v);
#pragma unroll
      for (int r = 0; r < SC_R; ++r) {
        const int u = ri - r;
        if (u >= 0 && u < K)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[r][j] = __fmaf_rn(tp[j][u], v[j], acc[r][j]);
      }
    }
#pragma unroll
    for (int r = 0; r < SC_R; ++r) {
      const int t = t0 + r;
      if (t >= S) break;
      const size_t o = ((size_t)b * S + t) * d + c0;
      if (OUTF32) {
        float4* p = reinterpret_cast<float4*>(static_cast<float*>(out) + o);
        p[0] = make_float4(acc[r][0], acc[r][1], acc[r][2], acc[r][3]);
        p[1] = make_float4(acc[r][4], acc[r][5], acc[r][6], acc[r][7]);
      } else {
        st8(static_cast<bf16*>(out) + o, acc[r]);
      }
    }
  }
}

__device__ __forceinline__ bool sc_last_cta(int* ticket) {
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

// CTA (channel block blockIdx.x of 256 channels, row block blockIdx.y of 128 rows); thread
// (channel group cg, strip st).  acc: [d * K] fixed-point totals (zero between uses), flag: the
// sticky overflow flag.  wread: the taps / Wl the forward used (softmax input); wupd: the SGD
// WRITE target (master, or the BSP accumulator).
template <int K>
__global__ void __launch_bounds__(SC_TPB) seqconv_wgrad_kernel(const bf16* __restrict__ dy, const bf16* __restrict__ x,
                                                               unsigned long long* acc, unsigned long long* flag,
                                                               int* ticket,
                                                               const float* __restrict__ wread, float* wupd, int H,
                                                               float lr, int T, int S, int d) {
  constexpr int P = K / 2, CH = WG_CG * 8;
  extern __shared__ float red[];  // [WG_STRIPS][CH * K]; later the totals [d * K] + head sums [H * K]
  ptx::pdl_wait();
  const int cg = threadIdx.x % WG_CG, st = threadIdx.x / WG_CG;
  const int c0 = (blockIdx.x * WG_CG + cg) * 8;
  const int r0 = blockIdx.y * WG_ROWS + st * WG_RS;
  float g[8][K];
#pragma unroll
  for (int j = 0; j < 8; ++j)
#pragma unroll
    for (int u = 0; u < K; ++u) g[j][u] = 0.f;
  if (c0 < d) {
    for (int r = 0; r < WG_RS; ++r) {
      const int t = r0 + r;
      if (t >= T) break;
      const int pos = t % S;
      float dv[8];
      ld8(dy + (size_t)t * d + c0, dv);
#pragma unroll
      for (int u = 0; u < K; ++u) {
        const int ps = pos + u - P;
        if (ps < 0 || ps >= S) continue;
        float xv[8];
        ld8(x + (size_t)(t + u - P) * d + c0, xv);
#pragma unroll
        for (int j = 0; j < 8; ++j) g[j][u] = __fmaf_rn(dv[j], xv[j], g[j][u]);
      }
    }
  }
#pragma unroll
  for (int j = 0; j < 8; ++j)
#pragma unroll
    for (int u = 0; u < K; ++u) red[(size_t)st * CH * K + (cg * 8 + j) * K + u] = g[j][u];
  __syncthreads();
  // strips summed in strip order -> this CTA's partial, added in fixed point
  for (int e = threadIdx.x; e < CH * K; e += SC_TPB) {
    const int ch = blockIdx.x * CH + e / K;
    if (ch >= d) continue;
    float s = 0.f;
#pragma unroll
    for (int k = 0; k < WG_STRIPS; ++k) s += red[(size_t)k * CH * K + e];
    fix_add(acc, ch * K + e % K, flag, s, FIX_B);
  }
  if (!sc_last_cta(ticket)) return;
  // the last CTA: totals, then clear for the next use
  float* tot = red;
  for (int e = threadIdx.x; e < d * K; e += SC_TPB) {
    tot[e] = (float)fix_get(acc, e, FIX_B);
    acc[e] = 0ull;
  }
  __syncthreads();
  if (H == 0) {  // Sep Conv: taps -= lr * g
    for (int e = threadIdx.x; e < d * K; e += SC_TPB) wupd[e] -= lr * tot[e];
  } else {  // Light Conv: G[h,v] = sum over the head's channels (channel order), softmax Jacobian
    const int cph = d / H;
    float* G = tot + (size_t)d * K;
    for (int e = threadIdx.x; e < H * K; e += SC_TPB) {
      const int h = e / K, v = e % K;
      float s = 0.f;
      for (int i = h * cph; i < (h + 1) * cph; ++i) s += tot[(size_t)i * K + v];
      G[e] = s;
    }
    __syncthreads();
    for (int e = threadIdx.x; e < H * K; e += SC_TPB) {
      const int h = e / K, u = e % K;
      float pr[K];
      channel_taps<K>(wread, H, d, h * cph, pr);
      float dot = 0.f;
#pragma unroll
      for (int v = 0; v < K; ++v) dot = __fmaf_rn(G[h * K + v], pr[v], dot);
      float pu = 0.f;
#pragma unroll
      for (int v = 0; v < K; ++v)
        if (v == u) pu = pr[v];
      wupd[e] -= lr * (pu * (G[e] - dot));
    }
  }
  if (threadIdx.x == 0) *ticket = 0;
}

// cols[t, u*d + i] = x[t+u-1, i] inside the sequence (else 0); 8 channels per thread
__global__ void conv3_cols_kernel(const bf16* __restrict__ x, bf16* __restrict__ cols, int T, int S, int d) {
  ptx::pdl_wait();
  const int G = d / 8;
  const size_t items = (size_t)T * 3 * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const int g = (int)(it % G);
    const int u = (int)((it / G) % 3);
    const int t = (int)(it / (3 * (size_t)G));
    const int ps = t % S + u - 1;
    uint4 v = make_uint4(0, 0, 0, 0);
    if (ps >= 0 && ps < S) v = *reinterpret_cast<const uint4*>(x + (size_t)(t + u - 1) * d + 8 * g);
    *reinterpret_cast<uint4*>(cols + (size_t)t * 3 * d + (size_t)u * d + 8 * g) = v;
  }
}

// dx[t, i] = sum_u dcols[t-u+1, u*d + i] (u = 0, 1, 2 in order; rows inside the sequence)
__global__ void conv3_cols_bwd_kernel(const float* __restrict__ dcols, float* __restrict__ dx, int T, int S, int d) {
  ptx::pdl_wait();
  const int G = d / 4;
  const size_t items = (size_t)T * G;
  for (size_t it = blockIdx.x * (size_t)blockDim.x + threadIdx.x; it < items; it += (size_t)gridDim.x * blockDim.x) {
    const int g = (int)(it % G);
    const int t = (int)(it / G);
    float4 a = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int u = 0; u < 3; ++u) {
      const int ps = t % S - u + 1;
      if (ps < 0 || ps >= S) continue;
      const float4 v = *reinterpret_cast<const float4*>(dcols + (size_t)(t - u + 1) * 3 * d + (size_t)u * d + 4 * g);
      a.x += v.x; a.y += v.y; a.z += v.z; a.w += v.w;
    }
    *reinterpret_cast<float4*>(dx + (size_t)t * d + 4 * g) = a;
  }
}

void sc_check(const char* what) {
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}
int sc_grid(size_t items) {
  const size_t g = (items + SC_TPB - 1) / SC_TPB;
  return (int)std::min<size_t>(std::max<size_t>(g, 1), (size_t)num_sms() * 8);
}

template <int K, bool FLIP, bool OUTF32>
void sc_launch(cudaStream_t s, const bf16* x, const float* w, int H, void* out, int T, int S, int d) {
  const size_t items = (size_t)(T / S) * ((S + SC_R - 1) / SC_R) * (d / 8);
  launch_pdl(seqconv_kernel<K, FLIP, OUTF32>, dim3(sc_grid(items)), dim3(SC_TPB), 0, s, x, w, H, out, T, S, d);
}

}  // namespace

void seqconv(cudaStream_t s, const bf16* x, const float* w, int H, int k, bool flip, bool out_f32, void* out, int T,
             int S, int d) {
  NP_REQUIRE(d % 8 == 0 && T % S == 0 && (H == 0 || d % H == 0), NASPIPE_EINVAL, "seqconv T=%d S=%d d=%d H=%d", T, S,
             d, H);
#define SC_CASE(KK)                                                                 \
  if (flip) {                                                                       \
    if (out_f32) sc_launch<KK, true, true>(s, x, w, H, out, T, S, d);               \
    else sc_launch<KK, true, false>(s, x, w, H, out, T, S, d);                      \
  } else {                                                                          \
    if (out_f32) sc_launch<KK, false, true>(s, x, w, H, out, T, S, d);              \
    else sc_launch<KK, false, false>(s, x, w, H, out, T, S, d);                     \
  }
  if (k == 5) { SC_CASE(5) }
  else if (k == 7) { SC_CASE(7) }
  else NP_REQUIRE(false, NASPIPE_EINVAL, "seqconv kernel %d (5 or 7)", k);
#undef SC_CASE
  sc_check("seqconv");
}

void seqconv_wgrad_sgd(cudaStream_t s, const bf16* dy, const bf16* x, unsigned long long* acc,
                       unsigned long long* flag, int* ticket, const float* wread, float* wupd, int H, int k, float lr,
                       int T, int S, int d) {
  NP_REQUIRE(d % 8 == 0 && T % S == 0 && (H == 0 || d % H == 0), NASPIPE_EINVAL, "seqconv_wgrad T=%d S=%d d=%d", T,
             S, d);
  NP_REQUIRE(d + H <= WG_STRIPS * WG_CG * 8, NASPIPE_EINVAL, "seqconv_wgrad d=%d H=%d too large", d, H);
  const dim3 grid((d + WG_CG * 8 - 1) / (WG_CG * 8), (T + WG_ROWS - 1) / WG_ROWS);
  const size_t sm = (size_t)WG_STRIPS * WG_CG * 8 * k * sizeof(float);
  if (k == 5) {
    static const bool once = cudaFuncSetAttribute(seqconv_wgrad_kernel<5>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                  (int)sm) == cudaSuccess;
    (void)once;
    launch_pdl(seqconv_wgrad_kernel<5>, grid, dim3(SC_TPB), sm, s, dy, x, acc, flag, ticket, wread, wupd, H, lr, T, S,
               d);
  } else if (k == 7) {
    static const bool once = cudaFuncSetAttribute(seqconv_wgrad_kernel<7>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                  (int)sm) == cudaSuccess;
    (void)once;
    launch_pdl(seqconv_wgrad_kernel<7>, grid, dim3(SC_TPB), sm, s, dy, x, acc, flag, ticket, wread, wupd, H, lr, T, S,
               d);
  } else {
    NP_REQUIRE(false, NASPIPE_EINVAL, "seqconv_wgrad kernel %d", k);
  }
  sc_check("seqconv_wgrad");
}

void conv3_cols(cudaStream_t s, const bf16* x, bf16* cols, int T, int S, int d) {
  NP_REQUIRE(d % 8 == 0 && T % S == 0, NASPIPE_EINVAL, "conv3_cols d=%d", d);
  launch_pdl(conv3_cols_kernel, dim3(sc_grid((size_t)T * 3 * (d / 8))), dim3(SC_TPB), 0, s, x, cols, T, S, d);
  sc_check("conv3_cols");
}

void conv3_cols_bwd(cudaStream_t s, const float* dcols, float* dx, int T, int S, int d) {
  NP_REQUIRE(d % 4 == 0 && T % S == 0, NASPIPE_EINVAL, "conv3_cols_bwd d=%d", d);
  launch_pdl(conv3_cols_bwd_kernel, dim3(sc_grid((size_t)T * (d / 4))), dim3(SC_TPB), 0, s, dcols, dx, T, S, d);
  sc_check("conv3_cols_bwd");
}

}  // namespace naspipe
