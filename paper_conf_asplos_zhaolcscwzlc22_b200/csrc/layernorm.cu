// LayerNorm forward / backward (eps 1e-5, biased variance; reading A17) and the fp32->bf16
// cast with column partial sums.  HBM-bound CUDA-core kernels: one warp per row with the
// row held in registers (one read of every input), float4 accesses, and fixed-order
// reductions (lane-strided sums, xor-shuffle tree, fixed warp tree) — no atomics.
//
// The column partials of ln_bwd (colsum of dx) and of cast_colsum are produced with the SAME
// summation order (rows of a 16-row block in order), so a bias gradient has identical bits whether its
// block's output gradient comes from the block above (ln_bwd) or from the stage boundary
// (cast_colsum): results do not depend on where stage boundaries sit.
#include <algorithm>
#include <cstdlib>

#include "common.h"
#include "kernels.h"
#include "launch.h"
#include "ptx.cuh"

namespace naspipe {
namespace {

constexpr int LN_ROWS_MAX = 32;  // rows per backward block (runtime, <= this): warp w takes rows w, w + 8, ...
constexpr int LN_WARPS = 8;
// NASPIPE_LN_ROWS (tuning; default 16) -- fixed per process, so partial counts are too
static int ln_rows() {
  static const int v = [] {  // thread-safe one-time init
    const char* e = getenv("NASPIPE_LN_ROWS");
    return e ? std::min(LN_ROWS_MAX, std::max(1, atoi(e))) : 16;
  }();
  return v;
}

inline void check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int s = 16; s >= 1; s >>= 1) v += __shfl_xor_sync(0xffffffffu, v, s);
  return v;
}
__device__ __forceinline__ float4 f4add(float4 a, float4 b) { return make_float4(a.x + b.x, a.y + b.y, a.z + b.z, a.w + b.w); }
__device__ __forceinline__ float4 f4mul(float4 a, float4 b) { return make_float4(a.x * b.x, a.y * b.y, a.z * b.z, a.w * b.w); }

// ------------------------------------------------------------------ forward (warp per row)
template <int VPL>
__global__ void __launch_bounds__(256) ln_fwd_kernel(const float* __restrict__ x, const float* __restrict__ g,
                                                     const float* __restrict__ b, bf16* __restrict__ y,
                                                     float* __restrict__ mean, float* __restrict__ rstd, int T, int d) {
  const int row = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  ptx::pdl_wait();
  if (row >= T) return;
  const int n4 = d / 4;
  const float4* xr = reinterpret_cast<const float4*>(x + (size_t)row * d);
  float4 v[VPL];
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int idx = lane + 32 * i;
    v[i] = idx < n4 ? xr[idx] : make_float4(0.f, 0.f, 0.f, 0.f);
    s += (v[i].x + v[i].y) + (v[i].z + v[i].w);
  }
  const float mu = warp_sum(s) / (float)d;
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    if (lane + 32 * i < n4) {
      const float a = v[i].x - mu, bb = v[i].y - mu, c = v[i].z - mu, e = v[i].w - mu;
      q += (a * a + bb * bb) + (c * c + e * e);
    }
  }
  const float rs = rsqrtf(warp_sum(q) / (float)d + 1e-5f);
  const float4* g4 = reinterpret_cast<const float4*>(g);
  const float4* b4 = reinterpret_cast<const float4*>(b);
  uint2* yr = reinterpret_cast<uint2*>(y + (size_t)row * d);
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int idx = lane + 32 * i;
    if (idx < n4) {
      const float4 gg = g4[idx], bb = b4[idx];
      uint2 o;
      o.x = ptx::pack_bf16((v[i].x - mu) * rs * gg.x + bb.x, (v[i].y - mu) * rs * gg.y + bb.y);
      o.y = ptx::pack_bf16((v[i].z - mu) * rs * gg.z + bb.z, (v[i].w - mu) * rs * gg.w + bb.w);
      yr[idx] = o;
    }
  }
  if (lane == 0) {
    mean[row] = mu;
    rstd[row] = rs;
  }
}

// ------------------------------------------------------------------ backward
// Block = LN_ROWS consecutive rows.  Pass 1 (warp w: rows w, w+8): per-row statistics
// m1 = mean(dy g), m2 = mean(dy g xhat) -> shared memory.  Pass 2 (thread per float4 column
// group, rows in order 0..15): dx = resid + rstd (dy g - m1 - xhat m2), its bf16 copy, and the
// column partials dgamma = sum dy xhat, dbeta = sum dy, colsum(dx) — each a sequential sum
// over the block's rows, the same order cast_colsum uses.
__global__ void __launch_bounds__(256) ln_bwd_kernel(const float* __restrict__ dy, const float* __restrict__ x,
                                                     const float* __restrict__ mean, const float* __restrict__ rstd,
                                                     const float* __restrict__ g, const float* __restrict__ resid,
                                                     float* __restrict__ dx, bf16* __restrict__ dx16,
                                                     float* __restrict__ pdg, float* __restrict__ pdb,
                                                     float* __restrict__ pcs, int T, int d, int LN_ROWS) {
  __shared__ float s_m1[LN_ROWS_MAX], s_m2[LN_ROWS_MAX], s_mu[LN_ROWS_MAX], s_rs[LN_ROWS_MAX];
  ptx::pdl_wait();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n4 = d / 4, r0 = blockIdx.x * LN_ROWS;
  const int nrows = min(LN_ROWS, T - r0);
  const float4* g4 = reinterpret_cast<const float4*>(g);
  for (int k = warp; k < nrows; k += LN_WARPS) {
    const int r = r0 + k;
    const float mu = mean[r], rs = rstd[r];
    const float4* xr = reinterpret_cast<const float4*>(x + (size_t)r * d);
    const float4* dr = reinterpret_cast<const float4*>(dy + (size_t)r * d);
    float s1 = 0.f, s2 = 0.f;
#pragma unroll 4
    for (int i = lane; i < n4; i += 32) {
      const float4 xv = xr[i], dv = dr[i], gg = g4[i];
      const float e0 = dv.x * gg.x, e1 = dv.y * gg.y, e2 = dv.z * gg.z, e3 = dv.w * gg.w;
      s1 += (e0 + e1) + (e2 + e3);
      s2 += (e0 * ((xv.x - mu) * rs) + e1 * ((xv.y - mu) * rs)) + (e2 * ((xv.z - mu) * rs) + e3 * ((xv.w - mu) * rs));
    }
    s1 = warp_sum(s1);
    s2 = warp_sum(s2);
    if (lane == 0) {
      s_m1[k] = s1 / (float)d;
      s_m2[k] = s2 / (float)d;
      s_mu[k] = mu;
      s_rs[k] = rs;
    }
  }
  __syncthreads();
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int c = threadIdx.x; c < n4; c += blockDim.x) {
    const float4 gg = g4[c];
    float4 ag = z4, ab = z4, ac = z4;
#pragma unroll 4
    for (int k = 0; k < nrows; ++k) {
      const size_t off = (size_t)(r0 + k) * n4 + c;
      const float4 xv = reinterpret_cast<const float4*>(x)[off];
      const float4 dv = reinterpret_cast<const float4*>(dy)[off];
      const float4 re = reinterpret_cast<const float4*>(resid)[off];
      const float mu = s_mu[k], rs = s_rs[k], m1 = s_m1[k], m2 = s_m2[k];
      const float4 xh = make_float4((xv.x - mu) * rs, (xv.y - mu) * rs, (xv.z - mu) * rs, (xv.w - mu) * rs);
      float4 o;
      o.x = re.x + rs * (dv.x * gg.x - m1 - xh.x * m2);
      o.y = re.y + rs * (dv.y * gg.y - m1 - xh.y * m2);
      o.z = re.z + rs * (dv.z * gg.z - m1 - xh.z * m2);
      o.w = re.w + rs * (dv.w * gg.w - m1 - xh.w * m2);
      reinterpret_cast<float4*>(dx)[off] = o;
      if (dx16) {
        uint2 p;
        p.x = ptx::pack_bf16(o.x, o.y);
        p.y = ptx::pack_bf16(o.z, o.w);
        reinterpret_cast<uint2*>(dx16)[off] = p;
      }
      ag = f4add(ag, f4mul(dv, xh));
      ab = f4add(ab, dv);
      ac = f4add(ac, o);
    }
    reinterpret_cast<float4*>(pdg + (size_t)blockIdx.x * d)[c] = ag;
    reinterpret_cast<float4*>(pdb + (size_t)blockIdx.x * d)[c] = ab;
    if (pcs) reinterpret_cast<float4*>(pcs + (size_t)blockIdx.x * d)[c] = ac;
  }
}

// X16 = bf16(X) and the column partials of X over LN_ROWS-row blocks, rows summed in order
// (ln_bwd's colsum order)
__global__ void __launch_bounds__(256) cast_colsum_kernel(const float* __restrict__ X, bf16* __restrict__ X16,
                                                          float* __restrict__ part, int T, int d, int LN_ROWS) {
  ptx::pdl_wait();
  const int n4 = d / 4, r0 = blockIdx.x * LN_ROWS;
  const int nrows = min(LN_ROWS, T - r0);
  for (int c = threadIdx.x; c < n4; c += blockDim.x) {
    float4 ac = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 4
    for (int k = 0; k < nrows; ++k) {
      const size_t off = (size_t)(r0 + k) * n4 + c;
      const float4 v = reinterpret_cast<const float4*>(X)[off];
      uint2 p;
      p.x = ptx::pack_bf16(v.x, v.y);
      p.y = ptx::pack_bf16(v.z, v.w);
      reinterpret_cast<uint2*>(X16)[off] = p;
      ac = f4add(ac, v);
    }
    reinterpret_cast<float4*>(part + (size_t)blockIdx.x * d)[c] = ac;
  }
}

int vpl_for(int d) {
  const int v = (d / 4 + 31) / 32;
  NP_REQUIRE(d % 4 == 0 && v <= 16, NASPIPE_EINVAL, "LayerNorm width %d unsupported (d %% 4, d <= 2048)", d);
  return v <= 1 ? 1 : v <= 2 ? 2 : v <= 4 ? 4 : v <= 8 ? 8 : 16;
}

}  // namespace

int ln_bwd_blocks(int T) { return (T + ln_rows() - 1) / ln_rows(); }

void ln_fwd(cudaStream_t s, const float* x, const float* g, const float* b, bf16* y16, float* mean, float* rstd,
            int T, int d) {
  const int grid = (T + 7) / 8;
  switch (vpl_for(d)) {
    case 1: launch_pdl(ln_fwd_kernel<1>, dim3(grid), dim3(256), 0, s, x, g, b, y16, mean, rstd, T, d); break;
    case 2: launch_pdl(ln_fwd_kernel<2>, dim3(grid), dim3(256), 0, s, x, g, b, y16, mean, rstd, T, d); break;
    case 4: launch_pdl(ln_fwd_kernel<4>, dim3(grid), dim3(256), 0, s, x, g, b, y16, mean, rstd, T, d); break;
    case 8: launch_pdl(ln_fwd_kernel<8>, dim3(grid), dim3(256), 0, s, x, g, b, y16, mean, rstd, T, d); break;
    default: launch_pdl(ln_fwd_kernel<16>, dim3(grid), dim3(256), 0, s, x, g, b, y16, mean, rstd, T, d); break;
  }
  check_launch("ln_fwd");
}

void ln_bwd(cudaStream_t s, const float* dy, const float* x, const float* mean, const float* rstd, const float* g,
            const float* resid, float* dx, bf16* dx16, float* part_dg, float* part_db, float* part_colsum, int T,
            int d) {
  NP_REQUIRE(d % 4 == 0, NASPIPE_EINVAL, "LayerNorm width %d must be a multiple of 4", d);
  launch_pdl(ln_bwd_kernel, dim3(ln_bwd_blocks(T)), dim3(256), 0, s, dy, x, mean, rstd, g, resid, dx, dx16, part_dg,
             part_db, part_colsum, T, d, ln_rows());
  check_launch("ln_bwd");
}

void cast_colsum(cudaStream_t s, const float* X, bf16* X16, float* part, int T, int N) {
  NP_REQUIRE(N % 4 == 0, NASPIPE_EINVAL, "cast_colsum width %d must be a multiple of 4", N);
  launch_pdl(cast_colsum_kernel, dim3(ln_bwd_blocks(T)), dim3(256), 0, s, X, X16, part, T, N, ln_rows());
  check_launch("cast_colsum");
}

}  // namespace naspipe
