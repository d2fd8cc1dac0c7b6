// CUDA-core kernels: LayerNorm fwd/bwd, deterministic column sums, SGD from partials,
// MSE loss, casts, synthetic data, and the fp32 MLP family (configs[0]).  All reductions
// use a fixed order (per-thread sequential, fixed shuffle tree, fixed partial order), never
// floating-point atomics, so every result is bitwise reproducible.
#include "common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace naspipe {
namespace {

constexpr int LN_ROWS = 16;    // rows per block in ln_bwd partials
constexpr int CS_ROWS = 64;    // rows per block in colsum partials

inline void check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int s = 16; s >= 1; s >>= 1) v += __shfl_xor_sync(0xffffffffu, v, s);
  return v;
}

// ---------------------------------------------------------------- LayerNorm forward
// one warp per row; d % 4 == 0
__global__ void ln_fwd_kernel(const float* __restrict__ x, const float* __restrict__ g, const float* __restrict__ b,
                              bf16* __restrict__ y, float* __restrict__ mean, float* __restrict__ rstd, int T, int d) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= T) return;
  const float4* xr = reinterpret_cast<const float4*>(x + (size_t)warp * d);
  const int n4 = d / 4;
  float s = 0.f;
  for (int i = lane; i < n4; i += 32) {
    const float4 v = xr[i];
    s += (v.x + v.y) + (v.z + v.w);
  }
  const float mu = warp_sum(s) / (float)d;
  float q = 0.f;
  for (int i = lane; i < n4; i += 32) {
    const float4 v = xr[i];
    const float a = v.x - mu, bb = v.y - mu, c = v.z - mu, e = v.w - mu;
    q += (a * a + bb * bb) + (c * c + e * e);
  }
  const float var = warp_sum(q) / (float)d;
  const float rs = rsqrtf(var + 1e-5f);
  const float4* g4 = reinterpret_cast<const float4*>(g);
  const float4* b4 = reinterpret_cast<const float4*>(b);
  uint2* yr = reinterpret_cast<uint2*>(y + (size_t)warp * d);
  for (int i = lane; i < n4; i += 32) {
    const float4 v = xr[i], gg = g4[i], bb = b4[i];
    uint2 o;
    o.x = ptx::pack_bf16((v.x - mu) * rs * gg.x + bb.x, (v.y - mu) * rs * gg.y + bb.y);
    o.y = ptx::pack_bf16((v.z - mu) * rs * gg.z + bb.z, (v.w - mu) * rs * gg.w + bb.w);
    yr[i] = o;
  }
  if (lane == 0) {
    mean[warp] = mu;
    rstd[warp] = rs;
  }
}

// ---------------------------------------------------------------- LayerNorm backward
// Phase 1 (warp per row): dx = resid + rstd (dxh - mean(dxh) - xhat mean(dxh xhat)), dxh = dy g.
// Phase 2 (thread per column): partial dgamma, dbeta, colsum(dx) over the block's rows.
__global__ void ln_bwd_kernel(const float* __restrict__ dy, const float* __restrict__ x,
                              const float* __restrict__ mean, const float* __restrict__ rstd,
                              const float* __restrict__ g, const float* __restrict__ resid, float* __restrict__ dx,
                              bf16* __restrict__ dx16, float* __restrict__ pdg, float* __restrict__ pdb,
                              float* __restrict__ pcs, int T, int d) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  const int r_begin = blockIdx.x * LN_ROWS, r_end = min(T, r_begin + LN_ROWS);
  const int n4 = d / 4;
  for (int r = r_begin + warp; r < r_end; r += nw) {
    const float mu = mean[r], rs = rstd[r];
    const float4* xr = reinterpret_cast<const float4*>(x + (size_t)r * d);
    const float4* dr = reinterpret_cast<const float4*>(dy + (size_t)r * d);
    const float4* g4 = reinterpret_cast<const float4*>(g);
    float s1 = 0.f, s2 = 0.f;
    for (int i = lane; i < n4; i += 32) {
      const float4 v = xr[i], dv = dr[i], gg = g4[i];
      const float h0 = (v.x - mu) * rs, h1 = (v.y - mu) * rs, h2 = (v.z - mu) * rs, h3 = (v.w - mu) * rs;
      const float e0 = dv.x * gg.x, e1 = dv.y * gg.y, e2 = dv.z * gg.z, e3 = dv.w * gg.w;
      s1 += (e0 + e1) + (e2 + e3);
      s2 += (e0 * h0 + e1 * h1) + (e2 * h2 + e3 * h3);
    }
    const float m1 = warp_sum(s1) / (float)d, m2 = warp_sum(s2) / (float)d;
    const float4* rr = reinterpret_cast<const float4*>(resid + (size_t)r * d);
    float4* outr = reinterpret_cast<float4*>(dx + (size_t)r * d);
    for (int i = lane; i < n4; i += 32) {
      const float4 v = xr[i], dv = dr[i], gg = g4[i], re = rr[i];
      float4 o;
      o.x = re.x + rs * (dv.x * gg.x - m1 - (v.x - mu) * rs * m2);
      o.y = re.y + rs * (dv.y * gg.y - m1 - (v.y - mu) * rs * m2);
      o.z = re.z + rs * (dv.z * gg.z - m1 - (v.z - mu) * rs * m2);
      o.w = re.w + rs * (dv.w * gg.w - m1 - (v.w - mu) * rs * m2);
      outr[i] = o;
      if (dx16) {
        uint2 p;
        p.x = ptx::pack_bf16(o.x, o.y);
        p.y = ptx::pack_bf16(o.z, o.w);
        reinterpret_cast<uint2*>(dx16 + (size_t)r * d)[i] = p;
      }
    }
  }
  __syncthreads();
  for (int c = threadIdx.x; c < d; c += blockDim.x) {
    float ag = 0.f, ab = 0.f, ac = 0.f;
    for (int r = r_begin; r < r_end; ++r) {
      const float dv = dy[(size_t)r * d + c];
      const float xh = (x[(size_t)r * d + c] - mean[r]) * rstd[r];
      ag += dv * xh;
      ab += dv;
      if (pcs) ac += dx[(size_t)r * d + c];
    }
    pdg[(size_t)blockIdx.x * d + c] = ag;
    pdb[(size_t)blockIdx.x * d + c] = ab;
    if (pcs) pcs[(size_t)blockIdx.x * d + c] = ac;
  }
}

// ---------------------------------------------------------------- column sums
template <typename T>
__device__ __forceinline__ float to_f(T v);
template <>
__device__ __forceinline__ float to_f<float>(float v) { return v; }
template <>
__device__ __forceinline__ float to_f<bf16>(bf16 v) { return __bfloat162float(v); }

template <typename T>
__global__ void colsum_kernel(const T* __restrict__ X, float* __restrict__ part, int T_rows, int N) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= N) return;
  const int r0 = blockIdx.y * CS_ROWS, r1 = min(T_rows, r0 + CS_ROWS);
  float acc = 0.f;
  for (int r = r0; r < r1; ++r) acc += to_f<T>(X[(size_t)r * N + c]);
  part[(size_t)blockIdx.y * N + c] = acc;
}

__global__ void cast_colsum_kernel(const float* __restrict__ X, bf16* __restrict__ X16, float* __restrict__ part,
                                   int T_rows, int N) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= N) return;
  // same row grouping and order as ln_bwd's colsum partials, so a bias gradient is
  // bitwise independent of whether its block sits at a stage boundary
  const int r0 = blockIdx.y * LN_ROWS, r1 = min(T_rows, r0 + LN_ROWS);
  float acc = 0.f;
  for (int r = r0; r < r1; ++r) {
    const float v = X[(size_t)r * N + c];
    X16[(size_t)r * N + c] = __float2bfloat16_rn(v);
    acc += v;
  }
  part[(size_t)blockIdx.y * N + c] = acc;
}

__global__ void sgd_partials_kernel(float* __restrict__ p, const float* __restrict__ part, int nblk, int n, float lr) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float g = 0.f;
  for (int j = 0; j < nblk; ++j) g += part[(size_t)j * n + i];
  p[i] -= lr * g;
}

// 32 columns x 8 row-groups per block; group g sums partials [g*G, (g+1)*G) in order, the 8
// group sums are added in group order.
__global__ void sgd_multi_kernel(SgdJobs jobs) {
  const SgdJob jb = jobs.job[blockIdx.y];
  const int lane = threadIdx.x & 31, grp = threadIdx.x >> 5;
  const int col = blockIdx.x * 32 + lane;
  if (blockIdx.x * 32 >= jb.n) return;  // block-uniform
  __shared__ float red[8][33];
  float acc = 0.f;
  if (col < jb.n) {
    const int G = (jb.nblk + 7) / 8;
    const int j0 = grp * G, j1 = min(jb.nblk, j0 + G);
#pragma unroll 8
    for (int j = j0; j < j1; ++j) acc += jb.part[(size_t)j * jb.n + col];
  }
  red[grp][lane] = acc;
  __syncthreads();
  if (grp == 0 && col < jb.n) {
    float g = 0.f;
#pragma unroll
    for (int k = 0; k < 8; ++k) g += red[k][lane];
    jb.p[col] -= jobs.lr * g;
  }
}

__global__ void f2bf_kernel(const float* __restrict__ a, bf16* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    b[i] = __float2bfloat16_rn(a[i]);
}

// ---------------------------------------------------------------- MSE loss (reading A18)
constexpr int MSE_THREADS = 256, MSE_PER_BLOCK = 8192;
__global__ void mse_part_kernel(const float* __restrict__ y, const float* __restrict__ t, float* __restrict__ dy,
                                float* __restrict__ part, size_t n, float two_over_n) {
  __shared__ float red[MSE_THREADS / 32];
  const size_t base = (size_t)blockIdx.x * MSE_PER_BLOCK;
  float acc = 0.f;
  for (int k = threadIdx.x; k < MSE_PER_BLOCK; k += MSE_THREADS) {
    const size_t i = base + k;
    if (i < n) {
      const float e = y[i] - t[i];
      acc += e * e;
      dy[i] = two_over_n * e;
    }
  }
  acc = warp_sum(acc);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    float s = 0.f;
    for (int w = 0; w < MSE_THREADS / 32; ++w) s += red[w];
    part[blockIdx.x] = s;
  }
}
__global__ void mse_final_kernel(const float* __restrict__ part, int nblk, float* __restrict__ loss, float inv_n) {
  if (threadIdx.x != 0) return;
  double s = 0.0;  // fixed order
  for (int j = 0; j < nblk; ++j) s += part[j];
  *loss = (float)(s * inv_n);
}

__global__ void synth_kernel(float* __restrict__ x, size_t n, uint64_t seed) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint64_t z = seed ^ (i * 0x9E3779B97F4A7C15ull);
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    const float u1 = ((float)(z >> 40) + 0.5f) * 5.9604644775390625e-08f;
    const float u2 = (float)((z >> 16) & 0xFFFFFF) * 5.9604644775390625e-08f;
    x[i] = sqrtf(-2.f * logf(u1)) * cospif(2.f * u2);
  }
}

// ---------------------------------------------------------------- MLP family (fp32)
// y = x + tanh(x W^T + b); one CTA, thread per output element, fixed k order
__global__ void mlp_fwd_kernel(const float* __restrict__ x, const float* __restrict__ W, const float* __restrict__ b,
                               float* __restrict__ y, float* __restrict__ h, int B, int d) {
  for (int idx = threadIdx.x; idx < B * d; idx += blockDim.x) {
    const int r = idx / d, j = idx % d;
    float z = b[j];
    for (int k = 0; k < d; ++k) z = fmaf(x[r * d + k], W[j * d + k], z);
    const float hv = tanhf(z);
    h[idx] = hv;
    y[idx] = x[idx] + hv;
  }
}

// dz = dy (1 - h^2); dx = dy + dz W (pre-update); W -= lr dz^T x; b -= lr sum_r dz
__global__ void mlp_bwd_kernel(const float* __restrict__ x, const float* __restrict__ h, const float* __restrict__ dy,
                               float* __restrict__ dx, float* __restrict__ W, float* __restrict__ b, float lr, int B,
                               int d) {
  extern __shared__ float dz[];
  for (int idx = threadIdx.x; idx < B * d; idx += blockDim.x) {
    const float hv = h[idx];
    dz[idx] = dy[idx] * (1.f - hv * hv);
  }
  __syncthreads();
  if (dx) {
    for (int idx = threadIdx.x; idx < B * d; idx += blockDim.x) {
      const int r = idx / d, k = idx % d;
      float acc = 0.f;
      for (int j = 0; j < d; ++j) acc = fmaf(dz[r * d + j], W[j * d + k], acc);
      dx[idx] = dy[idx] + acc;
    }
  }
  __syncthreads();  // every read of W above completes before the update below
  for (int idx = threadIdx.x; idx < d * d; idx += blockDim.x) {
    const int j = idx / d, k = idx % d;
    float g = 0.f;
    for (int r = 0; r < B; ++r) g = fmaf(dz[r * d + j], x[r * d + k], g);
    W[idx] -= lr * g;
  }
  for (int j = threadIdx.x; j < d; j += blockDim.x) {
    float g = 0.f;
    for (int r = 0; r < B; ++r) g += dz[r * d + j];
    b[j] -= lr * g;
  }
}

}  // namespace

void ln_fwd(cudaStream_t s, const float* x, const float* g, const float* b, bf16* y16, float* mean, float* rstd,
            int T, int d) {
  NP_REQUIRE(d % 4 == 0, NASPIPE_EINVAL, "ln d %% 4");
  const int warps_per_block = 8;
  ln_fwd_kernel<<<(T + warps_per_block - 1) / warps_per_block, 32 * warps_per_block, 0, s>>>(x, g, b, y16, mean,
                                                                                              rstd, T, d);
  check_launch("ln_fwd");
}

int ln_bwd_blocks(int T) { return (T + LN_ROWS - 1) / LN_ROWS; }

void ln_bwd(cudaStream_t s, const float* dy, const float* x, const float* mean, const float* rstd, const float* g,
            const float* resid, float* dx, bf16* dx16, float* part_dg, float* part_db, float* part_colsum, int T,
            int d) {
  ln_bwd_kernel<<<ln_bwd_blocks(T), 256, 0, s>>>(dy, x, mean, rstd, g, resid, dx, dx16, part_dg, part_db,
                                                 part_colsum, T, d);
  check_launch("ln_bwd");
}

int colsum_blocks(int T) { return (T + CS_ROWS - 1) / CS_ROWS; }

void colsum_bf16(cudaStream_t s, const bf16* X, float* part, int T, int N) {
  dim3 grid((N + 255) / 256, colsum_blocks(T));
  colsum_kernel<bf16><<<grid, 256, 0, s>>>(X, part, T, N);
  check_launch("colsum");
}

void cast_colsum(cudaStream_t s, const float* X, bf16* X16, float* part, int T, int N) {
  dim3 grid((N + 255) / 256, ln_bwd_blocks(T));
  cast_colsum_kernel<<<grid, 256, 0, s>>>(X, X16, part, T, N);
  check_launch("cast_colsum");
}

void sgd_from_partials(cudaStream_t s, float* p, const float* part, int nblk, int n, float lr) {
  sgd_partials_kernel<<<(n + 255) / 256, 256, 0, s>>>(p, part, nblk, n, lr);
  check_launch("sgd_from_partials");
}

void sgd_multi(cudaStream_t s, const SgdJobs& jobs) {
  int nmax = 0;
  for (int i = 0; i < jobs.count; ++i) nmax = std::max(nmax, jobs.job[i].n);
  dim3 grid((nmax + 31) / 32, jobs.count);
  sgd_multi_kernel<<<grid, 256, 0, s>>>(jobs);
  check_launch("sgd_multi");
}

void f32_to_bf16(cudaStream_t s, const float* w32, bf16* w16, size_t n) {
  const int blocks = (int)std::min<size_t>((n + 255) / 256, 148 * 16);
  f2bf_kernel<<<blocks, 256, 0, s>>>(w32, w16, n);
  check_launch("f32_to_bf16");
}

int mse_blocks(size_t n) { return (int)((n + MSE_PER_BLOCK - 1) / MSE_PER_BLOCK); }

void mse_loss(cudaStream_t s, const float* y, const float* t, float* dy, float* part, float* loss, size_t n) {
  const int nb = mse_blocks(n);
  mse_part_kernel<<<nb, MSE_THREADS, 0, s>>>(y, t, dy, part, n, 2.0f / (float)n);
  mse_final_kernel<<<1, 32, 0, s>>>(part, nb, loss, (float)(1.0 / (double)n));
  check_launch("mse_loss");
}

void synth_fill(cudaStream_t s, float* x, size_t n, uint64_t seed) {
  const int blocks = (int)std::min<size_t>((n + 255) / 256, 148 * 16);
  synth_kernel<<<blocks, 256, 0, s>>>(x, n, seed);
  check_launch("synth_fill");
}

void mlp_fwd(cudaStream_t s, const float* x, const float* W, const float* b, float* y, float* h, int B, int d) {
  mlp_fwd_kernel<<<1, 512, 0, s>>>(x, W, b, y, h, B, d);
  check_launch("mlp_fwd");
}

void mlp_bwd_sgd(cudaStream_t s, const float* x, const float* h, const float* dy, float* dx, float* W, float* b,
                 float lr, int B, int d) {
  const size_t smem = (size_t)B * d * sizeof(float);
  NP_REQUIRE(smem <= 200 * 1024, NASPIPE_EINVAL, "MLP batch*width too large for one CTA");
  if (smem > 48 * 1024)
    cudaFuncSetAttribute(mlp_bwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  mlp_bwd_kernel<<<1, 512, smem, s>>>(x, h, dy, dx, W, b, lr, B, d);
  check_launch("mlp_bwd_sgd");
}

}  // namespace naspipe
