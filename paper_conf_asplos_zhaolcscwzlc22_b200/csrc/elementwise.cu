// CUDA-core kernels: LayerNorm fwd/bwd, deterministic column sums, SGD from partials,
// MSE loss, casts, synthetic data, and the fp32 MLP family (configs[0]).  All reductions
// use a fixed order (per-thread sequential, fixed shuffle tree, fixed partial order), never
// floating-point atomics, so every result is bitwise reproducible.
#include <algorithm>
#include <cstdlib>

#include "common.h"
#include "kernels.h"
#include "launch.h"
#include "ptx.cuh"

namespace naspipe {
namespace {

// rows per block in colsum partials (a function of the process environment only, so the
// partial count is fixed per run: NASPIPE_CS_ROWS overrides it for tuning)
static int cs_rows() {
  static const int v = [] {  // thread-safe one-time init
    const char* e = getenv("NASPIPE_CS_ROWS");
    return e ? std::max(8, atoi(e)) : 16;
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

// ---------------------------------------------------------------- column sums
template <typename T>
__device__ __forceinline__ float to_f(T v);
template <>
__device__ __forceinline__ float to_f<float>(float v) { return v; }
template <>
__device__ __forceinline__ float to_f<bf16>(bf16 v) { return __bfloat162float(v); }

// thread = 8 consecutive bf16 columns (one 16-byte load per row), rows of the block in order
__global__ void colsum_bf16_kernel(const bf16* __restrict__ X, float* __restrict__ part, int T_rows, int N,
                                   int CS_ROWS) {
  ptx::pdl_wait();
  const int c8 = blockIdx.x * blockDim.x + threadIdx.x;
  if (c8 * 8 >= N) return;
  const int r0 = blockIdx.y * CS_ROWS, r1 = min(T_rows, r0 + CS_ROWS);
  float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll 8
  for (int r = r0; r < r1; ++r) {
    uint4 q = reinterpret_cast<const uint4*>(X + (size_t)r * N)[c8];
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&q);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const float2 f = __bfloat1622float2(h[j]);
      acc[2 * j] += f.x;
      acc[2 * j + 1] += f.y;
    }
  }
  float4* o = reinterpret_cast<float4*>(part + (size_t)blockIdx.y * N + c8 * 8);
  o[0] = make_float4(acc[0], acc[1], acc[2], acc[3]);
  o[1] = make_float4(acc[4], acc[5], acc[6], acc[7]);
}

// 32 columns x 8 row-groups per block; group g sums partials [g*G, (g+1)*G) in order, the 8
// group sums are added in group order.
__global__ void sgd_multi_kernel(SgdJobs jobs) {
  ptx::pdl_wait();
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
  ptx::pdl_wait();
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
  ptx::pdl_wait();
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
// W, b: the weights this subnet read (input gradient); Wu, bu: the SGD WRITE targets (== W, b
// in place; the bulk accumulator copy under BSP, reading A30)
__global__ void mlp_bwd_kernel(const float* __restrict__ x, const float* __restrict__ h, const float* __restrict__ dy,
                               float* __restrict__ dx, const float* W, float* Wu, float* bu, float lr, int B, int d) {
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
    Wu[idx] -= lr * g;
  }
  for (int j = threadIdx.x; j < d; j += blockDim.x) {
    float g = 0.f;
    for (int r = 0; r < B; ++r) g += dz[r * d + j];
    bu[j] -= lr * g;
  }
}

}  // namespace

int colsum_blocks(int T) { return (T + cs_rows() - 1) / cs_rows(); }

void colsum_bf16(cudaStream_t s, const bf16* X, float* part, int T, int N) {
  NP_REQUIRE(N % 8 == 0, NASPIPE_EINVAL, "colsum width %d must be a multiple of 8", N);
  dim3 grid((N / 8 + 127) / 128, colsum_blocks(T));
  launch_pdl(colsum_bf16_kernel, grid, dim3(128), 0, s, X, part, T, N, cs_rows());
  check_launch("colsum");
}

// p -= lr * (fixed-order sum of the nblk partial rows): 8 row groups per column, summed in
// group order (sgd_multi_kernel), so long partial lists do not serialise on one thread.
void sgd_from_partials(cudaStream_t s, float* p, const float* part, int nblk, int n, float lr) {
  SgdJobs j{};
  j.lr = lr;
  j.job[0] = {p, part, nblk, n};
  j.count = 1;
  sgd_multi(s, j);
}

void sgd_multi(cudaStream_t s, const SgdJobs& jobs) {
  int nmax = 0;
  for (int i = 0; i < jobs.count; ++i) nmax = std::max(nmax, jobs.job[i].n);
  dim3 grid((nmax + 31) / 32, jobs.count);
  launch_pdl(sgd_multi_kernel, grid, dim3(256), 0, s, jobs);
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
  launch_pdl(mse_part_kernel, dim3(nb), dim3(MSE_THREADS), 0, s, y, t, dy, part, n, 2.0f / (float)n);
  launch_pdl(mse_final_kernel, dim3(1), dim3(32), 0, s, part, nb, loss, (float)(1.0 / (double)n));
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

void mlp_bwd_sgd(cudaStream_t s, const float* x, const float* h, const float* dy, float* dx, const float* W, float* Wu,
                 float* bu, float lr, int B, int d) {
  const size_t smem = (size_t)B * d * sizeof(float);
  NP_REQUIRE(smem <= 200 * 1024, NASPIPE_EINVAL, "MLP batch*width too large for one CTA");
  if (smem > 48 * 1024)
    cudaFuncSetAttribute(mlp_bwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  mlp_bwd_kernel<<<1, 512, smem, s>>>(x, h, dy, dx, W, Wu, bu, lr, B, d);
  check_launch("mlp_bwd_sgd");
}

}  // namespace naspipe
