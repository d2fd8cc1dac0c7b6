// Non-causal multi-head attention on the 5th-generation tensor cores (tcgen05) for the
// configs[2]/[3] shapes: S = 128, head dim 64 or 128 (reading A17: softmax(Q K^T / sqrt(hd)) V,
// no mask, no dropout).  One CTA of 4 warps per (batch, head); every score and gradient
// tile is a single 128 x 128 (or 128 x hd) UMMA accumulator in TMEM, so forward and
// backward need no atomics and are bitwise deterministic (fixed K order per accumulator).
//
// Forward:  TMA(Q, K, V) -> S = Q K^T (TMEM) -> softmax per row (thread = query row, from
// TMEM; P written to shared memory in the SW128 K-major operand layout) -> O = P V (V as an
// MN-major operand, no transpose) -> O / rowsum, LSE.
// Backward: TMA(Q, K, V, dO); S = Q K^T and dP = dO V^T (TMEM); thread = query row:
// P = exp(S scale - LSE), Di = rowsum(dO o O), dS = P (dP - Di) -> shared memory (bf16);
// then dV = P^T dO, dK = dS^T Q, dQ = dS K: the transposed operands are MN-major views of the
// same shared tiles (a 128-byte-swizzled [rows][64] tile is both a K-major operand with the
// row index as M/N and an MN-major operand with the row index as K).
// Numerics follow the mma.sync kernels of attention.cu (fp32 accumulation, P and dS rounded
// to bf16 for the second products); other shapes use those kernels.
#include "common.h"
#include "kernels.h"
#include "launch.h"
#include "ptx.cuh"
#include "tma.h"

namespace naspipe {
namespace {

constexpr int AS = 128;                   // sequence length of the tcgen05 path
constexpr int TILE = 128 * 128;           // bytes of one [128 rows][64 bf16] SW128 tile
constexpr float LOG2E = 1.4426950408889634f;

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// K-major SW128 operand: k-step kk (16 elements) of a [128][64*nch] operand made of
// 64-column tiles TILE bytes apart
__device__ __forceinline__ uint64_t desc_k(const uint8_t* base, int kk) {
  return ptx::umma_desc_sw128(ptx::smem_u32(base + (kk / 4) * TILE) + (kk % 4) * 32, 16, 1024);
}
// MN-major SW128 operand: k-step kk = rows 16 kk .. 16 kk + 15 of the same tiles (the MN
// dimension runs along the 64-column tiles, TILE bytes apart)
__device__ __forceinline__ uint64_t desc_mn(const uint8_t* base, int kk) {
  return ptx::umma_desc_sw128(ptx::smem_u32(base) + kk * 2048, TILE, 1024);
}
// store 8 consecutive bf16 values of row r, columns [c, c+8) (c % 8 == 0, c < 128) into a
// [128][128] operand made of two SW128 tiles (the layout TMA's 128-byte swizzle produces)
__device__ __forceinline__ void st_sw128(uint8_t* base, int r, int c, const float (&v)[8]) {
  uint4 q;
  q.x = ptx::pack_bf16(v[0], v[1]);
  q.y = ptx::pack_bf16(v[2], v[3]);
  q.z = ptx::pack_bf16(v[4], v[5]);
  q.w = ptx::pack_bf16(v[6], v[7]);
  const int chunk = (c % 64) / 8;
  *reinterpret_cast<uint4*>(base + (c / 64) * TILE + r * 128 + ((chunk ^ (r & 7)) * 16)) = q;
}
__device__ __forceinline__ uint8_t* align1024(uint8_t* p) {
  return reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(p) + 1023) & ~uintptr_t(1023));
}

// 8 warps: warps w and w + 4 share TMEM lane quarter w % 4 (query rows 32 (w % 4) ..) and
// split the 128 key columns (softmax) and the HD output columns in halves; the row maximum
// and sum combine the two halves through shared memory (sum = half 0 + half 1, fixed order).
template <int HD>
__global__ void __launch_bounds__(256, 1) attn_fwd_tc_kernel(const __grid_constant__ CUtensorMap tq, bf16* __restrict__ o,
                                                              float* __restrict__ lse, int d, int h) {
  constexpr int NCH = HD / 64;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sQ = align1024(smem_raw);
  uint8_t* sK = sQ + NCH * TILE;
  uint8_t* sV = sK + NCH * TILE;
  uint8_t* sP = sV + NCH * TILE;  // [128 q][128 k], two tiles
  uint64_t* bar = reinterpret_cast<uint64_t*>(sP + 2 * TILE);  // [0] TMA, [1] S, [2] O
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bar + 3);
  float* xch = reinterpret_cast<float*>(bar + 4);  // [2 halves][2 (max, sum)][128 rows]
  const int bh = blockIdx.x, b = bh / h, hh = bh % h;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int r = 32 * (warp & 3) + lane, hf = warp >> 2;  // TMEM lane (query row), column half
  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tq);
    for (int i = 0; i < 3; ++i) ptx::mbar_init(&bar[i], 1);
    ptx::fence_mbar_init();
  }
  ptx::pdl_wait();  // qkv of the predecessor; TMEM only after the wait (gemm.cu)
  if (warp == 0) ptx::tmem_alloc<256>(tmem_holder);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_holder;
  if (warp == 0) {  // lane 0 issues; lanes 1-31 wait at the __syncwarp, not spinning on an mbarrier
    if (lane == 0) {
      ptx::mbar_arrive_expect_tx(&bar[0], 3 * NCH * TILE);
      for (int j = 0; j < NCH; ++j) {
        ptx::tma_load_2d(sQ + j * TILE, &tq, &bar[0], hh * HD + 64 * j, b * AS);
        ptx::tma_load_2d(sK + j * TILE, &tq, &bar[0], d + hh * HD + 64 * j, b * AS);
        ptx::tma_load_2d(sV + j * TILE, &tq, &bar[0], 2 * d + hh * HD + 64 * j, b * AS);
      }
      ptx::mbar_wait(&bar[0], 0);
      ptx::tc_fence_after();
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(128, 128, 0, 0);
  #pragma unroll
      for (int kk = 0; kk < HD / 16; ++kk) ptx::umma_bf16(tmem, desc_k(sQ, kk), desc_k(sK, kk), idesc, kk > 0);
      ptx::umma_commit(&bar[1]);
    }
    __syncwarp();
  }
  ptx::mbar_wait(&bar[1], 0);
  ptx::tc_fence_after();
  const uint32_t trow = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
  const float sl2 = LOG2E / sqrtf((float)HD);
  const int k0 = hf * (AS / 2);  // this warp's key columns [k0, k0 + 64)
  float mx = -INFINITY;
#pragma unroll
  for (int c0 = k0; c0 < k0 + AS / 2; c0 += 32) {
    uint32_t v[32];
    ptx::tmem_ld32(trow + c0, v);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int i = 0; i < 32; ++i) mx = fmaxf(mx, __uint_as_float(v[i]));
  }
  xch[hf * 256 + r] = mx;
  __syncthreads();
  mx = fmaxf(xch[r], xch[256 + r]);
  float sum = 0.f;
#pragma unroll
  for (int c0 = k0; c0 < k0 + AS / 2; c0 += 32) {
    uint32_t v[32];
    ptx::tmem_ld32(trow + c0, v);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float p[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        p[i] = exp2f((__uint_as_float(v[8 * q + i]) - mx) * sl2);
        sum += p[i];
      }
      st_sw128(sP, r, c0 + 8 * q, p);
    }
  }
  xch[hf * 256 + 128 + r] = sum;
  fence_proxy_async();  // P (generic-proxy stores) visible to the tensor core (async proxy)
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  sum = xch[128 + r] + xch[256 + 128 + r];  // half 0 + half 1
  if (warp == 0) {  // lane 0 issues; lanes 1-31 wait at the __syncwarp, not spinning on an mbarrier
    if (lane == 0) {
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(128, HD, 0, 1);  // A = P K-major, B = V MN-major
  #pragma unroll
      for (int kk = 0; kk < AS / 16; ++kk) ptx::umma_bf16(tmem + 128, desc_k(sP, kk), desc_mn(sV, kk), idesc, kk > 0);
      ptx::umma_commit(&bar[2]);
    }
    __syncwarp();
  }
  ptx::mbar_wait(&bar[2], 0);
  ptx::tc_fence_after();
  const float inv = 1.f / sum;
  bf16* orow = o + ((size_t)b * AS + r) * d + hh * HD;
#pragma unroll
  for (int c0 = hf * (HD / 2); c0 < hf * (HD / 2) + HD / 2; c0 += 32) {
    uint32_t v[32];
    ptx::tmem_ld32(trow + 128 + c0, v);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint4 w;
      w.x = ptx::pack_bf16(__uint_as_float(v[8 * q]) * inv, __uint_as_float(v[8 * q + 1]) * inv);
      w.y = ptx::pack_bf16(__uint_as_float(v[8 * q + 2]) * inv, __uint_as_float(v[8 * q + 3]) * inv);
      w.z = ptx::pack_bf16(__uint_as_float(v[8 * q + 4]) * inv, __uint_as_float(v[8 * q + 5]) * inv);
      w.w = ptx::pack_bf16(__uint_as_float(v[8 * q + 6]) * inv, __uint_as_float(v[8 * q + 7]) * inv);
      *reinterpret_cast<uint4*>(orow + c0 + 8 * q) = w;
    }
  }
  if (hf == 0) lse[(size_t)bh * AS + r] = mx * sl2 * 0.6931471805599453f + logf(sum);
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<256>(tmem);
  }
}

// Di = rowsum(dO o O) of the CTA's 128 query rows into sDi, coalesced: a warp reads LPR = HD/8
// lanes x 16 bytes per row (RPI rows per load instruction, every load of the warp's rows in
// flight at once), each lane sums its 8 products in column order, then a fixed xor tree over
// the row's LPR lanes (bitwise deterministic).  (A thread-per-row loop left ~25 % of the
// backward's stall samples on these loads: 4 dependent round trips of uncoalesced rows.)
template <int HD, int NWARPS>
__device__ __forceinline__ void attn_di_rows(const bf16* __restrict__ dout, const bf16* __restrict__ o, int b, int hh,
                                             int d, float* sDi) {
  constexpr int LPR = HD / 8, RPI = 32 / LPR, ROWS = AS / NWARPS, IT = ROWS / RPI;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int sub = lane / LPR, cl = (lane % LPR) * 8;
  uint4 a[IT], q[IT];
#pragma unroll
  for (int it = 0; it < IT; ++it) {
    const int row = warp * ROWS + it * RPI + sub;
    const size_t off = ((size_t)b * AS + row) * d + hh * HD + cl;
    a[it] = *reinterpret_cast<const uint4*>(dout + off);
    q[it] = *reinterpret_cast<const uint4*>(o + off);
  }
#pragma unroll
  for (int it = 0; it < IT; ++it) {
    const uint32_t aw[4] = {a[it].x, a[it].y, a[it].z, a[it].w}, qw[4] = {q[it].x, q[it].y, q[it].z, q[it].w};
    float di = 0.f;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      di = fmaf(__uint_as_float(aw[i] << 16), __uint_as_float(qw[i] << 16), di);
      di = fmaf(__uint_as_float(aw[i] & 0xffff0000u), __uint_as_float(qw[i] & 0xffff0000u), di);
    }
#pragma unroll
    for (int off = LPR / 2; off >= 1; off >>= 1) di += __shfl_xor_sync(0xffffffffu, di, off);
    if (lane % LPR == 0) sDi[warp * ROWS + it * RPI + sub] = di;
  }
}

// 8 warps: warps w and w + 4 share TMEM lane quarter w % 4 (query / key rows 32 (w % 4) ..)
// and split the columns of the softmax phase and of the gradient epilogue in halves.
template <int HD>
__global__ void __launch_bounds__(256, 1) attn_bwd_tc_kernel(const __grid_constant__ CUtensorMap tq,
                                                              const __grid_constant__ CUtensorMap tdo,
                                                              const bf16* __restrict__ o, const float* __restrict__ lse,
                                                              const bf16* __restrict__ dout, bf16* __restrict__ dqkv,
                                                              int d, int h) {
  constexpr int NCH = HD / 64;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sQ = align1024(smem_raw);
  uint8_t* sK = sQ + NCH * TILE;
  uint8_t* sV = sK + NCH * TILE;
  uint8_t* sdO = sV + NCH * TILE;
  uint8_t* sP = sdO + NCH * TILE;   // [128 q][128 k]
  uint8_t* sdS = sP + 2 * TILE;     // [128 q][128 k]
  uint64_t* bar = reinterpret_cast<uint64_t*>(sdS + 2 * TILE);  // [0] TMA, [1] S + dP, [2] gradients
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bar + 3);
  float* sDi = reinterpret_cast<float*>(bar + 4);  // [128]
  const int bh = blockIdx.x, b = bh / h, hh = bh % h;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int r = 32 * (warp & 3) + lane, hf = warp >> 2;  // TMEM lane (row) and column half
  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tq);
    ptx::tma_prefetch(&tdo);
    for (int i = 0; i < 3; ++i) ptx::mbar_init(&bar[i], 1);
    ptx::fence_mbar_init();
  }
  ptx::pdl_wait();
  if (warp == 0) ptx::tmem_alloc<512>(tmem_holder);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_holder;
  if (warp == 0) {  // lane 0 issues; lanes 1-31 wait at the __syncwarp, not spinning on an mbarrier
    if (lane == 0) {
      ptx::mbar_arrive_expect_tx(&bar[0], 4 * NCH * TILE);
      for (int j = 0; j < NCH; ++j) {
        ptx::tma_load_2d(sQ + j * TILE, &tq, &bar[0], hh * HD + 64 * j, b * AS);
        ptx::tma_load_2d(sK + j * TILE, &tq, &bar[0], d + hh * HD + 64 * j, b * AS);
        ptx::tma_load_2d(sV + j * TILE, &tq, &bar[0], 2 * d + hh * HD + 64 * j, b * AS);
        ptx::tma_load_2d(sdO + j * TILE, &tdo, &bar[0], hh * HD + 64 * j, b * AS);
      }
      ptx::mbar_wait(&bar[0], 0);
      ptx::tc_fence_after();
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(128, 128, 0, 0);
  #pragma unroll
      for (int kk = 0; kk < HD / 16; ++kk) {
        ptx::umma_bf16(tmem, desc_k(sQ, kk), desc_k(sK, kk), idesc, kk > 0);         // S = Q K^T
        ptx::umma_bf16(tmem + 128, desc_k(sdO, kk), desc_k(sV, kk), idesc, kk > 0);  // dP = dO V^T
      }
      ptx::umma_commit(&bar[1]);
    }
    __syncwarp();
  }
  // Di = rowsum(dO o O) while the MMAs run
  attn_di_rows<HD, 8>(dout, o, b, hh, d, sDi);
  const float l2 = lse[(size_t)bh * AS + r] * LOG2E;
  const float scale = 1.f / sqrtf((float)HD), sl2 = LOG2E * scale;
  __syncthreads();
  const float di = sDi[r];
  ptx::mbar_wait(&bar[1], 0);
  ptx::tc_fence_after();
  const uint32_t trow = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
#pragma unroll
  for (int c0 = hf * (AS / 2); c0 < hf * (AS / 2) + AS / 2; c0 += 32) {
    uint32_t s[32], dp[32];
    ptx::tmem_ld32(trow + c0, s);
    ptx::tmem_ld32(trow + 128 + c0, dp);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float p[8], ds[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        p[i] = exp2f(__uint_as_float(s[8 * q + i]) * sl2 - l2);
        ds[i] = p[i] * (__uint_as_float(dp[8 * q + i]) - di);
      }
      st_sw128(sP, r, c0 + 8 * q, p);
      st_sw128(sdS, r, c0 + 8 * q, ds);
    }
  }
  fence_proxy_async();
  ptx::tc_fence_before();
  __syncthreads();  // every thread has read S and dP: their TMEM columns are reused below
  ptx::tc_fence_after();
  if (warp == 0) {  // lane 0 issues; lanes 1-31 wait at the __syncwarp, not spinning on an mbarrier
    if (lane == 0) {
      constexpr uint32_t idesc_t = ptx::umma_idesc_bf16(128, HD, 1, 1);  // A, B MN-major
      constexpr uint32_t idesc_q = ptx::umma_idesc_bf16(128, HD, 0, 1);  // A K-major, B MN-major
  #pragma unroll
      for (int kk = 0; kk < AS / 16; ++kk) {
        ptx::umma_bf16(tmem, desc_mn(sP, kk), desc_mn(sdO, kk), idesc_t, kk > 0);        // dV = P^T dO
        ptx::umma_bf16(tmem + HD, desc_mn(sdS, kk), desc_mn(sQ, kk), idesc_t, kk > 0);   // dK = dS^T Q
        ptx::umma_bf16(tmem + 256, desc_k(sdS, kk), desc_mn(sK, kk), idesc_q, kk > 0);   // dQ = dS K
      }
      ptx::umma_commit(&bar[2]);
    }
    __syncwarp();
  }
  ptx::mbar_wait(&bar[2], 0);
  ptx::tc_fence_after();
  // TMEM lane r: key r for dV, dK; query r for dQ (all three have M = 128 rows)
  const size_t ld = 3 * (size_t)d;
  bf16* qrow = dqkv + ((size_t)b * AS + r) * ld + hh * HD;
  bf16* krow = qrow + d;
  bf16* vrow = qrow + 2 * d;
#pragma unroll
  for (int c0 = hf * (HD / 2); c0 < hf * (HD / 2) + HD / 2; c0 += 32) {
    uint32_t dv[32], dk[32], dq[32];
    ptx::tmem_ld32(trow + c0, dv);
    ptx::tmem_ld32(trow + HD + c0, dk);
    ptx::tmem_ld32(trow + 256 + c0, dq);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint4 a, k4, qq;
      uint32_t* aw = &a.x;
      uint32_t* kw = &k4.x;
      uint32_t* qw = &qq.x;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int j = 8 * q + 2 * i;
        aw[i] = ptx::pack_bf16(__uint_as_float(dv[j]), __uint_as_float(dv[j + 1]));
        kw[i] = ptx::pack_bf16(__uint_as_float(dk[j]) * scale, __uint_as_float(dk[j + 1]) * scale);
        qw[i] = ptx::pack_bf16(__uint_as_float(dq[j]) * scale, __uint_as_float(dq[j + 1]) * scale);
      }
      *reinterpret_cast<uint4*>(vrow + c0 + 8 * q) = a;
      *reinterpret_cast<uint4*>(krow + c0 + 8 * q) = k4;
      *reinterpret_cast<uint4*>(qrow + c0 + 8 * q) = qq;
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<512>(tmem);
  }
}

// Backward for head dim 64 with ONE [128][128] operand buffer (P, then dS) and 256 TMEM
// columns, so two CTAs share an SM (96 KB of shared memory, half the TMEM): dS is kept in
// registers (bf16 pairs) while dV = P^T dO runs, then replaces P for dK = dS^T Q and
// dQ = dS K.  Same arithmetic as attn_bwd_tc_kernel (same operands, same K order).
__global__ void __launch_bounds__(128, 2) attn_bwd_tc64_kernel(const __grid_constant__ CUtensorMap tq,
                                                                const __grid_constant__ CUtensorMap tdo,
                                                                const bf16* __restrict__ o, const float* __restrict__ lse,
                                                                const bf16* __restrict__ dout, bf16* __restrict__ dqkv,
                                                                int d, int h) {
  constexpr int HD = 64;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sQ = align1024(smem_raw);
  uint8_t* sK = sQ + TILE;
  uint8_t* sV = sK + TILE;
  uint8_t* sdO = sV + TILE;
  uint8_t* sB = sdO + TILE;  // [128 q][128 k]: P, then dS
  uint64_t* bar = reinterpret_cast<uint64_t*>(sB + 2 * TILE);  // [0] TMA, [1] S + dP, [2] dV, [3] dK + dQ
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bar + 4);
  float* sDi = reinterpret_cast<float*>(bar + 5);  // [128]
  const int bh = blockIdx.x, b = bh / h, hh = bh % h;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, r = threadIdx.x;
  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tq);
    ptx::tma_prefetch(&tdo);
    for (int i = 0; i < 4; ++i) ptx::mbar_init(&bar[i], 1);
    ptx::fence_mbar_init();
  }
  ptx::pdl_wait();
  if (warp == 0) ptx::tmem_alloc<256>(tmem_holder);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_holder;
  if (warp == 0) {  // lane 0 issues; lanes 1-31 wait at the __syncwarp, not spinning on an mbarrier
    if (lane == 0) {
      ptx::mbar_arrive_expect_tx(&bar[0], 4 * TILE);
      ptx::tma_load_2d(sQ, &tq, &bar[0], hh * HD, b * AS);
      ptx::tma_load_2d(sK, &tq, &bar[0], d + hh * HD, b * AS);
      ptx::tma_load_2d(sV, &tq, &bar[0], 2 * d + hh * HD, b * AS);
      ptx::tma_load_2d(sdO, &tdo, &bar[0], hh * HD, b * AS);
      ptx::mbar_wait(&bar[0], 0);
      ptx::tc_fence_after();
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(128, 128, 0, 0);
  #pragma unroll
      for (int kk = 0; kk < HD / 16; ++kk) {
        ptx::umma_bf16(tmem, desc_k(sQ, kk), desc_k(sK, kk), idesc, kk > 0);         // S = Q K^T
        ptx::umma_bf16(tmem + 128, desc_k(sdO, kk), desc_k(sV, kk), idesc, kk > 0);  // dP = dO V^T
      }
      ptx::umma_commit(&bar[1]);
    }
    __syncwarp();
  }
  attn_di_rows<HD, 4>(dout, o, b, hh, d, sDi);
  __syncthreads();
  const float di = sDi[r];
  const float l2 = lse[(size_t)bh * AS + r] * LOG2E;
  const float scale = 1.f / sqrtf((float)HD), sl2 = LOG2E * scale;
  ptx::mbar_wait(&bar[1], 0);
  ptx::tc_fence_after();
  const uint32_t trow = tmem + ((uint32_t)(warp * 32) << 16);
  uint32_t dsr[64];  // dS of this row, bf16 pairs
#pragma unroll
  for (int c0 = 0; c0 < AS; c0 += 32) {
    uint32_t sv[32], dp[32];
    ptx::tmem_ld32(trow + c0, sv);
    ptx::tmem_ld32(trow + 128 + c0, dp);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float p[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) p[i] = exp2f(__uint_as_float(sv[8 * q + i]) * sl2 - l2);
#pragma unroll
      for (int i = 0; i < 4; ++i)
        dsr[(c0 + 8 * q) / 2 + i] = ptx::pack_bf16(p[2 * i] * (__uint_as_float(dp[8 * q + 2 * i]) - di),
                                                   p[2 * i + 1] * (__uint_as_float(dp[8 * q + 2 * i + 1]) - di));
      st_sw128(sB, r, c0 + 8 * q, p);
    }
  }
  fence_proxy_async();
  ptx::tc_fence_before();
  __syncthreads();  // S and dP read by every thread; P complete
  ptx::tc_fence_after();
  constexpr uint32_t idesc_t = ptx::umma_idesc_bf16(128, HD, 1, 1);
  constexpr uint32_t idesc_q = ptx::umma_idesc_bf16(128, HD, 0, 1);
  if (warp == 0) {  // lane 0 issues; lanes 1-31 wait at the __syncwarp, not spinning on an mbarrier
    if (lane == 0) {
  #pragma unroll
      for (int kk = 0; kk < AS / 16; ++kk) ptx::umma_bf16(tmem, desc_mn(sB, kk), desc_mn(sdO, kk), idesc_t, kk > 0);  // dV
      ptx::umma_commit(&bar[2]);
    }
    __syncwarp();
  }
  ptx::mbar_wait(&bar[2], 0);  // dV done: the tensor core no longer reads P
  ptx::tc_fence_after();
#pragma unroll
  for (int c = 0; c < AS; c += 8) {
    uint4 qv = make_uint4(dsr[c / 2], dsr[c / 2 + 1], dsr[c / 2 + 2], dsr[c / 2 + 3]);
    const int chunk = (c % 64) / 8;
    *reinterpret_cast<uint4*>(sB + (c / 64) * TILE + r * 128 + ((chunk ^ (r & 7)) * 16)) = qv;
  }
  fence_proxy_async();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 0) {  // lane 0 issues; lanes 1-31 wait at the __syncwarp, not spinning on an mbarrier
    if (lane == 0) {
  #pragma unroll
      for (int kk = 0; kk < AS / 16; ++kk) {
        ptx::umma_bf16(tmem + HD, desc_mn(sB, kk), desc_mn(sQ, kk), idesc_t, kk > 0);      // dK = dS^T Q
        ptx::umma_bf16(tmem + 2 * HD, desc_k(sB, kk), desc_mn(sK, kk), idesc_q, kk > 0);   // dQ = dS K
      }
      ptx::umma_commit(&bar[3]);
    }
    __syncwarp();
  }
  ptx::mbar_wait(&bar[3], 0);
  ptx::tc_fence_after();
  const size_t ld = 3 * (size_t)d;
  bf16* qrow = dqkv + ((size_t)b * AS + r) * ld + hh * HD;
  bf16* krow = qrow + d;
  bf16* vrow = qrow + 2 * d;
#pragma unroll
  for (int c0 = 0; c0 < HD; c0 += 32) {
    uint32_t dv[32], dk[32], dq[32];
    ptx::tmem_ld32(trow + c0, dv);
    ptx::tmem_ld32(trow + HD + c0, dk);
    ptx::tmem_ld32(trow + 2 * HD + c0, dq);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint4 a, k4, qq;
      uint32_t* aw = &a.x;
      uint32_t* kw = &k4.x;
      uint32_t* qw = &qq.x;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int j = 8 * q + 2 * i;
        aw[i] = ptx::pack_bf16(__uint_as_float(dv[j]), __uint_as_float(dv[j + 1]));
        kw[i] = ptx::pack_bf16(__uint_as_float(dk[j]) * scale, __uint_as_float(dk[j + 1]) * scale);
        qw[i] = ptx::pack_bf16(__uint_as_float(dq[j]) * scale, __uint_as_float(dq[j + 1]) * scale);
      }
      *reinterpret_cast<uint4*>(vrow + c0 + 8 * q) = a;
      *reinterpret_cast<uint4*>(krow + c0 + 8 * q) = k4;
      *reinterpret_cast<uint4*>(qrow + c0 + 8 * q) = qq;
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<256>(tmem);
  }
}

// (set on every launch: a static "done" flag per template instantiation would be shared by
// the <64> and <128> kernels, which have the same function type)
template <typename K>
void set_smem_attr(K kern, int bytes) {
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

}  // namespace

bool attn_tc_supported(int S, int d, int h) {
  static const bool off = [] {
    const char* e = getenv("NASPIPE_ATTN_MMA_SYNC");
    return e && e[0] == '1';
  }();
  const int hd = d / h;
  return !off && S == AS && (hd == 64 || hd == 128) && d % 8 == 0;
}

void attn_fwd_tc(cudaStream_t s, const bf16* qkv, bf16* o, float* lse, int B, int S, int d, int h) {
  const int hd = d / h;
  const CUtensorMap tq = tma_map_bf16(qkv, 3 * (uint64_t)d, (uint64_t)B * S, 3 * (uint64_t)d, 128);
  if (hd == 64) {
    const int smem = 5 * TILE + 1024 + 64 + 2048;
    set_smem_attr(attn_fwd_tc_kernel<64>, smem);
    launch_pdl(attn_fwd_tc_kernel<64>, dim3(B * h), dim3(256), smem, s, tq, o, lse, d, h);
  } else {
    const int smem = 8 * TILE + 1024 + 64 + 2048;
    set_smem_attr(attn_fwd_tc_kernel<128>, smem);
    launch_pdl(attn_fwd_tc_kernel<128>, dim3(B * h), dim3(256), smem, s, tq, o, lse, d, h);
  }
  const cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "attn_fwd_tc: %s", cudaGetErrorString(e));
}

void attn_bwd_tc(cudaStream_t s, const bf16* qkv, const bf16* o, const float* lse, const bf16* dout, bf16* dqkv, int B,
                 int S, int d, int h) {
  const int hd = d / h;
  const CUtensorMap tq = tma_map_bf16(qkv, 3 * (uint64_t)d, (uint64_t)B * S, 3 * (uint64_t)d, 128);
  const CUtensorMap tdo = tma_map_bf16(dout, (uint64_t)d, (uint64_t)B * S, (uint64_t)d, 128);
  if (hd == 64) {  // one P/dS buffer, two CTAs per SM
    const int smem = 6 * TILE + 1024 + 64 + 512;
    set_smem_attr(attn_bwd_tc64_kernel, smem);
    launch_pdl(attn_bwd_tc64_kernel, dim3(B * h), dim3(128), smem, s, tq, tdo, o, lse, dout, dqkv, d, h);
  } else {
    const int smem = 12 * TILE + 1024 + 64 + 512;
    set_smem_attr(attn_bwd_tc_kernel<128>, smem);
    launch_pdl(attn_bwd_tc_kernel<128>, dim3(B * h), dim3(256), smem, s, tq, tdo, o, lse, dout, dqkv, d, h);
  }
  const cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "attn_bwd_tc: %s", cudaGetErrorString(e));
}

}  // namespace naspipe
