// tcgen05 GEMM for sm_100a (persistent, warp-specialised).
//
//   TMA (128B swizzle) -> 4-stage shared-memory ring -> single-thread tcgen05.mma
//   (M=128, N=256, K=16 per instruction) accumulating in TMEM (2 x 256 columns, double
//   buffered) -> tcgen05.ld epilogue with fused bias / residual / GELU / GELU' / SGD update.
//
// One CTA per SM (192 KB ring), 6 warps: warp 0 = TMA producer, warp 1 = MMA issuer (also
// allocates TMEM), warps 2-5 = epilogue (warp w reads TMEM lanes 32*(w%4)..+31).  Tiles are
// assigned statically (tile = blockIdx.x + i*gridDim.x), so the epilogue of tile i overlaps
// the main loop of tile i+1.  Deterministic split-K (for the wgrad GEMMs, K = B*S, whose
// outputs are too small to fill 148 SMs): each K slice writes an fp32 partial tile to a
// workspace and a second kernel sums the slices in fixed order and applies the epilogue.
// Every output element is produced with a fixed K order: results are bitwise reproducible.
#include <cuda.h>

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <mutex>
#include <vector>

#include "common.h"
#include "kernels.h"
#include "bnfuse.cuh"
#include "fixpoint.cuh"
#include "launch.h"
#include "ptx.cuh"
#include "tma.h"

namespace naspipe {

namespace {

constexpr int BM = 128;
constexpr int BN = 256;  // tile N of the plain (1-pass) GEMM
constexpr int BK = 64;   // 64 bf16 = 128 B = one swizzle row
constexpr int A_BYTES = BM * BK * 2;  // 16 KB
constexpr int THREADS = 320;  // 2 control warps + 8 epilogue warps
constexpr int EPI_PARTIAL = 100;  // internal: fp32 partial tile of one K slice

// Tile configuration: N tile TN; SPLIT = 3-pass bf16x2 product (A_hi B_hi + A_hi B_lo +
// A_lo B_hi, fp32 accumulation: ~16-bit-mantissa operands, used by the SPOS forward 1x1
// convs, A28).  The ring holds as many stages as fit in ~200 KB.
template <int TN, bool SPLIT>
struct TileCfg {
  static constexpr int B_BYTES = TN * BK * 2;
  static constexpr int OPS = SPLIT ? 2 : 1;
  static constexpr int STAGE_BYTES = OPS * (A_BYTES + B_BYTES);
  static constexpr int STAGES = (200 * 1024) / STAGE_BYTES > 6 ? 6 : (200 * 1024) / STAGE_BYTES;
  static constexpr int BAR_OFF = STAGES * STAGE_BYTES;
  static constexpr int STG_OFF = BAR_OFF + (2 * STAGES + 4) * 8 + 16;
  // per-warp column sums of the fused BatchNorm statistics (EPI_X2 forward, EPI_BNBWD backward)
  static constexpr int SST_OFF = STG_OFF + 8 * 32 * 20 * 4;
  static constexpr int SST_BYTES = 8 * (TN / 2) * 2 * 4;
  static constexpr int SMEM_TOTAL = SST_OFF + SST_BYTES + 1024;  // + epilogue staging, alignment slack
  static constexpr int TMEM_COLS = 2 * TN <= 128 ? 128 : (2 * TN <= 256 ? 256 : 512);
};

__device__ __forceinline__ float gelu_tanh(float z) {
  const float c = 0.7978845608028654f;
  const float u = c * (z + 0.044715f * z * z * z);
  return 0.5f * z * (1.f + ptx::tanh_fast(u));
}
__device__ __forceinline__ float gelu_tanh_grad(float z) {
  const float c = 0.7978845608028654f;
  const float t = ptx::tanh_fast(c * (z + 0.044715f * z * z * z));
  return 0.5f * (1.f + t) + 0.5f * z * (1.f - t * t) * c * (1.f + 3.f * 0.044715f * z * z);
}

__device__ __forceinline__ void store16_bf16(bf16* dst, const float (&v)[16]) {
  uint32_t p[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) p[i] = ptx::pack_bf16(v[2 * i], v[2 * i + 1]);
  uint4* o4 = reinterpret_cast<uint4*>(dst);
  o4[0] = make_uint4(p[0], p[1], p[2], p[3]);
  o4[1] = make_uint4(p[4], p[5], p[6], p[7]);
}
__device__ __forceinline__ void store16_f32(float* dst, const float (&v)[16]) {
  float4* o4 = reinterpret_cast<float4*>(dst);
#pragma unroll
  for (int i = 0; i < 4; ++i) o4[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
}

// Epilogue EPI on 4 consecutive output columns (row-major element offset `off`, column
// `col`): the operands it reads (bias, residual, fp32 master, pre-activation) and the
// outputs it writes are 16-byte (fp32) / 8-byte (bf16) vectors.
__device__ __forceinline__ uint2 pack4_bf16(float4 v) {
  return make_uint2(ptx::pack_bf16(v.x, v.y), ptx::pack_bf16(v.z, v.w));
}
__device__ __forceinline__ float bf_lo(float v) { return v - __bfloat162float(__float2bfloat16_rn(v)); }
// Per-element operand of the epilogue (residual / fp32 master / pre-activation bits), loaded
// for all of a lane's rows before any store of the chunk so the loads overlap each other and
// the TMEM read (the compiler cannot hoist them across stores it cannot disambiguate).
template <int EPI>
__device__ __forceinline__ float4 preload4(size_t off, const GemmEpiParams& ep) {
  if constexpr (EPI == EPI_BIAS_RESID_F32) return *reinterpret_cast<const float4*>(ep.resid + off);
  if constexpr (EPI == EPI_SGD) return *reinterpret_cast<const float4*>(ep.w32 + off);
  if constexpr (EPI == EPI_DGELU) {
    const uint2 z = *reinterpret_cast<const uint2*>(ep.aux16 + off);
    return make_float4(__uint_as_float(z.x), __uint_as_float(z.y), 0.f, 0.f);
  }
  return make_float4(0.f, 0.f, 0.f, 0.f);
}
template <int EPI>
__device__ __forceinline__ void epilogue4(float4 v, float4 pre, float4 b, size_t off, const GemmEpiParams& ep,
                                          int split) {
  if constexpr (EPI == EPI_PARTIAL) {
    *reinterpret_cast<float4*>(ep.ws + (size_t)split * ep.ws_stride + off) = v;
    return;
  }
  if constexpr (EPI == EPI_BIAS_BF16 || EPI == EPI_BIAS_RESID_F32 || EPI == EPI_BIAS_GELU) {
    v.x += b.x; v.y += b.y; v.z += b.z; v.w += b.w;
  }
  if constexpr (EPI == EPI_BIAS_RESID_F32) {
    v.x += pre.x; v.y += pre.y; v.z += pre.z; v.w += pre.w;
  }
  if constexpr (EPI == EPI_DGELU) {
    const uint2 zz = make_uint2(__float_as_uint(pre.x), __float_as_uint(pre.y));
    const bf16* z = reinterpret_cast<const bf16*>(&zz);
    v.x *= gelu_tanh_grad(__bfloat162float(z[0]));
    v.y *= gelu_tanh_grad(__bfloat162float(z[1]));
    v.z *= gelu_tanh_grad(__bfloat162float(z[2]));
    v.w *= gelu_tanh_grad(__bfloat162float(z[3]));
  }
  if constexpr (EPI == EPI_F32 || EPI == EPI_BIAS_RESID_F32) {
    *reinterpret_cast<float4*>(reinterpret_cast<float*>(ep.out) + off) = v;
  } else if constexpr (EPI == EPI_X2) {
    *reinterpret_cast<uint2*>(reinterpret_cast<bf16*>(ep.out) + off) = pack4_bf16(v);
    *reinterpret_cast<uint2*>(ep.out2 + off) = pack4_bf16(make_float4(bf_lo(v.x), bf_lo(v.y), bf_lo(v.z), bf_lo(v.w)));
  } else if constexpr (EPI == EPI_SGD) {
    float4 w = pre;
    w.x -= ep.lr * v.x; w.y -= ep.lr * v.y; w.z -= ep.lr * v.z; w.w -= ep.lr * v.w;
    *reinterpret_cast<float4*>(ep.w32 + off) = w;
    if (ep.w16) *reinterpret_cast<uint2*>(ep.w16 + off) = pack4_bf16(w);  // no shadow: BSP accumulator
    if (ep.w16lo)
      *reinterpret_cast<uint2*>(ep.w16lo + off) =
          pack4_bf16(make_float4(bf_lo(w.x), bf_lo(w.y), bf_lo(w.z), bf_lo(w.w)));
  } else {
    *reinterpret_cast<uint2*>(reinterpret_cast<bf16*>(ep.out) + off) = pack4_bf16(v);
    if constexpr (EPI == EPI_BIAS_GELU)
      *reinterpret_cast<uint2*>(ep.out2 + off) =
          pack4_bf16(make_float4(gelu_tanh(v.x), gelu_tanh(v.y), gelu_tanh(v.z), gelu_tanh(v.w)));
  }
}

// One epilogue warp's share of an accumulator tile: rows row0..row0+31 (its TMEM lane
// quarter, `taddr` = lane base | column base), tile columns [cbeg, cend) at output column
// n0 + c.  Chunks of EC columns go TMEM -> registers (thread = row) -> the warp's padded
// staging buffer `stg` [32][EC+4] -> registers (EC/4 lanes per row, float4 each) so that
// every global load/store of the epilogue is a coalesced row segment of 4*EC (fp32) or
// 2*EC (bf16) bytes, instead of 32 rows x 16 bytes per instruction.  The padding makes
// both staging passes bank-conflict free.
// sst (EPI_X2 with ep.stats, EPI_BNBWD with ep.bnb.acc): this warp's [cend - cbeg][2]
// column sums of its 32 rows
template <int EPI, int EC>
__device__ __forceinline__ void epilogue_warp(uint32_t taddr, float* stg, int row0, int cbeg, int cend, int n0,
                                              int M, int N, const GemmEpiParams& ep, int split, int lane,
                                              float* sst = nullptr) {
  constexpr int LD = EC + 4, LPR = EC / 4, RPI = 32 / LPR, NIT = 32 / RPI;
  constexpr bool HAS_PRE = EPI == EPI_BIAS_RESID_F32 || EPI == EPI_SGD || EPI == EPI_DGELU;
  constexpr bool HAS_BIAS = EPI == EPI_BIAS_BF16 || EPI == EPI_BIAS_RESID_F32 || EPI == EPI_BIAS_GELU;
  constexpr bool BNB = EPI == EPI_BNBWD;
  const int cc = (lane % LPR) * 4;
#pragma unroll 1
  for (int c0 = cbeg; c0 < cend; c0 += EC) {
    const int col = n0 + c0;
    if (col >= N) break;  // warp-uniform
    const int gcol = col + cc;
    float4 pre[NIT], b = make_float4(0.f, 0.f, 0.f, 0.f);
    if constexpr (HAS_BIAS) {
      if (gcol < N) b = *reinterpret_cast<const float4*>(ep.bias + gcol);
    }
    // EPI_BNBWD: the unit's per-column mean, rstd, g, b and its z (hi, lo) per element
    float4 bmu = b, brs = b, bga = b, bbe = b;
    uint2 zh[NIT], zl[NIT];
    if constexpr (BNB) {
      if (gcol < N) {
        bmu = *reinterpret_cast<const float4*>(ep.bnb.mean + gcol);
        brs = *reinterpret_cast<const float4*>(ep.bnb.rstd + gcol);
        bga = *reinterpret_cast<const float4*>(ep.bnb.g + gcol);
        bbe = *reinterpret_cast<const float4*>(ep.bnb.b + gcol);
      }
    }
#pragma unroll
    for (int it = 0; it < NIT; ++it) {
      const int grow = row0 + it * RPI + lane / LPR;
      pre[it] = make_float4(0.f, 0.f, 0.f, 0.f);
      if constexpr (HAS_PRE) {
        if (grow < M && gcol < N) pre[it] = preload4<EPI>((size_t)grow * N + gcol, ep);
      }
      if constexpr (BNB) {
        zh[it] = zl[it] = make_uint2(0u, 0u);
        if (grow < M && gcol < N) {
          const size_t off = (size_t)grow * N + gcol;
          zh[it] = *reinterpret_cast<const uint2*>(ep.bnb.z + off);
          zl[it] = *reinterpret_cast<const uint2*>(ep.bnb.z + ep.bnb.zplane + off);
        }
      }
    }
    uint32_t r[EC];
    if constexpr (EC == 32) ptx::tmem_ld32(taddr + c0, r);
    else ptx::tmem_ld16(taddr + c0, r);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int j = 0; j < EC / 4; ++j)
      *reinterpret_cast<float4*>(stg + lane * LD + 4 * j) =
          make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]), __uint_as_float(r[4 * j + 2]),
                      __uint_as_float(r[4 * j + 3]));
    __syncwarp();
    float bs[4] = {0.f, 0.f, 0.f, 0.f}, bq[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int it = 0; it < NIT; ++it) {
      const int rr = it * RPI + lane / LPR;
      const int grow = row0 + rr;
      const float4 v = *reinterpret_cast<const float4*>(stg + rr * LD + cc);
      if (grow < M && gcol < N) {
        epilogue4<EPI>(v, pre[it], b, (size_t)grow * N + gcol, ep, split);
        if constexpr (EPI == EPI_X2) {  // statistics of the stored value hi + lo
          const float vv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float hi = __bfloat162float(__float2bfloat16_rn(vv[i]));
            const float st = hi + __bfloat162float(__float2bfloat16_rn(vv[i] - hi));
            bs[i] += st;
            bq[i] = __fmaf_rn(st, st, bq[i]);
          }
        }
        if constexpr (BNB) {  // BatchNorm-backward sums of the stored dy (bn_bwd_reduce's terms)
          const float vv[4] = {v.x, v.y, v.z, v.w};
          const float zz[4] = {__uint_as_float(zh[it].x << 16) + __uint_as_float(zl[it].x << 16),
                               __uint_as_float(zh[it].x & 0xffff0000u) + __uint_as_float(zl[it].x & 0xffff0000u),
                               __uint_as_float(zh[it].y << 16) + __uint_as_float(zl[it].y << 16),
                               __uint_as_float(zh[it].y & 0xffff0000u) + __uint_as_float(zl[it].y & 0xffff0000u)};
          const float mu[4] = {bmu.x, bmu.y, bmu.z, bmu.w}, rs[4] = {brs.x, brs.y, brs.z, brs.w};
          const float ga[4] = {bga.x, bga.y, bga.z, bga.w}, be[4] = {bbe.x, bbe.y, bbe.z, bbe.w};
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            float d = __bfloat162float(__float2bfloat16_rn(vv[i])), xh;
            bn_bwd_elem(d, zz[i], mu[i], rs[i], ga[i], be[i], ep.bnb.relu, xh);
            bs[i] += d;
            bq[i] = __fmaf_rn(d, xh, bq[i]);
          }
        }
      }
    }
    if constexpr (EPI == EPI_X2 || BNB) {
      if (sst != nullptr) {  // fixed xor tree over the 8 row groups of the warp (lanes cc + 4 LPR k)
#pragma unroll
        for (int o = LPR; o < 32; o <<= 1)
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            bs[i] += __shfl_xor_sync(0xffffffffu, bs[i], o);
            bq[i] += __shfl_xor_sync(0xffffffffu, bq[i], o);
          }
        if (lane < LPR)
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            sst[(c0 - cbeg + cc + i) * 2] = bs[i];
            sst[(c0 - cbeg + cc + i) * 2 + 1] = bq[i];
          }
      }
    }
    __syncwarp();
  }
}

struct TileSpace {
  int MT, NT, splits, nk_per_split, nk;
  __device__ __forceinline__ void decode(int t, int& tm, int& tn, int& ks) const {
    ks = t % splits;
    const int r = t / splits;
    tm = r % MT;
    tn = r / MT;
  }
};

template <bool A_MN, bool B_MN, int EPI, int TN, bool SPLIT>
__global__ void __launch_bounds__(THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb,
                   const __grid_constant__ CUtensorMap ta2, const __grid_constant__ CUtensorMap tb2, int M, int N,
                   TileSpace ts, GemmEpiParams ep) {
  using Cf = TileCfg<TN, SPLIT>;
  constexpr int STAGES = Cf::STAGES, STAGE_BYTES = Cf::STAGE_BYTES, BAR_OFF = Cf::BAR_OFF;
  constexpr int B_BYTES = Cf::B_BYTES;
  constexpr int OPB = A_BYTES + B_BYTES;  // bytes of one (A, B) operand pair in a stage
  static_assert(!SPLIT || (!A_MN && !B_MN), "the 3-pass GEMM takes K-major operands");
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + BAR_OFF);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;  // [2]
  uint64_t* tempty = tfull + 2;      // [2]
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(tempty + 2);
  float* stg = reinterpret_cast<float*>(smem + Cf::STG_OFF);  // [8 warps][32][20]

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n_tiles = ts.MT * ts.NT * ts.splits;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&ta);
    ptx::tma_prefetch(&tb);
    if (SPLIT) {
      ptx::tma_prefetch(&ta2);
      ptx::tma_prefetch(&tb2);
    }
    for (int s = 0; s < STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 8);
    }
    ptx::fence_mbar_init();
  }
  // PDL: wait for the predecessor grid BEFORE taking TMEM.  An early-launched CTA that held
  // TMEM columns while it waited could sit on an SM beside a predecessor CTA that still owns
  // its accumulators; after the wait no earlier kernel of the stream is running.
  ptx::pdl_wait();  // predecessors' outputs (A, B, residual, ...) are visible from here
  if (warp == 1) ptx::tmem_alloc<Cf::TMEM_COLS>(tmem_holder);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp == 0) {
    if (lane == 0) {  // ---------------- TMA producer
      int s = 0, ph = 0;
      for (int t = blockIdx.x; t < n_tiles; t += gridDim.x) {
        int tm, tn, ks;
        ts.decode(t, tm, tn, ks);
        const int m0 = tm * BM, n0 = tn * TN;
        const int kb0 = ks * ts.nk_per_split, kb1 = min(ts.nk, kb0 + ts.nk_per_split);
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&empty[s], ph ^ 1);
          uint8_t* sa = smem + s * STAGE_BYTES;
          uint8_t* sb = sa + A_BYTES;
          ptx::mbar_arrive_expect_tx(&full[s], STAGE_BYTES);
          const int k0 = kb * BK;
          if (!A_MN) {
            ptx::tma_load_2d(sa, &ta, &full[s], k0, m0);
          } else {
#pragma unroll
            for (int j = 0; j < BM / 64; ++j) ptx::tma_load_2d(sa + j * 8192, &ta, &full[s], m0 + 64 * j, k0);
          }
          if (!B_MN) {
            ptx::tma_load_2d(sb, &tb, &full[s], k0, n0);
          } else {
#pragma unroll
            for (int j = 0; j < TN / 64; ++j) ptx::tma_load_2d(sb + j * 8192, &tb, &full[s], n0 + 64 * j, k0);
          }
          if (SPLIT) {  // lo planes of both operands behind the hi pair
            ptx::tma_load_2d(sa + OPB, &ta2, &full[s], k0, m0);
            ptx::tma_load_2d(sb + OPB, &tb2, &full[s], k0, n0);
          }
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
      }
    }
    ptx::pdl_trigger();
  } else if (warp == 1) {
    if (lane == 0) {  // ---------------- MMA issuer
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(BM, TN, A_MN ? 1 : 0, B_MN ? 1 : 0);
      int s = 0, ph = 0, it = 0;
      for (int t = blockIdx.x; t < n_tiles; t += gridDim.x, ++it) {
        int tm, tn, ks;
        ts.decode(t, tm, tn, ks);
        const int kb0 = ks * ts.nk_per_split, kb1 = min(ts.nk, kb0 + ts.nk_per_split);
        const int acc = it & 1;
        ptx::mbar_wait(&tempty[acc], ((it >> 1) & 1) ^ 1);  // epilogue drained this buffer
        ptx::tc_fence_after();
        const uint32_t d = tmem + acc * TN;
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&full[s], ph);
          ptx::tc_fence_after();
          const uint32_t sa = ptx::smem_u32(smem + s * STAGE_BYTES);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            // K-major: 128-B rows, 8-row groups 1024 B apart (SBO); a K step of 16 = +32 B.
            // MN-major: 64-element MN chunks 8 KB apart (LBO), 8 K-rows = 1024 B (SBO);
            //           a K step of 16 rows = +2048 B.
            const uint64_t ad = A_MN ? ptx::umma_desc_sw128(sa + k * 2048, 8192, 1024)
                                     : ptx::umma_desc_sw128(sa + k * 32, 16, 1024);
            const uint64_t bd = B_MN ? ptx::umma_desc_sw128(sb + k * 2048, 8192, 1024)
                                     : ptx::umma_desc_sw128(sb + k * 32, 16, 1024);
            ptx::umma_bf16(d, ad, bd, idesc, (kb > kb0 || k > 0) ? 1u : 0u);
            if (SPLIT) {  // + A_hi B_lo + A_lo B_hi
              ptx::umma_bf16(d, ad, ptx::umma_desc_sw128(sb + OPB + k * 32, 16, 1024), idesc, 1u);
              ptx::umma_bf16(d, ptx::umma_desc_sw128(sa + OPB + k * 32, 16, 1024), bd, idesc, 1u);
            }
          }
          ptx::umma_commit(&empty[s]);  // frees the smem stage when these MMAs complete
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
        ptx::umma_commit(&tfull[acc]);  // accumulator ready for the epilogue
      }
    }
    ptx::pdl_trigger();
  } else {
    // ---------------- epilogue warps 2..9: TMEM lane quarter (warp % 4), column half
    const int lane_base = 32 * (warp & 3);
    const int cbeg = ((warp - 2) >> 2) * (TN / 2);
    int it = 0;
    float run1 = 0.f, run2 = 0.f;  // fused BatchNorm sums of this thread's column over the CTA's tiles
    for (int t = blockIdx.x; t < n_tiles; t += gridDim.x, ++it) {
      int tm, tn, ks;
      ts.decode(t, tm, tn, ks);
      const int acc = it & 1;
      ptx::mbar_wait(&tfull[acc], (it >> 1) & 1);
      ptx::tc_fence_after();
      if (t + (int)gridDim.x >= n_tiles) ptx::pdl_trigger();  // last tile: let the next kernel launch
      const uint32_t taddr = tmem + ((uint32_t)lane_base << 16) + acc * TN;
      float* sst = nullptr;
      unsigned long long* sacc = EPI == EPI_BNBWD ? ep.bnb.acc : ep.stats;  // fused BatchNorm sums
      if constexpr (EPI == EPI_X2 || EPI == EPI_BNBWD)
        if (sacc != nullptr) sst = reinterpret_cast<float*>(smem + Cf::SST_OFF) + (warp - 2) * (TN / 2) * 2;
      epilogue_warp<EPI, 16>(taddr, stg + (warp - 2) * 32 * 20, tm * BM + lane_base, cbeg, cbeg + TN / 2, tn * TN, M,
                             N, ep, ks, lane, sst);
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[acc]);
      if constexpr (EPI == EPI_X2 || EPI == EPI_BNBWD) {
        if (sacc != nullptr) {
          // fused BatchNorm sums: the 4 warps of this column half (lane quarters 0..3)
          // combine their 32-row column sums in quarter order, one fixed-point add per column
          const int half = (warp - 2) >> 2;
          ptx::named_bar_sync(1 + half, 128);
          const float* base = reinterpret_cast<const float*>(smem + Cf::SST_OFF) + half * 4 * (TN / 2) * 2;
          // TN / 2 <= 128: thread (warp & 3, lane) owns column j of the half.  The CTA's tiles of
          // one column block are summed in tile order in registers and added in fixed point
          // once, when the next tile of the CTA is in another column block or there is none
          // (a per-tile add put #tiles atomics -- 1568 on a 200704-row 1x1 conv -- on each address)
          const int j = (warp & 3) * 32 + lane;
          const int gcol = tn * TN + cbeg + j;
          if (j < TN / 2 && gcol < N) {
            float s1 = 0.f, s2 = 0.f;
#pragma unroll
            for (int q = 0; q < 4; ++q) {  // quarter q is warp 2 + 4 half + ((q + 2) & 3)
              const float* w = base + ((q + 2) & 3) * (TN / 2) * 2;
              s1 += w[j * 2];
              s2 += w[j * 2 + 1];
            }
            run1 += s1;
            run2 += s2;
            int tn_next = -1;
            if (t + (int)gridDim.x < n_tiles) {
              int tm2, ks2;
              ts.decode(t + (int)gridDim.x, tm2, tn_next, ks2);
            }
            if (tn_next != tn) {
              fix_add(sacc, gcol, sacc + 2 * N, run1, EPI == EPI_BNBWD ? FIX_B : FIX_S1);
              fix_add(sacc, N + gcol, sacc + 2 * N, run2, EPI == EPI_BNBWD ? FIX_B : FIX_S2);
              run1 = run2 = 0.f;
            }
          }
          ptx::named_bar_sync(1 + half, 128);  // the slots are rewritten by the next tile
        }
      }
    }
  }
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<Cf::TMEM_COLS>(tmem);
  }
}

// CTA-pair variant (cta_group::2): a 2-CTA cluster on one TPC computes a 256 x 256 output
// tile.  CTA r loads rows [m0 + 128r, +128) of A and rows [n0 + 128r, +128) of B (the B
// half), i.e. 32 KB per 64-deep K block instead of the 48 KB a single CTA needs for its
// 128 x 256 tile: the operand traffic from L2 per flop drops by a third, which is what
// bounds the 1-CTA kernel on the step's shapes (its tensor pipe idles ~55 % of the active
// time waiting for TMA; profiles/r1_ncu_full_prof_gemm_tf.csv).  The leader (rank 0) issues
// the M=256 MMAs reading both CTAs' stages; its commits arrive on the `empty` / `tfull`
// barriers of both CTAs (multicast); both producers' TMA completions land on the leader's
// `full` barrier; both CTAs' epilogue warps release the leader's `tempty` barrier.  Each
// CTA's TMEM holds the accumulator of its own 128 rows, so the epilogue is the 1-CTA one.
// Same tile-to-K order per output element as the 1-CTA kernel: bitwise reproducible.
constexpr int PAIR_STAGE_BYTES = A_BYTES + 128 * BK * 2;  // 32 KB per CTA
constexpr int PAIR_STAGES = 5;
constexpr int PAIR_BAR_OFF = PAIR_STAGES * PAIR_STAGE_BYTES;
constexpr int PAIR_STG_OFF = PAIR_BAR_OFF + (2 * PAIR_STAGES + 4) * 8 + 16;
constexpr int PAIR_SMEM_TOTAL = PAIR_STG_OFF + 8 * 32 * 36 * 4 + 1024;

template <bool A_MN, bool B_MN, int EPI>
__global__ void __launch_bounds__(THREADS, 1)
    gemm_pair_kernel(const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb, int M, int N,
                     TileSpace ts, GemmEpiParams ep, int trig) {
  constexpr int TN = 256, STAGES = PAIR_STAGES, STAGE_BYTES = PAIR_STAGE_BYTES;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + PAIR_BAR_OFF);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;  // [2]
  uint64_t* tempty = tfull + 2;      // [2]
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(tempty + 2);
  float* stg = reinterpret_cast<float*>(smem + PAIR_STG_OFF);  // [8 warps][32][36]

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  const int pair = blockIdx.x >> 1, n_pairs = gridDim.x >> 1;
  const int n_tiles = ts.MT * ts.NT * ts.splits;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&ta);
    ptx::tma_prefetch(&tb);
    for (int s = 0; s < STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 16);  // 8 epilogue warps x 2 CTAs (only the leader's is used)
    }
    ptx::fence_mbar_init();
  }
  ptx::pdl_wait();  // before taking TMEM (see gemm_tc_kernel)
  if (warp == 1) ptx::tmem_alloc_pair<512>(tmem_holder);
  ptx::tc_fence_before();
  ptx::cluster_sync();  // barriers of both CTAs initialised, TMEM allocated
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp == 0) {
    if (lane == 0) {  // ---------------- TMA producer (both CTAs)
      int s = 0, ph = 0;
      for (int t = pair; t < n_tiles; t += n_pairs) {
        int tm, tn, ks;
        ts.decode(t, tm, tn, ks);
        const int m0 = tm * 256 + 128 * (int)rank, n0 = tn * TN + 128 * (int)rank;
        const int kb0 = ks * ts.nk_per_split, kb1 = min(ts.nk, kb0 + ts.nk_per_split);
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&empty[s], ph ^ 1);
          uint8_t* sa = smem + s * STAGE_BYTES;
          uint8_t* sb = sa + A_BYTES;
          const uint32_t fb = ptx::mapa(ptx::smem_u32(&full[s]), 0);
          if (rank == 0) ptx::mbar_arrive_expect_tx(&full[s], 2 * STAGE_BYTES);
          const int k0 = kb * BK;
          if (!A_MN) {
            ptx::tma_load_2d_pair(sa, &ta, fb, k0, m0);
          } else {
            ptx::tma_load_2d_pair(sa, &ta, fb, m0, k0);
            ptx::tma_load_2d_pair(sa + 8192, &ta, fb, m0 + 64, k0);
          }
          if (!B_MN) {
            ptx::tma_load_2d_pair(sb, &tb, fb, k0, n0);
          } else {
            ptx::tma_load_2d_pair(sb, &tb, fb, n0, k0);
            ptx::tma_load_2d_pair(sb + 8192, &tb, fb, n0 + 64, k0);
          }
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
      }
    }
    if (trig) ptx::pdl_trigger();
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {  // ---------------- MMA issuer (leader only)
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(256, TN, A_MN ? 1 : 0, B_MN ? 1 : 0);
      int s = 0, ph = 0, it = 0;
      for (int t = pair; t < n_tiles; t += n_pairs, ++it) {
        int tm, tn, ks;
        ts.decode(t, tm, tn, ks);
        const int kb0 = ks * ts.nk_per_split, kb1 = min(ts.nk, kb0 + ts.nk_per_split);
        const int acc = it & 1;
        ptx::mbar_wait_cluster(&tempty[acc], ((it >> 1) & 1) ^ 1);  // both CTAs drained this buffer
        ptx::tc_fence_after();
        const uint32_t d = tmem + acc * TN;
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&full[s], ph);
          ptx::tc_fence_after();
          const uint32_t sa = ptx::smem_u32(smem + s * STAGE_BYTES);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            const uint64_t ad = A_MN ? ptx::umma_desc_sw128(sa + k * 2048, 8192, 1024)
                                     : ptx::umma_desc_sw128(sa + k * 32, 16, 1024);
            const uint64_t bd = B_MN ? ptx::umma_desc_sw128(sb + k * 2048, 8192, 1024)
                                     : ptx::umma_desc_sw128(sb + k * 32, 16, 1024);
            ptx::umma_bf16_pair(d, ad, bd, idesc, (kb > kb0 || k > 0) ? 1u : 0u);
          }
          ptx::umma_commit_pair(&empty[s], 0x3);  // frees this stage in both CTAs
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
        ptx::umma_commit_pair(&tfull[acc], 0x3);  // both CTAs' accumulators ready
      }
    }
    if (trig) ptx::pdl_trigger();
  } else {
    // ---------------- epilogue warps 2..9 of both CTAs: this CTA's 128 rows
    const int lane_base = 32 * (warp & 3);
    const int cbeg = ((warp - 2) >> 2) * (TN / 2);
    int it = 0;
    float run1 = 0.f, run2 = 0.f;  // fused BatchNorm sums of this thread's column over the CTA's tiles
    for (int t = pair; t < n_tiles; t += n_pairs, ++it) {
      int tm, tn, ks;
      ts.decode(t, tm, tn, ks);
      const int acc = it & 1;
      ptx::mbar_wait(&tfull[acc], (it >> 1) & 1);
      ptx::tc_fence_after();
      if (trig && t + n_pairs >= n_tiles) ptx::pdl_trigger();
      const uint32_t taddr = tmem + ((uint32_t)lane_base << 16) + acc * TN;
      epilogue_warp<EPI, 32>(taddr, stg + (warp - 2) * 32 * 36, tm * 256 + 128 * (int)rank + lane_base, cbeg,
                             cbeg + TN / 2, tn * TN, M, N, ep, ks, lane);
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive_cluster(ptx::mapa(ptx::smem_u32(&tempty[acc]), 0));
    }
  }
  __syncthreads();
  ptx::cluster_sync();  // no remote arrive / MMA operand read is still in flight
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_pair<512>(tmem);
  }
}

// Fixed-order sum of the split-K partial tiles, then the final epilogue (EPI_F32 / EPI_SGD).
// L lanes (a power of two, L | 32) per float4 of output: lane j sums slices j, j+L, ... in
// order, the lanes are combined by a fixed xor tree; L = 1 (plain slice order) for <= 4
// slices, so the transformer's wgrads keep their order.
__device__ __forceinline__ float4 f4add(float4 a, float4 b) { return make_float4(a.x + b.x, a.y + b.y, a.z + b.z, a.w + b.w); }
template <int EPI>
__global__ void splitk_reduce_kernel(int M, int N, int splits, int L, GemmEpiParams ep) {
  ptx::pdl_wait();
  const size_t total = (size_t)M * N / 4;
  const int j = threadIdx.x % L;
  const size_t per_block = blockDim.x / L;
  for (size_t i = blockIdx.x * per_block + threadIdx.x / L; i - threadIdx.x / L < total; i += (size_t)gridDim.x * per_block) {
    const bool ok = i < total;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    if (ok) {
      acc = reinterpret_cast<const float4*>(ep.ws + (size_t)j * ep.ws_stride)[i];
      for (int k = j + L; k < splits; k += L) acc = f4add(acc, reinterpret_cast<const float4*>(ep.ws + (size_t)k * ep.ws_stride)[i]);
    }
    for (int o = 1; o < L; o <<= 1) {
      float4 t;
      t.x = __shfl_xor_sync(0xffffffffu, acc.x, o);
      t.y = __shfl_xor_sync(0xffffffffu, acc.y, o);
      t.z = __shfl_xor_sync(0xffffffffu, acc.z, o);
      t.w = __shfl_xor_sync(0xffffffffu, acc.w, o);
      acc = (j & o) ? f4add(t, acc) : f4add(acc, t);  // same operand order on both partners
    }
    if (!ok || j != 0) continue;
    if constexpr (EPI == EPI_F32) {
      reinterpret_cast<float4*>(ep.out)[i] = acc;
    } else {
      float4 w = reinterpret_cast<float4*>(ep.w32)[i];
      w.x -= ep.lr * acc.x; w.y -= ep.lr * acc.y; w.z -= ep.lr * acc.z; w.w -= ep.lr * acc.w;
      reinterpret_cast<float4*>(ep.w32)[i] = w;
      if (!ep.w16) continue;  // no shadow: BSP accumulator
      uint2 o;
      o.x = ptx::pack_bf16(w.x, w.y);
      o.y = ptx::pack_bf16(w.z, w.w);
      reinterpret_cast<uint2*>(ep.w16)[i] = o;
      if (ep.w16lo) {
        auto lo = [](float v) { return v - __bfloat162float(__float2bfloat16_rn(v)); };
        o.x = ptx::pack_bf16(lo(w.x), lo(w.y));
        o.y = ptx::pack_bf16(lo(w.z), lo(w.w));
        reinterpret_cast<uint2*>(ep.w16lo)[i] = o;
      }
    }
  }
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  });
  NP_REQUIRE(fn != nullptr, NASPIPE_ECUDA, "cuTensorMapEncodeTiled unavailable");
  return fn;
}

// 2-D bf16 tensor map: inner dim (contiguous) `inner` elements, `outer` rows, row pitch
// `ld` elements; box {64, box_outer}; 128-byte swizzle; OOB elements read as zero.
CUtensorMap make_map(const bf16* base, uint64_t inner, uint64_t outer, uint64_t ld, uint32_t box_outer) {
  CUtensorMap m;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {ld * 2};
  cuuint32_t box[2] = {64, box_outer};
  cuuint32_t es[2] = {1, 1};
  NP_REQUIRE(((uintptr_t)base & 15) == 0 && (ld * 2) % 16 == 0, NASPIPE_EINVAL,
             "GEMM operand must be 16-byte aligned with a 16-byte multiple row pitch");
  CUresult r = encode_fn()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<bf16*>(base), dims, strides, box,
                           es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  NP_REQUIRE(r == CUDA_SUCCESS, NASPIPE_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return m;
}

std::atomic<uint64_t> g_gemm_launches{0};
std::atomic<uint64_t> g_gemm_flops{0};  // algorithmic 2*M*N*K of every GEMM call (bf16x2: one product)


std::mutex g_cap_mu;
std::vector<std::pair<cudaStream_t, int>> g_caps;  // per-stream CTA caps (a handful of side streams)
int stream_cap(cudaStream_t s) {
  std::lock_guard<std::mutex> lk(g_cap_mu);
  for (const auto& c : g_caps)
    if (c.first == s) return c.second;
  return 0;
}

template <bool A_MN, bool B_MN, int EPI, int TN = BN, bool SPLIT = false>
void launch(cudaStream_t s, int M, int N, const TileSpace& ts, const CUtensorMap& ta, const CUtensorMap& tb,
            const GemmEpiParams& ep, const CUtensorMap* ta2 = nullptr, const CUtensorMap* tb2 = nullptr) {
  auto kern = gemm_tc_kernel<A_MN, B_MN, EPI, TN, SPLIT>;
  constexpr int SMEM = TileCfg<TN, SPLIT>::SMEM_TOTAL;
  static uint32_t configured = 0;  // per instantiation, per device bit
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(configured & (1u << dev))) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
    configured |= 1u << dev;
  }
  const int tiles = ts.MT * ts.NT * ts.splits;
  const int cap = stream_cap(s);
  const int grid = std::min(tiles, cap > 0 ? std::min(cap, num_sms()) : num_sms());
  launch_pdl(kern, dim3(grid), dim3(THREADS), SMEM, s, ta, tb, ta2 ? *ta2 : ta, tb2 ? *tb2 : tb, M, N, ts, ep);
  g_gemm_launches.fetch_add(1, std::memory_order_relaxed);
}

template <bool A_MN, bool B_MN, int EPI>
void launch_pair(cudaStream_t s, int M, int N, const TileSpace& ts, const CUtensorMap& ta, const CUtensorMap& tb,
                 const GemmEpiParams& ep) {
  auto kern = gemm_pair_kernel<A_MN, B_MN, EPI>;
  static uint32_t configured = 0;
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(configured & (1u << dev))) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, PAIR_SMEM_TOTAL);
    cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    configured |= 1u << dev;
  }
  const int tiles = ts.MT * ts.NT * ts.splits;
  const int cap = stream_cap(s);
  const int pairs = std::min(tiles, (cap > 0 ? std::min(cap, num_sms()) : num_sms()) / 2);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(2 * pairs);
  cfg.blockDim = dim3(THREADS);
  cfg.dynamicSmemBytes = PAIR_SMEM_TOTAL;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  at[1].id = cudaLaunchAttributeClusterDimension;
  at[1].val.clusterDim.x = 2;
  at[1].val.clusterDim.y = 1;
  at[1].val.clusterDim.z = 1;
  // The pair kernel is launched with the PDL attribute (it may start while its predecessor
  // drains) but does NOT trigger its own dependents early (trig = 0): with early triggers
  // the 40-step configs[2] run deadlocked on the GPU (tools/hangtest.sh: hang with triggers;
  // no hang and the best step time without them).  NASPIPE_PAIR_TRIGGER=1 re-enables them
  // for diagnosis, NASPIPE_PAIR_PDL=0 drops the attribute.
  static const int pair_pdl = [] {
    const char* e1 = getenv("NASPIPE_PAIR_PDL");
    return (e1 && e1[0] == '0') ? 0 : 1;
  }();
  static const int pair_trig = [] {
    const char* e2 = getenv("NASPIPE_PAIR_TRIGGER");
    return (e2 && e2[0] == '1') ? 1 : 0;
  }();
  if (pdl_enabled() && pair_pdl) {
    cfg.attrs = at;
    cfg.numAttrs = 2;
  } else {
    cfg.attrs = at + 1;
    cfg.numAttrs = 1;
  }
  const cudaError_t e = cudaLaunchKernelEx(&cfg, kern, ta, tb, M, N, ts, ep, pair_trig);
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "pair GEMM launch: %s", cudaGetErrorString(e));
  g_gemm_launches.fetch_add(1, std::memory_order_relaxed);
}

template <bool A_MN, bool B_MN>
void dispatch_pair(cudaStream_t s, int M, int N, const TileSpace& ts, const CUtensorMap& ta, const CUtensorMap& tb,
                   int epi, const GemmEpiParams& ep) {
  switch (epi) {
    case EPI_BF16: return launch_pair<A_MN, B_MN, EPI_BF16>(s, M, N, ts, ta, tb, ep);
    case EPI_F32: return launch_pair<A_MN, B_MN, EPI_F32>(s, M, N, ts, ta, tb, ep);
    case EPI_BIAS_BF16: return launch_pair<A_MN, B_MN, EPI_BIAS_BF16>(s, M, N, ts, ta, tb, ep);
    case EPI_BIAS_RESID_F32: return launch_pair<A_MN, B_MN, EPI_BIAS_RESID_F32>(s, M, N, ts, ta, tb, ep);
    case EPI_BIAS_GELU: return launch_pair<A_MN, B_MN, EPI_BIAS_GELU>(s, M, N, ts, ta, tb, ep);
    case EPI_DGELU: return launch_pair<A_MN, B_MN, EPI_DGELU>(s, M, N, ts, ta, tb, ep);
    case EPI_SGD: return launch_pair<A_MN, B_MN, EPI_SGD>(s, M, N, ts, ta, tb, ep);
    case EPI_PARTIAL: return launch_pair<A_MN, B_MN, EPI_PARTIAL>(s, M, N, ts, ta, tb, ep);
    default: NP_REQUIRE(false, NASPIPE_EINVAL, "bad epilogue %d", epi);
  }
}

bool pair_enabled() {
  static const int v = [] {  // thread-safe one-time init
    const char* e = getenv("NASPIPE_GEMM_PAIR");
    return (e && e[0] == '0') ? 0 : 1;
  }();
  return v == 1;
}

// N tile of the 1-CTA kernel: narrow outputs (the SPOS 1x1-conv input gradients and weight
// gradients, N = C_in <= 320) get 64- or 128-wide tiles instead of wasting 3/4 or 1/2 of a
// 256-wide tile's MMA and TMEM work on zero columns (epilogues without per-column operands).
bool small_n_epi(int epi) {
  return epi == EPI_BF16 || epi == EPI_F32 || epi == EPI_SGD || epi == EPI_PARTIAL || epi == EPI_BNBWD;
}
int tile_n(int N, int epi) { return !small_n_epi(epi) ? BN : (N <= 64 ? 64 : (N <= 128 ? 128 : BN)); }

template <bool A_MN, bool B_MN, int TN>
void dispatch_narrow(cudaStream_t s, int M, int N, const TileSpace& ts, const CUtensorMap& ta, const CUtensorMap& tb,
                     int epi, const GemmEpiParams& ep) {
  switch (epi) {
    case EPI_BF16: return launch<A_MN, B_MN, EPI_BF16, TN>(s, M, N, ts, ta, tb, ep);
    case EPI_F32: return launch<A_MN, B_MN, EPI_F32, TN>(s, M, N, ts, ta, tb, ep);
    case EPI_SGD: return launch<A_MN, B_MN, EPI_SGD, TN>(s, M, N, ts, ta, tb, ep);
    case EPI_PARTIAL: return launch<A_MN, B_MN, EPI_PARTIAL, TN>(s, M, N, ts, ta, tb, ep);
    case EPI_BNBWD: return launch<A_MN, B_MN, EPI_BNBWD, TN>(s, M, N, ts, ta, tb, ep);
    default: NP_REQUIRE(false, NASPIPE_EINVAL, "narrow-tile epilogue %d", epi);
  }
}

template <bool A_MN, bool B_MN>
void dispatch_epi(cudaStream_t s, int M, int N, const TileSpace& ts, const CUtensorMap& ta, const CUtensorMap& tb,
                  int epi, const GemmEpiParams& ep) {
  const int tn = tile_n(N, epi);
  if (tn == 64) return dispatch_narrow<A_MN, B_MN, 64>(s, M, N, ts, ta, tb, epi, ep);
  if (tn == 128) return dispatch_narrow<A_MN, B_MN, 128>(s, M, N, ts, ta, tb, epi, ep);
  switch (epi) {
    case EPI_BF16: return launch<A_MN, B_MN, EPI_BF16>(s, M, N, ts, ta, tb, ep);
    case EPI_F32: return launch<A_MN, B_MN, EPI_F32>(s, M, N, ts, ta, tb, ep);
    case EPI_BIAS_BF16: return launch<A_MN, B_MN, EPI_BIAS_BF16>(s, M, N, ts, ta, tb, ep);
    case EPI_BIAS_RESID_F32: return launch<A_MN, B_MN, EPI_BIAS_RESID_F32>(s, M, N, ts, ta, tb, ep);
    case EPI_BIAS_GELU: return launch<A_MN, B_MN, EPI_BIAS_GELU>(s, M, N, ts, ta, tb, ep);
    case EPI_DGELU: return launch<A_MN, B_MN, EPI_DGELU>(s, M, N, ts, ta, tb, ep);
    case EPI_SGD: return launch<A_MN, B_MN, EPI_SGD>(s, M, N, ts, ta, tb, ep);
    case EPI_PARTIAL: return launch<A_MN, B_MN, EPI_PARTIAL>(s, M, N, ts, ta, tb, ep);
    case EPI_BNBWD: return launch<A_MN, B_MN, EPI_BNBWD>(s, M, N, ts, ta, tb, ep);
    default: NP_REQUIRE(false, NASPIPE_EINVAL, "bad epilogue %d", epi);
  }
}

}  // namespace

int num_sms() {
  static const int n = [] {
    int dev = 0, v = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    return v > 0 ? v : 148;
  }();
  return n;
}

CUtensorMap tma_map_bf16(const bf16* base, uint64_t inner, uint64_t outer, uint64_t ld, uint32_t box_outer) {
  return make_map(base, inner, outer, ld, box_outer);
}

void gemm_set_stream_cap(cudaStream_t s, int max_ctas) {
  std::lock_guard<std::mutex> lk(g_cap_mu);
  for (auto& c : g_caps)
    if (c.first == s) {
      c.second = max_ctas;
      return;
    }
  g_caps.emplace_back(s, max_ctas);
}

int side_stream_sms() {
  static const int v = [] {
    const char* e = getenv("NASPIPE_SIDE_SMS");
    return e ? std::max(0, atoi(e)) : 0;
  }();
  return v;
}

uint64_t gemm_launch_count() { return g_gemm_launches.load(); }
uint64_t gemm_flop_count() { return g_gemm_flops.load(); }

// The CTA-pair kernel serves every GEMM with M, N >= 256 (the transformer's and the SPOS
// head's); smaller ones (SPOS 1x1 convs with N < 256, the 3-pass product) use 1-CTA tiles.
bool gemm_uses_pair(int M, int N) { return pair_enabled() && M >= 256 && N >= 256; }

int gemm_splitk_factor(int M, int N, int K) {
  const bool pair = gemm_uses_pair(M, N);
  const int bm = pair ? 2 * BM : BM;
  const int bn = pair ? BN : tile_n(N, EPI_PARTIAL);  // split-K runs the partial epilogue
  const int tiles = ((M + bm - 1) / bm) * ((N + bn - 1) / bn);
  const int nk = (K + BK - 1) / BK;
  const int sms = pair ? num_sms() / 2 : num_sms();
  // cost in k-block rounds (~0.3 us each): rounds * k-blocks per round, plus the fp32
  // round trip of the split-K reduction ((s + 2.5) * M * N * 4 bytes at ~6 TB/s)
  auto cost = [&](int s) {
    const double rounds = (double)((tiles * s + sms - 1) / sms);
    const double red_us = s > 1 ? (s + 2.5) * 4.0 * M * (double)N / 6e12 * 1e6 : 0.0;
    return rounds * ((nk + s - 1) / s) + red_us / 0.3;
  };
  int best = 1;
  for (int s = 2; s <= 256; s *= 2)
    if (nk / s >= 8 && cost(s) < 0.9 * cost(best)) best = s;
  return best;
}

void gemm_bf16_tc(cudaStream_t s, int M, int N, int K, const bf16* A, bool a_mn, int lda, const bf16* B,
                  bool b_mn, int ldb, int epi, const GemmEpiParams& ep_in) {
  NP_REQUIRE(M > 0 && N > 0 && K > 0 && N % 16 == 0, NASPIPE_EINVAL, "gemm dims M=%d N=%d K=%d (N%%16)", M, N, K);
  GemmEpiParams ep = ep_in;
  g_gemm_flops.fetch_add(2ull * (uint64_t)M * (uint64_t)N * (uint64_t)K, std::memory_order_relaxed);
  // the fused BatchNorm-backward epilogue exists in the 1-CTA kernel only
  const bool pair = gemm_uses_pair(M, N) && epi != EPI_BNBWD;
  NP_REQUIRE(epi != EPI_BNBWD || (ep.bnb.acc != nullptr && ep.bnb.z != nullptr && N % 4 == 0), NASPIPE_EINVAL,
             "EPI_BNBWD needs bnb.acc / bnb.z (N=%d)", N);
  int splits = 1;
  if ((epi == EPI_SGD || epi == EPI_F32) && ep.ws != nullptr) {
    splits = gemm_splitk_factor(M, N, K);
    if ((size_t)splits * M * N > ep.ws_elems || (M * (size_t)N) % 4 != 0) splits = 1;
    static const bool no_split = getenv("NASPIPE_NO_SPLITK") != nullptr;  // diagnostics
    if (no_split) splits = 1;
  }
  const int tn = pair ? BN : tile_n(N, splits > 1 ? EPI_PARTIAL : epi);
  const CUtensorMap ta = a_mn ? make_map(A, (uint64_t)M, (uint64_t)K, (uint64_t)lda, BK)
                              : make_map(A, (uint64_t)K, (uint64_t)M, (uint64_t)lda, BM);
  const CUtensorMap tb = b_mn ? make_map(B, (uint64_t)N, (uint64_t)K, (uint64_t)ldb, BK)
                              : make_map(B, (uint64_t)K, (uint64_t)N, (uint64_t)ldb, pair ? BN / 2 : tn);
  TileSpace ts;
  ts.MT = (M + (pair ? 2 * BM : BM) - 1) / (pair ? 2 * BM : BM);
  ts.NT = (N + tn - 1) / tn;
  ts.nk = (K + BK - 1) / BK;
  ts.splits = splits;
  ts.nk_per_split = (ts.nk + ts.splits - 1) / ts.splits;
  // effective split count: every split owns >= 1 k-block (with ceil-sized splits the last
  // ones could otherwise be empty and leave their workspace slice unwritten)
  ts.splits = (ts.nk + ts.nk_per_split - 1) / ts.nk_per_split;
  const int run_epi = ts.splits > 1 ? EPI_PARTIAL : epi;
  ep.ws_stride = (size_t)M * N;
  if (pair) {
    if (!a_mn && !b_mn) dispatch_pair<false, false>(s, M, N, ts, ta, tb, run_epi, ep);
    else if (!a_mn && b_mn) dispatch_pair<false, true>(s, M, N, ts, ta, tb, run_epi, ep);
    else if (a_mn && b_mn) dispatch_pair<true, true>(s, M, N, ts, ta, tb, run_epi, ep);
    else dispatch_pair<true, false>(s, M, N, ts, ta, tb, run_epi, ep);
  } else if (!a_mn && !b_mn) dispatch_epi<false, false>(s, M, N, ts, ta, tb, run_epi, ep);
  else if (!a_mn && b_mn) dispatch_epi<false, true>(s, M, N, ts, ta, tb, run_epi, ep);
  else if (a_mn && b_mn) dispatch_epi<true, true>(s, M, N, ts, ta, tb, run_epi, ep);
  else dispatch_epi<true, false>(s, M, N, ts, ta, tb, run_epi, ep);
  if (ts.splits > 1) {
    int L = 1;  // lanes per output vector: a power of two (xor tree), <= splits / 4
    while (2 * L <= 32 && 2 * L <= ts.splits / 4) L *= 2;
    const size_t per_block = 256 / L;
    static const int per_sm = [] {  // CTAs per SM of the reduce; NASPIPE_SPLITK_CTAS_PER_SM overrides (tuning)
      const char* e = getenv("NASPIPE_SPLITK_CTAS_PER_SM");
      return e ? std::max(1, atoi(e)) : 4;
    }();
    const int blocks = (int)std::min<size_t>(((size_t)M * N / 4 + per_block - 1) / per_block, (size_t)per_sm * num_sms());
    if (epi == EPI_F32)
      launch_pdl(splitk_reduce_kernel<EPI_F32>, dim3(blocks), dim3(256), 0, s, M, N, ts.splits, L, ep);
    else
      launch_pdl(splitk_reduce_kernel<EPI_SGD>, dim3(blocks), dim3(256), 0, s, M, N, ts.splits, L, ep);
  }
}

void gemm_bf16x2_tc(cudaStream_t s, int M, int N, int K, const bf16* A_hi, const bf16* A_lo, int lda,
                    const bf16* B_hi, const bf16* B_lo, int ldb, int epi, const GemmEpiParams& ep) {
  NP_REQUIRE(M > 0 && N > 0 && K > 0 && N % 16 == 0, NASPIPE_EINVAL, "gemm x2 dims M=%d N=%d K=%d (N%%16)", M, N, K);
  NP_REQUIRE(epi == EPI_X2 || epi == EPI_BF16 || epi == EPI_F32, NASPIPE_EINVAL, "gemm x2 epilogue %d", epi);
  g_gemm_flops.fetch_add(2ull * (uint64_t)M * (uint64_t)N * (uint64_t)K, std::memory_order_relaxed);
  const int tn = N <= 64 ? 64 : (N <= 128 ? 128 : 256);
  const CUtensorMap ta = make_map(A_hi, (uint64_t)K, (uint64_t)M, (uint64_t)lda, BM);
  const CUtensorMap ta2 = make_map(A_lo, (uint64_t)K, (uint64_t)M, (uint64_t)lda, BM);
  const CUtensorMap tb = make_map(B_hi, (uint64_t)K, (uint64_t)N, (uint64_t)ldb, tn);
  const CUtensorMap tb2 = make_map(B_lo, (uint64_t)K, (uint64_t)N, (uint64_t)ldb, tn);
  TileSpace ts;
  ts.MT = (M + BM - 1) / BM;
  ts.NT = (N + tn - 1) / tn;
  ts.nk = (K + BK - 1) / BK;
  ts.splits = 1;
  ts.nk_per_split = ts.nk;
  GemmEpiParams e = ep;
  e.ws_stride = (size_t)M * N;
#define X2_CASE(TNV)                                                                       \
  if (tn == TNV) {                                                                         \
    if (epi == EPI_X2) launch<false, false, EPI_X2, TNV, true>(s, M, N, ts, ta, tb, e, &ta2, &tb2);   \
    else if (epi == EPI_BF16) launch<false, false, EPI_BF16, TNV, true>(s, M, N, ts, ta, tb, e, &ta2, &tb2); \
    else launch<false, false, EPI_F32, TNV, true>(s, M, N, ts, ta, tb, e, &ta2, &tb2);    \
    return;                                                                                \
  }
  X2_CASE(64)
  X2_CASE(128)
  X2_CASE(256)
#undef X2_CASE
}

}  // namespace naspipe
