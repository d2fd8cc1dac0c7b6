// tcgen05 GEMM for sm_100a: TMA (128B swizzle) -> shared memory ring -> single-thread
// tcgen05.mma (M=128, N=BN, K=16 per instruction) accumulating in TMEM -> fused epilogue
// (bias / residual / GELU / GELU' / SGD update) from tcgen05.ld.
//
// Warp roles (128 threads): warp 0 lane 0 = TMA producer, warp 1 lane 0 = MMA issuer,
// warp 2 = TMEM allocator; after the main loop all four warps run the epilogue, warp w
// owning accumulator rows (TMEM lanes) 32w..32w+31.  One output tile per CTA; the kernel
// is sized so that two CTAs co-reside per SM, overlapping one CTA's epilogue with the
// other's main loop.  Every output element is produced by exactly one CTA with a fixed K
// order, so results are bitwise deterministic.
#include <cuda.h>

#include <atomic>
#include <mutex>

#include "common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace naspipe {

namespace {

constexpr int BM = 128;
constexpr int BK = 64;  // 64 bf16 = 128 B = one swizzle row

__device__ __forceinline__ float gelu_tanh(float z) {
  const float c = 0.7978845608028654f;
  const float u = c * (z + 0.044715f * z * z * z);
  return 0.5f * z * (1.f + tanhf(u));
}
__device__ __forceinline__ float gelu_tanh_grad(float z) {
  const float c = 0.7978845608028654f;
  const float t = tanhf(c * (z + 0.044715f * z * z * z));
  return 0.5f * (1.f + t) + 0.5f * z * (1.f - t * t) * c * (1.f + 3.f * 0.044715f * z * z);
}

template <int BN, int STAGES>
struct GemmSmem {
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int BAR_OFF = STAGES * STAGE_BYTES;
  static constexpr int TOTAL = BAR_OFF + (2 * STAGES + 1) * 8 + 16 + 1024;  // +1024 alignment slack
};

template <int BN, int STAGES, bool A_MN, bool B_MN, int EPI>
__global__ void __launch_bounds__(128, 2)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb, int M,
                   int N, int K, GemmEpiParams ep) {
  using L = GemmSmem<BN, STAGES>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + L::BAR_OFF);
  uint64_t* empty = full + STAGES;
  uint64_t* tmem_full = empty + STAGES;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(tmem_full + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
  const int nk = (K + BK - 1) / BK;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&ta);
    ptx::tma_prefetch(&tb);
    for (int s = 0; s < STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    ptx::mbar_init(tmem_full, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 2) ptx::tmem_alloc<BN>(tmem_holder);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp == 0 && lane == 0) {
    // ---------------- TMA producer
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % STAGES;
      if (kb >= STAGES) ptx::mbar_wait(&empty[s], ((kb / STAGES) - 1) & 1);
      uint8_t* sa = smem + s * L::STAGE_BYTES;
      uint8_t* sb = sa + L::A_BYTES;
      ptx::mbar_arrive_expect_tx(&full[s], L::STAGE_BYTES);
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
        for (int j = 0; j < BN / 64; ++j) ptx::tma_load_2d(sb + j * 8192, &tb, &full[s], n0 + 64 * j, k0);
      }
    }
  } else if (warp == 1 && lane == 0) {
    // ---------------- MMA issuer
    constexpr uint32_t idesc = ptx::umma_idesc_bf16(BM, BN, A_MN ? 1 : 0, B_MN ? 1 : 0);
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % STAGES;
      ptx::mbar_wait(&full[s], (kb / STAGES) & 1);
      ptx::tc_fence_after();
      const uint32_t sa = ptx::smem_u32(smem + s * L::STAGE_BYTES);
      const uint32_t sb = sa + L::A_BYTES;
#pragma unroll
      for (int k = 0; k < BK / 16; ++k) {
        // K-major: rows of 128 B, 8-row groups 1024 B apart; a K step of 16 = +32 B.
        // MN-major: 64-element MN chunks 8 KB apart (LBO), 8 K-rows = 1024 B (SBO);
        //           a K step of 16 rows = +2048 B.
        const uint64_t ad = A_MN ? ptx::umma_desc_sw128(sa + k * 2048, 8192, 1024)
                                 : ptx::umma_desc_sw128(sa + k * 32, 16, 1024);
        const uint64_t bd = B_MN ? ptx::umma_desc_sw128(sb + k * 2048, 8192, 1024)
                                 : ptx::umma_desc_sw128(sb + k * 32, 16, 1024);
        ptx::umma_bf16(tmem, ad, bd, idesc, (kb | k) != 0 ? 1u : 0u);
      }
      ptx::umma_commit(&empty[s]);  // frees the smem stage when these MMAs complete
    }
    ptx::umma_commit(tmem_full);
  }
  __syncwarp();

  // ---------------- epilogue: all 4 warps
  ptx::mbar_wait(tmem_full, 0);
  ptx::tc_fence_after();
  const int row = m0 + warp * 32 + lane;
  const bool row_ok = row < M;
#pragma unroll 1
  for (int c0 = 0; c0 < BN; c0 += 16) {
    uint32_t r[16];
    ptx::tmem_ld16(tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0, r);
    ptx::tmem_ld_wait();
    const int col = n0 + c0;
    if (!row_ok || col >= N) continue;
    float v[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
    const size_t off = (size_t)row * N + col;
    if constexpr (EPI == EPI_BIAS_BF16 || EPI == EPI_BIAS_RESID_F32 || EPI == EPI_BIAS_GELU) {
      const float4* b4 = reinterpret_cast<const float4*>(ep.bias + col);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float4 b = b4[i];
        v[4 * i] += b.x; v[4 * i + 1] += b.y; v[4 * i + 2] += b.z; v[4 * i + 3] += b.w;
      }
    }
    if constexpr (EPI == EPI_BIAS_RESID_F32) {
      const float4* r4 = reinterpret_cast<const float4*>(ep.resid + off);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float4 q = r4[i];
        v[4 * i] += q.x; v[4 * i + 1] += q.y; v[4 * i + 2] += q.z; v[4 * i + 3] += q.w;
      }
    }
    if constexpr (EPI == EPI_DGELU) {
      const uint4* z4 = reinterpret_cast<const uint4*>(ep.aux16 + off);
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        uint4 q = z4[i];
        const __nv_bfloat16* zz = reinterpret_cast<const __nv_bfloat16*>(&q);
#pragma unroll
        for (int j = 0; j < 8; ++j) v[8 * i + j] *= gelu_tanh_grad(__bfloat162float(zz[j]));
      }
    }
    if constexpr (EPI == EPI_F32 || EPI == EPI_BIAS_RESID_F32) {
      float4* o4 = reinterpret_cast<float4*>(reinterpret_cast<float*>(ep.out) + off);
#pragma unroll
      for (int i = 0; i < 4; ++i) o4[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
    } else if constexpr (EPI == EPI_SGD) {
      float4* w4 = reinterpret_cast<float4*>(ep.w32 + off);
      uint32_t p[8];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        float4 w = w4[i];
        w.x -= ep.lr * v[4 * i]; w.y -= ep.lr * v[4 * i + 1];
        w.z -= ep.lr * v[4 * i + 2]; w.w -= ep.lr * v[4 * i + 3];
        w4[i] = w;
        p[2 * i] = ptx::pack_bf16(w.x, w.y);
        p[2 * i + 1] = ptx::pack_bf16(w.z, w.w);
      }
      uint4* o4 = reinterpret_cast<uint4*>(ep.w16 + off);
      o4[0] = make_uint4(p[0], p[1], p[2], p[3]);
      o4[1] = make_uint4(p[4], p[5], p[6], p[7]);
    } else {
      uint32_t p[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) p[i] = ptx::pack_bf16(v[2 * i], v[2 * i + 1]);
      uint4* o4 = reinterpret_cast<uint4*>(reinterpret_cast<bf16*>(ep.out) + off);
      o4[0] = make_uint4(p[0], p[1], p[2], p[3]);
      o4[1] = make_uint4(p[4], p[5], p[6], p[7]);
      if constexpr (EPI == EPI_BIAS_GELU) {
#pragma unroll
        for (int i = 0; i < 8; ++i) p[i] = ptx::pack_bf16(gelu_tanh(v[2 * i]), gelu_tanh(v[2 * i + 1]));
        uint4* g4 = reinterpret_cast<uint4*>(ep.out2 + off);
        g4[0] = make_uint4(p[0], p[1], p[2], p[3]);
        g4[1] = make_uint4(p[4], p[5], p[6], p[7]);
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 2) ptx::tmem_dealloc<BN>(tmem);
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

template <int BN, int STAGES, bool A_MN, bool B_MN, int EPI>
void launch(cudaStream_t s, int M, int N, int K, const CUtensorMap& ta, const CUtensorMap& tb,
            const GemmEpiParams& ep) {
  using L = GemmSmem<BN, STAGES>;
  auto kern = gemm_tc_kernel<BN, STAGES, A_MN, B_MN, EPI>;
  static bool configured = false;  // per instantiation
  if (!configured) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, L::TOTAL);
    configured = true;
  }
  dim3 grid((N + BN - 1) / BN, (M + BM - 1) / BM);
  kern<<<grid, 128, L::TOTAL, s>>>(ta, tb, M, N, K, ep);
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "gemm launch: %s", cudaGetErrorString(e));
  g_gemm_launches.fetch_add(1, std::memory_order_relaxed);
}

template <bool A_MN, bool B_MN>
void dispatch_epi(cudaStream_t s, int M, int N, int K, const CUtensorMap& ta, const CUtensorMap& tb, int epi,
                  const GemmEpiParams& ep) {
  constexpr int BN = 128, ST = 3;
  switch (epi) {
    case EPI_BF16: return launch<BN, ST, A_MN, B_MN, EPI_BF16>(s, M, N, K, ta, tb, ep);
    case EPI_F32: return launch<BN, ST, A_MN, B_MN, EPI_F32>(s, M, N, K, ta, tb, ep);
    case EPI_BIAS_BF16: return launch<BN, ST, A_MN, B_MN, EPI_BIAS_BF16>(s, M, N, K, ta, tb, ep);
    case EPI_BIAS_RESID_F32: return launch<BN, ST, A_MN, B_MN, EPI_BIAS_RESID_F32>(s, M, N, K, ta, tb, ep);
    case EPI_BIAS_GELU: return launch<BN, ST, A_MN, B_MN, EPI_BIAS_GELU>(s, M, N, K, ta, tb, ep);
    case EPI_DGELU: return launch<BN, ST, A_MN, B_MN, EPI_DGELU>(s, M, N, K, ta, tb, ep);
    case EPI_SGD: return launch<BN, ST, A_MN, B_MN, EPI_SGD>(s, M, N, K, ta, tb, ep);
    default: NP_REQUIRE(false, NASPIPE_EINVAL, "bad epilogue %d", epi);
  }
}

}  // namespace

uint64_t gemm_launch_count() { return g_gemm_launches.load(); }

void gemm_bf16_tc(cudaStream_t s, int M, int N, int K, const bf16* A, bool a_mn, int lda, const bf16* B,
                  bool b_mn, int ldb, int epi, const GemmEpiParams& ep) {
  NP_REQUIRE(M > 0 && N > 0 && K > 0 && N % 16 == 0, NASPIPE_EINVAL, "gemm dims M=%d N=%d K=%d (N%%16)", M, N, K);
  constexpr int BN = 128;
  const CUtensorMap ta = a_mn ? make_map(A, (uint64_t)M, (uint64_t)K, (uint64_t)lda, BK)
                              : make_map(A, (uint64_t)K, (uint64_t)M, (uint64_t)lda, BM);
  const CUtensorMap tb = b_mn ? make_map(B, (uint64_t)N, (uint64_t)K, (uint64_t)ldb, BK)
                              : make_map(B, (uint64_t)K, (uint64_t)N, (uint64_t)ldb, BN);
  if (!a_mn && !b_mn) return dispatch_epi<false, false>(s, M, N, K, ta, tb, epi, ep);
  if (!a_mn && b_mn) return dispatch_epi<false, true>(s, M, N, K, ta, tb, epi, ep);
  if (a_mn && b_mn) return dispatch_epi<true, true>(s, M, N, K, ta, tb, epi, ep);
  return dispatch_epi<true, false>(s, M, N, K, ta, tb, epi, ep);
}

}  // namespace naspipe
