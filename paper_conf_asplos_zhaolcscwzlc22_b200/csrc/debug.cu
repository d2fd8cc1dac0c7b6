// Kernel-level C entry points for the kernel unit tests (include/naspipe_debug.h).
#include "common.h"
#include "kernels.h"
#include "naspipe_debug.h"

using namespace naspipe;

namespace naspipe {
void set_last_error(const std::string& msg);
}

template <class F>
static int dguard(F&& f) {
  try {
    f();
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) throw Error(NASPIPE_ECUDA, cudaGetErrorString(e));
    return NASPIPE_OK;
  } catch (const Error& e) {
    set_last_error(e.what());
    return e.code;
  } catch (const std::exception& e) {
    set_last_error(e.what());
    return NASPIPE_EINTERNAL;
  }
}

extern "C" {

int naspipe_debug_gemm(int M, int N, int K, const void* A, int a_mn, int lda, const void* B, int b_mn, int ldb,
                       int epi, const float* bias, const float* resid, const void* aux16, void* out, void* out2,
                       float* w32, void* w16, float lr, void* stream) {
  return dguard([&] {
    GemmEpiParams ep;
    ep.bias = bias;
    ep.resid = resid;
    ep.aux16 = static_cast<const bf16*>(aux16);
    ep.out = out;
    ep.out2 = static_cast<bf16*>(out2);
    ep.w32 = w32;
    ep.w16 = static_cast<bf16*>(w16);
    ep.lr = lr;
    // exercise split-K exactly as the engine would (workspace of splits * M * N floats)
    const int splits = gemm_splitk_factor(M, N, K);
    cudaStream_t s = (cudaStream_t)stream;
    static float* ws = nullptr;  // grown on demand, kept for the process (test helper)
    static size_t ws_cap = 0;
    if (splits > 1 && (epi == EPI_F32 || epi == EPI_SGD)) {
      const size_t need = (size_t)splits * M * N;
      if (need > ws_cap) {
        cudaDeviceSynchronize();
        if (ws) cudaFree(ws);
        NP_REQUIRE(cudaMalloc(&ws, need * 4) == cudaSuccess, NASPIPE_ENOMEM, "ws");
        ws_cap = need;
      }
      ep.ws = ws;
      ep.ws_elems = ws_cap;
    }
    gemm_bf16_tc(s, M, N, K, static_cast<const bf16*>(A), a_mn != 0, lda, static_cast<const bf16*>(B), b_mn != 0,
                 ldb, epi, ep);
  });
}

int naspipe_debug_attn_fwd(const void* qkv, void* o, float* lse, int B, int S, int d, int h, void* stream) {
  return dguard([&] {
    attn_fwd((cudaStream_t)stream, static_cast<const bf16*>(qkv), static_cast<bf16*>(o), lse, B, S, d, h);
  });
}

int naspipe_debug_attn_bwd(const void* qkv, const void* o, const float* lse, const void* dout, void* dqkv, int B,
                           int S, int d, int h, void* stream) {
  return dguard([&] {
    attn_bwd((cudaStream_t)stream, static_cast<const bf16*>(qkv), static_cast<const bf16*>(o), lse,
             static_cast<const bf16*>(dout), static_cast<bf16*>(dqkv), B, S, d, h);
  });
}

int naspipe_debug_ln_fwd(const float* x, const float* g, const float* b, void* y16, float* mean, float* rstd, int T,
                         int d, void* stream) {
  return dguard([&] { ln_fwd((cudaStream_t)stream, x, g, b, static_cast<bf16*>(y16), mean, rstd, T, d); });
}

int naspipe_debug_ln_bwd(const float* dy, const float* x, const float* mean, const float* rstd, const float* g,
                         const float* resid, float* dx, void* dx16, float* dgamma, float* dbeta, float* colsum,
                         int T, int d, void* stream) {
  return dguard([&] {
    cudaStream_t s = (cudaStream_t)stream;
    const int nb = ln_bwd_blocks(T);
    float* part = nullptr;
    NP_REQUIRE(cudaMallocAsync(&part, sizeof(float) * 3 * (size_t)nb * d, s) == cudaSuccess, NASPIPE_ENOMEM,
               "workspace");
    ln_bwd(s, dy, x, mean, rstd, g, resid, dx, static_cast<bf16*>(dx16), part, part + (size_t)nb * d,
           part + 2 * (size_t)nb * d, T, d);
    cudaMemsetAsync(dgamma, 0, d * 4, s);
    cudaMemsetAsync(dbeta, 0, d * 4, s);
    cudaMemsetAsync(colsum, 0, d * 4, s);
    sgd_from_partials(s, dgamma, part, nb, d, -1.0f);  // p -= (-1) * sum  ==  sum
    sgd_from_partials(s, dbeta, part + (size_t)nb * d, nb, d, -1.0f);
    sgd_from_partials(s, colsum, part + 2 * (size_t)nb * d, nb, d, -1.0f);
    cudaFreeAsync(part, s);
  });
}

}  // extern "C"
