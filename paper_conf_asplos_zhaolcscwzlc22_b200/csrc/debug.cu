// Kernel-level C entry points for the kernel unit tests (include/naspipe_debug.h).
#include <vector>

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


int naspipe_debug_dw(const void* x, const float* w, void* z, const void* dz, const void* add, void* dx,
                     float* dwsum, int B, int H, int C, int k, int S, int dil, void* stream) {
  return dguard([&] {
    cudaStream_t s = (cudaStream_t)stream;
    if (x && z) dw_fwd(s, (const bf16*)x, w, (bf16*)z, B, H, C, k, S, dil);
    if (dz && dx) dw_dgrad(s, (const bf16*)dz, w, (const bf16*)add, (bf16*)dx, B, H, C, k, S, dil);
    if (dz && x && dwsum) {
      unsigned long long* acc = nullptr;
      int* ticket = nullptr;
      NP_REQUIRE(cudaMalloc(&acc, ((size_t)C * k * k + 1) * 8) == cudaSuccess, NASPIPE_ENOMEM, "malloc");
      NP_REQUIRE(cudaMalloc(&ticket, 4) == cudaSuccess, NASPIPE_ENOMEM, "malloc");
      cudaMemsetAsync(acc, 0, ((size_t)C * k * k + 1) * 8, s);
      cudaMemsetAsync(ticket, 0, 4, s);
      cudaMemsetAsync(dwsum, 0, (size_t)C * k * k * 4, s);
      dw_wgrad_sgd(s, (const bf16*)dz, (const bf16*)x, acc, ticket, dwsum, -1.0f, B, H, C, k, S, dil);  // 0 + sum
      cudaStreamSynchronize(s);
      cudaFree(acc);
      cudaFree(ticket);
    }
  });
}

int naspipe_debug_bn_fwd(const void* z, int P, int C, const float* g, const float* b, int relu, void* y, int ldy,
                         size_t yplane, float* mean, float* rstd, void* stream) {
  return dguard([&] {
    cudaStream_t s = (cudaStream_t)stream;
    unsigned long long* acc = nullptr;
    int* ticket = nullptr;
    NP_REQUIRE(cudaMalloc(&acc, (size_t)2 * C * 8) == cudaSuccess, NASPIPE_ENOMEM, "malloc");
    NP_REQUIRE(cudaMalloc(&ticket, 4) == cudaSuccess, NASPIPE_ENOMEM, "malloc");
    cudaMemsetAsync(acc, 0, (size_t)2 * C * 8, s);
    cudaMemsetAsync(ticket, 0, 4, s);
    bn_stats(s, (const bf16*)z, P, C, acc);
    bn_apply(s, (const bf16*)z, P, C, acc, ticket, mean, rstd, g, b, relu, (bf16*)y, ldy, yplane);
    cudaStreamSynchronize(s);
    cudaFree(acc);
    cudaFree(ticket);
  });
}

// sums [2][C] (s1, s2) and old [2][C] (g, b before the WRITE) are reported for the tests
int naspipe_debug_bn_bwd(const void* dy, int lddy, const void* z, int P, int C, const float* mean,
                         const float* rstd, float* g, float* b, int relu, void* dz, float* sums, float* old, float lr,
                         int update, void* stream) {
  return dguard([&] {
    cudaStream_t s = (cudaStream_t)stream;
    unsigned long long* acc = nullptr;
    int* ticket = nullptr;
    NP_REQUIRE(cudaMalloc(&acc, (size_t)2 * C * 8) == cudaSuccess, NASPIPE_ENOMEM, "malloc");
    NP_REQUIRE(cudaMalloc(&ticket, 4) == cudaSuccess, NASPIPE_ENOMEM, "malloc");
    cudaMemsetAsync(acc, 0, (size_t)2 * C * 8, s);
    cudaMemsetAsync(ticket, 0, 4, s);
    cudaMemcpyAsync(old, g, (size_t)C * 4, cudaMemcpyDeviceToDevice, s);
    cudaMemcpyAsync(old + C, b, (size_t)C * 4, cudaMemcpyDeviceToDevice, s);
    bn_bwd_reduce(s, (const bf16*)dy, lddy, (const bf16*)z, P, C, mean, rstd, g, b, relu, acc);
    cudaStreamSynchronize(s);
    std::vector<unsigned long long> h(2 * (size_t)C);
    cudaMemcpy(h.data(), acc, h.size() * 8, cudaMemcpyDeviceToHost);
    std::vector<float> f(h.size());
    for (size_t i = 0; i < h.size(); ++i) f[i] = (float)((double)(long long)h[i] / 1099511627776.0);
    cudaMemcpy(sums, f.data(), f.size() * 4, cudaMemcpyHostToDevice);
    bn_bwd_apply(s, (const bf16*)dy, lddy, (const bf16*)z, P, C, mean, rstd, g, b, g, b, lr, update, acc, ticket, relu,
                 (bf16*)dz);
    cudaStreamSynchronize(s);
    cudaFree(acc);
    cudaFree(ticket);
  });
}

int naspipe_debug_dense_cols(const void* x, void* cols, const float* dcols, const void* add, void* dx, int B, int H,
                             int C, int k, int S, void* stream) {
  return dguard([&] {
    cudaStream_t s = (cudaStream_t)stream;
    const int Ho = (H - 1) / S + 1;
    if (x && cols)
      im2col_x2(s, (const bf16*)x, (size_t)B * H * H * C, B, H, C, k, S, (bf16*)cols, (size_t)B * Ho * Ho * k * k * C);
    if (dcols && dx) col2im(s, dcols, B, H, C, k, S, (const bf16*)add, (bf16*)dx);
  });
}

int naspipe_debug_dw_bn_fold(const void* zin, int B, int H, int C, const float* g, const float* b, int relu,
                             const float* w, int k, int S, int dil, const void* dz, void* out_ref, void* out,
                             float* dwsum_ref, float* dwsum, float* meta, float* mean_ref, float* rstd_ref,
                             void* stream) {
  return dguard([&] {
    cudaStream_t s = (cudaStream_t)stream;
    const int P = B * H * H;
    const size_t n = (size_t)P * C;
    unsigned long long *acc = nullptr, *acc2 = nullptr, *wacc = nullptr;
    int* tick = nullptr;
    bf16* y = nullptr;
    NP_REQUIRE(cudaMalloc(&acc, (2 * (size_t)C + 1) * 8) == cudaSuccess && cudaMalloc(&acc2, (2 * (size_t)C + 1) * 8) == cudaSuccess &&
                   cudaMalloc(&wacc, ((size_t)C * k * k + 1) * 8) == cudaSuccess && cudaMalloc(&tick, 16) == cudaSuccess &&
                   cudaMalloc(&y, 2 * n * sizeof(bf16)) == cudaSuccess,
               NASPIPE_ENOMEM, "malloc");
    cudaMemsetAsync(acc, 0, (2 * (size_t)C + 1) * 8, s);
    cudaMemsetAsync(acc2, 0, (2 * (size_t)C + 1) * 8, s);
    cudaMemsetAsync(wacc, 0, ((size_t)C * k * k + 1) * 8, s);
    cudaMemsetAsync(tick, 0, 16, s);
    cudaMemsetAsync(dwsum_ref, 0, (size_t)C * k * k * 4, s);
    cudaMemsetAsync(dwsum, 0, (size_t)C * k * k * 4, s);
    // stored path
    bn_stats(s, (const bf16*)zin, P, C, acc);
    bn_apply(s, (const bf16*)zin, P, C, acc, tick, mean_ref, rstd_ref, g, b, relu, y, C, n);
    dw_fwd(s, y, w, (bf16*)out_ref, B, H, C, k, S, dil, acc2);
    cudaMemsetAsync(acc2, 0, (2 * (size_t)C + 1) * 8, s);
    dw_wgrad_sgd(s, (const bf16*)dz, y, wacc, tick + 1, dwsum_ref, -1.0f, B, H, C, k, S, dil);  // 0 + sum
    // folded path
    BnApplyIn xin;
    xin.z = (const bf16*)zin;
    xin.zplane = n;
    xin.P = P;
    xin.acc = acc;
    xin.ticket = tick + 2;
    xin.mean = meta;
    xin.rstd = meta + C;
    xin.g = g;
    xin.b = b;
    xin.gsnap = meta + 2 * C;
    xin.bsnap = meta + 3 * C;
    xin.relu = relu;
    bn_stats(s, (const bf16*)zin, P, C, acc);
    dw_fwd_bn(s, xin, w, (bf16*)out, B, H, C, k, S, dil, acc2);
    dw_wgrad_sgd(s, (const bf16*)dz, nullptr, wacc, tick + 1, dwsum, -1.0f, B, H, C, k, S, dil, &xin);
    cudaStreamSynchronize(s);
    std::vector<unsigned long long> h(2 * (size_t)C);
    cudaMemcpy(h.data(), acc, h.size() * 8, cudaMemcpyDeviceToHost);
    for (auto v : h) NP_REQUIRE(v == 0, NASPIPE_EINTERNAL, "dw_fwd_bn left its input sums uncleared");
    cudaFree(acc);
    cudaFree(acc2);
    cudaFree(wacc);
    cudaFree(tick);
    cudaFree(y);
  });
}

int naspipe_debug_bnb_fused(int kind, const void* dz, const float* w, const void* w16, void* dx, int B, int H, int C,
                            int Cout, int k, int dil, const void* z, const float* mean, const float* rstd,
                            const float* g, const float* b, int relu, float* sums, void* stream) {
  return dguard([&] {
    cudaStream_t s = (cudaStream_t)stream;
    const int P = B * H * H;
    unsigned long long* acc = nullptr;
    NP_REQUIRE(cudaMalloc(&acc, (2 * (size_t)C + 1) * 8) == cudaSuccess, NASPIPE_ENOMEM, "malloc");
    cudaMemsetAsync(acc, 0, (2 * (size_t)C + 1) * 8, s);
    BnBwdFuse f;
    f.z = (const bf16*)z;
    f.zplane = (size_t)P * C;
    f.mean = mean;
    f.rstd = rstd;
    f.g = g;
    f.b = b;
    f.relu = relu;
    f.acc = acc;
    if (kind == 0 || kind == 2) {
      dw_dgrad(s, (const bf16*)dz, w, nullptr, (bf16*)dx, B, H, C, k, kind == 2 ? 2 : 1, dil, f);
    } else {
      GemmEpiParams e;
      e.out = dx;
      e.bnb = f;
      gemm_bf16_tc(s, P, C, Cout, (const bf16*)dz, false, Cout, (const bf16*)w16, true, C, EPI_BNBWD, e);
    }
    cudaStreamSynchronize(s);
    std::vector<unsigned long long> h(2 * (size_t)C + 1);
    cudaMemcpy(h.data(), acc, h.size() * 8, cudaMemcpyDeviceToHost);
    NP_REQUIRE(h[2 * (size_t)C] == 0, NASPIPE_EINTERNAL, "fixed-point overflow flag set");
    std::vector<float> fs(2 * (size_t)C);
    for (size_t i = 0; i < fs.size(); ++i) fs[i] = (float)((double)(long long)h[i] / 1099511627776.0);
    cudaMemcpy(sums, fs.data(), fs.size() * 4, cudaMemcpyHostToDevice);
    cudaFree(acc);
  });
}

int naspipe_debug_chan_split(const void* x, int P, int Ch, void* out, int ldo, size_t oplane, void* xm,
                             void* stream) {
  return dguard([&] { chan_split((cudaStream_t)stream, (const bf16*)x, P, Ch, (bf16*)out, ldo, oplane, (bf16*)xm); });
}

int naspipe_debug_gemm_x2(int M, int N, int K, const void* A_hi, const void* A_lo, int lda, const void* B_hi,
                          const void* B_lo, int ldb, void* out_hi, void* out_lo, void* stream) {
  return dguard([&] {
    GemmEpiParams ep;
    ep.out = out_hi;
    ep.out2 = static_cast<bf16*>(out_lo);
    gemm_bf16x2_tc((cudaStream_t)stream, M, N, K, (const bf16*)A_hi, (const bf16*)A_lo, lda, (const bf16*)B_hi,
                   (const bf16*)B_lo, ldb, EPI_X2, ep);
  });
}

int naspipe_debug_chan_merge(const void* dproj, int ldp, const void* dm, int P, int Ch, void* dx, void* stream) {
  return dguard([&] { chan_merge((cudaStream_t)stream, (const bf16*)dproj, ldp, (const bf16*)dm, P, Ch, (bf16*)dx); });
}

int naspipe_debug_stem(const float* x, const float* w, void* z, int B, int H, int C0, void* stream) {
  return dguard([&] { spos_stem_conv((cudaStream_t)stream, x, w, (bf16*)z, B, H, C0); });
}

}  // extern "C"
