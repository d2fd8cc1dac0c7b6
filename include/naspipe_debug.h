/*
 * naspipe_debug.h — kernel-level entry points used by the kernel unit tests (SURVEY §4
 * tier T2).  Not part of the training API.  All pointers are DEVICE pointers on the
 * current CUDA device; every call enqueues on `stream` (a cudaStream_t, 0 = legacy default)
 * and returns naspipe_status (see naspipe.h).  bf16 buffers are raw 16-bit bfloat16.
 */
#ifndef NASPIPE_DEBUG_H_
#define NASPIPE_DEBUG_H_
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif
#if defined(__GNUC__)
#pragma GCC visibility push(default)
#endif

/* C[M,N] = sum_k A[m,k] B[n,k] on the tcgen05 path, with epilogue `epi` (kernels.h GemmEpi):
 * 0 bf16, 1 f32, 2 bias+bf16, 3 bias+resid f32, 4 bias+GELU (out=z, out2=g), 5 GELU' (aux=z),
 * 6 SGD (w32 -= lr*C, w16 = bf16(w32)).  a_mn / b_mn select MN-major operand storage. */
int naspipe_debug_gemm(int M, int N, int K, const void* A, int a_mn, int lda, const void* B, int b_mn, int ldb,
                       int epi, const float* bias, const float* resid, const void* aux16, void* out, void* out2,
                       float* w32, void* w16, float lr, void* stream);
int naspipe_debug_attn_fwd(const void* qkv, void* o, float* lse, int B, int S, int d, int h, void* stream);
int naspipe_debug_attn_bwd(const void* qkv, const void* o, const float* lse, const void* dout, void* dqkv, int B,
                           int S, int d, int h, void* stream);
int naspipe_debug_ln_fwd(const float* x, const float* g, const float* b, void* y16, float* mean, float* rstd, int T,
                         int d, void* stream);
/* dx = resid + LN'(dy); dgamma, dbeta, colsum(dx) reduced to [d] (fixed order) */
int naspipe_debug_ln_bwd(const float* dy, const float* x, const float* mean, const float* rstd, const float* g,
                         const float* resid, float* dx, void* dx16, float* dgamma, float* dbeta, float* colsum,
                         int T, int d, void* stream);

/* SPOS CNN kernels (spos.cu).  NHWC tensors [P = B*H*W rows][C]; forward tensors are
 * bf16x2 (hi plane followed by the lo plane; value = hi + lo), gradients plain bf16.
 * depthwise k x k, stride S, dilation dil (1 or 2), pad dil*(k/2), w fp32 [C][k][k]: z = dw(x) (x2 -> x2) if x && z;
 * dx = dw'(dz) (+ add) if dz && dx; dwsum[C*k*k] = sum(dz * x_hi) if dz && x && dwsum. */
int naspipe_debug_dw(const void* x, const float* w, void* z, const void* dz, const void* add, void* dx,
                     float* dwsum, int B, int H, int C, int k, int S, int dil, void* stream);
/* BatchNorm forward: mean/rstd of z (x2) over P rows (biased variance, eps 1e-5), then
 * y[p*ldy + c] = relu?(g (z - mean) rstd + b) (x2, lo plane yplane elements after hi). */
int naspipe_debug_bn_fwd(const void* z, int P, int C, const float* g, const float* b, int relu, void* y, int ldy,
                         size_t yplane, float* mean, float* rstd, void* stream);
/* BatchNorm backward: sums[2][C] = (sum dy', sum dy' xh), old[2][C] = (g, b) before the
 * SGD step g -= lr*sums[1], b -= lr*sums[0] (if update), dz = rstd g (dy' - s1/P - xh s2/P). */
int naspipe_debug_bn_bwd(const void* dy, int lddy, const void* z, int P, int C, const float* mean,
                         const float* rstd, float* g, float* b, int relu, void* dz, float* sums, float* old, float lr,
                         int update, void* stream);
/* stride-1 channel split (x2) / merge (bf16) and the frozen stem conv (x fp32 [B,H,H,3] ->
 * z x2); 3-pass bf16x2 GEMM out = A B^T (K-major hi/lo planes) -> x2 planes [M][N]. */
int naspipe_debug_chan_split(const void* x, int P, int Ch, void* out, int ldo, size_t oplane, void* xm,
                             void* stream);
int naspipe_debug_gemm_x2(int M, int N, int K, const void* A_hi, const void* A_lo, int lda, const void* B_hi,
                          const void* B_lo, int ldb, void* out_hi, void* out_lo, void* stream);
int naspipe_debug_chan_merge(const void* dproj, int ldp, const void* dm, int P, int Ch, void* dx, void* stream);
int naspipe_debug_stem(const float* x, const float* w, void* z, int B, int H, int C0, void* stream);
/* Input gradient with the fused BatchNorm-backward reduction (bn_bwd_reduce fused into its
 * producer): kind 0 / 2 = stride-1 / stride-2 depthwise dx = dw'(dz) (w fp32 [C][k][k], dx
 * [B,H,H,C], dz [B,Ho,Ho,C]),
 * kind 1 = 1x1-conv dx = dz W on the tcgen05 GEMM (EPI_BNBWD; dz bf16 [P][Cout], w16 bf16
 * [Cout][C], P = B*H*H).  dx is the output gradient of the unit z (x2 [P][C]) -> BN(mean,
 * rstd, g, b) [-> ReLU]: sums[2][C] = (sum dy', sum dy' xh) over the stored dx. */
/* bn_apply folded into the depthwise consumer (BnApplyIn): the unit zin (x2 [B,H,H,C]) ->
 * BN(g, b) [-> ReLU] -> depthwise k x k stride S dilation dil (w fp32 [C][k][k]).  Stored path:
 * bn_stats, bn_apply -> y, dw_fwd(y) -> out_ref (x2 [B,Ho,Ho,C]) and the weight gradient
 * dwsum_ref[C*k*k] = sum dz * y_hi; folded path: bn_stats, dw_fwd_bn -> out (and the published
 * meta[4][C] = mean, rstd, g, b), dw_wgrad with BN on load -> dwsum.  mean_ref / rstd_ref [C]
 * are bn_apply's. */
int naspipe_debug_dw_bn_fold(const void* zin, int B, int H, int C, const float* g, const float* b, int relu,
                             const float* w, int k, int S, int dil, const void* dz, void* out_ref, void* out,
                             float* dwsum_ref, float* dwsum, float* meta, float* mean_ref, float* rstd_ref,
                             void* stream);
/* Dense k x k conv columns (A40): cols x2 [B*Ho*Ho][k*k*C] (hi plane then lo plane) of x x2
 * [B,H,H,C] (if x && cols); dx bf16 [B,H,H,C] = col2im(dcols fp32 [B*Ho*Ho][k*k*C]) (+ add)
 * (if dcols && dx). */
int naspipe_debug_dense_cols(const void* x, void* cols, const float* dcols, const void* add, void* dx, int B, int H,
                             int C, int k, int S, void* stream);
int naspipe_debug_bnb_fused(int kind, const void* dz, const float* w, const void* w16, void* dx, int B, int H, int C,
                            int Cout, int k, int dil, const void* z, const float* mean, const float* rstd,
                            const float* g, const float* b, int relu, float* sums, void* stream);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif
