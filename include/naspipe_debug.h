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

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif
