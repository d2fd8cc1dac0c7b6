// Host-side launchers of the sm_100a kernels (implemented in *.cu).  All launchers are
// asynchronous on the given stream, deterministic (fixed tiling and reduction order, no
// floating-point atomics) and throw naspipe::Error(NASPIPE_ECUDA) on launch failure.
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

namespace naspipe {

using bf16 = __nv_bfloat16;

// ------------------------------------------------------------------ tcgen05 GEMM
// C[M,N] = sum_k A[m,k] * B[n,k], bf16 operands, fp32 accumulation in TMEM.
//   A K-major: A stored [M][lda] (k contiguous);  A MN-major: stored [K][lda] (m contiguous)
//   B K-major: B stored [N][ldb];                 B MN-major: stored [K][ldb] (n contiguous)
// Epilogues (row m, column n, acc = C[m,n]):
enum GemmEpi {
  EPI_BF16 = 0,           // out16 = bf16(acc)
  EPI_F32 = 1,            // out32 = acc
  EPI_BIAS_BF16 = 2,      // out16 = bf16(acc + bias[n])
  EPI_BIAS_RESID_F32 = 3, // out32 = acc + bias[n] + resid[m,n]
  EPI_BIAS_GELU = 4,      // z = acc + bias[n]; out16 = bf16(z); out2 = bf16(gelu_tanh(z))
  EPI_DGELU = 5,          // out16 = bf16(acc * gelu_tanh'(aux16[m,n]))
  EPI_SGD = 6,            // w32[m,n] -= lr * acc; w16[m,n] = bf16(w32[m,n])   (the WRITE)
                          //   (+ w16lo[m,n] = bf16(w32 - w16) when w16lo != nullptr)
  EPI_X2 = 7,             // out16 = hi = bf16(acc), out2 = lo = bf16(acc - hi)  (bf16x2 planes)
  EPI_BNBWD = 8,          // out16 = dy = bf16(acc), plus the BatchNorm-backward sums of the unit
                          //   whose output gradient dy is (bn_bwd_reduce fused, see `bnb`)
};
// A depthwise conv whose input is the output of a conv -> BN [-> ReLU] unit that was never
// materialised (bn_apply folded into its consumer): the consumer reads the unit's z and
// applies y = relu?(g (z - mean) rstd + b) on load, rounding y to bf16x2 exactly as bn_apply
// stores it (so the numerics are those of the stored path).  Forward: mean/rstd come from
// the fixed-point sums acc of z; the consumer's last CTA (ticket) publishes mean, rstd and
// the g, b it used (gsnap, bsnap: the backward recomputes y with them even if g, b have been
// written since) and zeroes acc and the ticket.  Backward (depthwise weight gradient): mean,
// rstd, gsnap, bsnap as published.
struct BnApplyIn {
  const bf16* z = nullptr;  // x2 [P, C], lo plane zplane elements after hi
  size_t zplane = 0;
  int P = 0;
  unsigned long long* acc = nullptr;  // forward: the sums of z (zero after the consumer)
  int* ticket = nullptr;
  float *mean = nullptr, *rstd = nullptr;  // [C], published by the forward consumer
  const float *g = nullptr, *b = nullptr;  // the unit's g, b (forward)
  float *gsnap = nullptr, *bsnap = nullptr;  // [C], the g, b the forward applied
  int relu = 0;
};

// EPI_BNBWD / the depthwise input gradient with fused BatchNorm-backward sums: the unit
// z -> BN(mean, rstd, g, b) [-> ReLU] whose output gradient the kernel produces; per output
// element dy (as stored, bf16) it adds dy' = dy masked by the ReLU and dy' * xh, xh = (z -
// mean) rstd, to acc[0..C) / acc[C..2C) in fixed point (FIX_B; acc[2C] = overflow flag):
// exactly what bn_bwd_reduce would add, so bn_bwd_apply follows without a reduce launch.
struct BnBwdFuse {
  const bf16* z = nullptr;  // x2 [P, C], lo plane zplane elements after hi
  size_t zplane = 0;
  const float *mean = nullptr, *rstd = nullptr, *g = nullptr, *b = nullptr;
  int relu = 0;
  unsigned long long* acc = nullptr;  // nullptr: no fused sums
};
struct GemmEpiParams {
  const float* bias = nullptr;
  const float* resid = nullptr;
  const bf16* aux16 = nullptr;
  void* out = nullptr;
  bf16* out2 = nullptr;
  float* w32 = nullptr;
  bf16* w16 = nullptr;
  bf16* w16lo = nullptr;
  float lr = 0.f;
  // optional fp32 workspace enabling deterministic split-K for EPI_F32 / EPI_SGD
  float* ws = nullptr;
  size_t ws_elems = 0;
  size_t ws_stride = 0;  // set by the launcher
  // EPI_X2 only: add the per-column BatchNorm sums (sum, sum of squares of the STORED hi+lo
  // values) of the output to stats[0..2N) in fixed point (fixpoint.cuh; stats[2N] = the
  // overflow flag): the SPOS forward 1x1 conv with bn_stats fused
  unsigned long long* stats = nullptr;
  BnBwdFuse bnb;  // EPI_BNBWD only (stats of the fused BatchNorm backward; 1-CTA kernel)
};
// Cap on the CTAs (CTA pairs: 2 per pair) of every GEMM launched on stream s (0 = all SMs).
// The families cap their weight-gradient side streams (NASPIPE_SIDE_SMS), so the persistent
// wgrad GEMMs leave SMs to the stage stream's critical chain; results are unchanged (tiles
// are assigned statically and computed independently of the grid).
void gemm_set_stream_cap(cudaStream_t s, int max_ctas);
int side_stream_sms();  // NASPIPE_SIDE_SMS (0 = no cap)
// split-K factor the launcher uses for an (M, N, K) GEMM given a large enough workspace
int gemm_splitk_factor(int M, int N, int K);
void gemm_bf16_tc(cudaStream_t s, int M, int N, int K, const bf16* A, bool a_mn, int lda, const bf16* B,
                  bool b_mn, int ldb, int epi, const GemmEpiParams& ep);
// 3-pass bf16x2 GEMM (K-major A and B given as hi/lo planes): C = A_hi B_hi + A_hi B_lo +
// A_lo B_hi (the A_lo B_lo term, < 2^-16 relative, is dropped); epilogues EPI_X2 / EPI_BF16 /
// EPI_F32.  Tile N adapts to N (64 / 128 / 256).
void gemm_bf16x2_tc(cudaStream_t s, int M, int N, int K, const bf16* A_hi, const bf16* A_lo, int lda,
                    const bf16* B_hi, const bf16* B_lo, int ldb, int epi, const GemmEpiParams& ep);
// number of tcgen05 GEMM launches so far in this process (stats)
uint64_t gemm_launch_count();
int num_sms();  // SMs of the current device (cached)
uint64_t gemm_flop_count();  // algorithmic flops of every GEMM call of this process

// ------------------------------------------------------------------ attention (S <= 128)
// qkv [B*S, 3d] bf16 (q | k | v thirds, head j = columns [j*hd, (j+1)*hd) of each third);
// o [B*S, d] bf16; lse [B*h*S] f32 (natural log of the softmax denominator incl. scale).
// tcgen05 attention (attention_tc.cu) for S = 128 and head dim 64 / 128; attn_fwd / attn_bwd
// dispatch to it when attn_tc_supported
bool attn_tc_supported(int S, int d, int h);
void attn_fwd_tc(cudaStream_t s, const bf16* qkv, bf16* o, float* lse, int B, int S, int d, int h);
void attn_bwd_tc(cudaStream_t s, const bf16* qkv, const bf16* o, const float* lse, const bf16* dout, bf16* dqkv,
                 int B, int S, int d, int h);
void attn_fwd(cudaStream_t s, const bf16* qkv, bf16* o, float* lse, int B, int S, int d, int h);
// do_ [B*S, d] bf16 -> dqkv [B*S, 3d] bf16
void attn_bwd(cudaStream_t s, const bf16* qkv, const bf16* o, const float* lse, const bf16* do_,
              bf16* dqkv, int B, int S, int d, int h);

// ------------------------------------------------------------------ LayerNorm (eps 1e-5)
// y16 = bf16(g * (x - mu) * rstd + b); saves mean, rstd [T]
void ln_fwd(cudaStream_t s, const float* x, const float* g, const float* b, bf16* y16, float* mean,
            float* rstd, int T, int d);
// dx = resid + LN'(dy); dx16 = bf16(dx) (optional); per-row-block partials of
// dgamma, dbeta [nblk, d] and of colsum(dx) [nblk, d] (optional).
int ln_bwd_blocks(int T);
void ln_bwd(cudaStream_t s, const float* dy, const float* x, const float* mean, const float* rstd,
            const float* g, const float* resid, float* dx, bf16* dx16, float* part_dg, float* part_db,
            float* part_colsum, int T, int d);

// ------------------------------------------------------------------ reductions / elementwise
int colsum_blocks(int T);
// per-row-block column partial sums of X [T, N] (bf16 or f32) -> part [nblk, N]
void colsum_bf16(cudaStream_t s, const bf16* X, float* part, int T, int N);
// f32 -> bf16 copy plus column partial sums [ln_bwd_blocks(T), N] (ln_bwd's grouping)
void cast_colsum(cudaStream_t s, const float* X, bf16* X16, float* part, int T, int N);
// p[i] -= lr * sum_{j < nblk} part[j * n + i]   (fixed order)
void sgd_from_partials(cudaStream_t s, float* p, const float* part, int nblk, int n, float lr);
// Several of the above in one launch.  The sum is split into 8 fixed row groups of
// ceil(nblk/8) partials each, combined in group order — fixed for a given (nblk, n), so a
// parameter's update is bitwise independent of which stage or launch computes it.
struct SgdJob {
  float* p;
  const float* part;
  int nblk, n;
};
constexpr int kMaxSgdJobs = 8;
struct SgdJobs {
  SgdJob job[kMaxSgdJobs];
  int count;
  float lr;
};
void sgd_multi(cudaStream_t s, const SgdJobs& jobs);
// w16 = bf16(w32), n elements
void f32_to_bf16(cudaStream_t s, const float* w32, bf16* w16, size_t n);
// loss[0] = mean((y - t)^2); dy = 2 (y - t) / n.  part: workspace of mse_blocks(n) floats
int mse_blocks(size_t n);
void mse_loss(cudaStream_t s, const float* y, const float* t, float* dy, float* part, float* loss,
              size_t n);
// synthetic N(0,1)-like data from a counter hash (perf runs only)
void synth_fill(cudaStream_t s, float* x, size_t n, uint64_t seed);

// ------------------------------------------------------------------ MLP family (fp32)
// y = x + tanh(x W^T + b), x [B, d]; saves h = tanh(.) for backward
void mlp_fwd(cudaStream_t s, const float* x, const float* W, const float* b, float* y, float* h, int B, int d);
// dz = dy (1 - h^2); dx = dy + dz W (the W this subnet read); then the WRITE
// Wu -= lr dz^T x, bu -= lr sum dz (Wu, bu = W, b in place; the BSP accumulator, reading A30)
void mlp_bwd_sgd(cudaStream_t s, const float* x, const float* h, const float* dy, float* dx, const float* W, float* Wu,
                 float* bu, float lr, int B, int d);

// ------------------------------------------------------------------ SPOS CNN (spos.cu)
// NHWC activations [P = B*H*W rows, C channels]; C % 8 == 0 everywhere.  Forward tensors
// are bf16x2 (hi plane, lo plane `plane` elements later; contiguous tensors: plane = P*C),
// backward tensors plain bf16 (A28).
// w16 hi/lo planes of an fp32 vector
void f32_to_bf16x2(cudaStream_t s, const float* w32, bf16* hi, bf16* lo, size_t n);
// frozen stem: x fp32 [B,H,H,3], w fp32 [C0][3][3][3], stride 2, pad 1 -> z x2 [B,H/2,H/2,C0]
void spos_stem_conv(cudaStream_t s, const float* x, const float* w, bf16* z, int B, int H, int C0);
// BatchNorm (training mode, biased variance, eps 1e-5).  Reductions over the P rows are
// fixed-order fp32 row-block partials accumulated in 64-bit fixed point with integer atomics
// into acc [2][C] (+1: the overflow flag; unsigned long long, zero between uses): bitwise independent of the CTA
// order, no finalize launch.  The consumer kernel (bn_apply / bn_bwd_apply) derives the
// per-channel results from acc in every CTA; its last CTA (ticket: an int, 0 between uses)
// publishes them and zeroes acc and the ticket.
// Ticket-free ("ring") mode of the apply kernels (ticket == nullptr): the producers of
// consecutive BatchNorm uses add into a ring of 3 accumulators, so the apply kernel of use u
// needs no arrival ticket (round 2: the last-CTA ticket, its fences and the serial tail cost
// ~2 us per launch): CTA 0 publishes mean / rstd itself and zeroes `clear` [0, clear_n) -- the
// ring slot of use u-1, whose reader has finished and whose next producer (use u+2) runs
// after this kernel.  The backward's gamma / beta WRITE of use u cannot be done inside its own
// apply (other CTAs still read the pre-update values), so it is deferred: CTA 0 of the NEXT
// backward apply performs use u-1's WRITE (`prev`) and zeroes its slot, and bn_write_flush
// performs the task's last one.
struct BnWrite {
  float *gu = nullptr, *bu = nullptr;        // the WRITE targets (g, b in place; the BSP accumulator)
  const float *g = nullptr, *b = nullptr;    // the values the update starts from when gu == g / bu == b
  unsigned long long* acc = nullptr;         // the use's sums (nullptr: nothing pending); zeroed after
  int C = 0, update = 0;
  float lr = 0.f;
};
void bn_write_flush(cudaStream_t s, const BnWrite& w);
// acc <- (sum z, sum z^2) of z (x2) over its P rows
void bn_stats(cudaStream_t s, const bf16* z, int P, int C, unsigned long long* acc);
// y[p*ldy + c] = relu?(g (z - mean) rstd + b) with mean, rstd from acc; z x2 (plane P*C), y
// x2 (planes yplane apart); writes mean, rstd [C] (for the backward), clears acc
void bn_apply(cudaStream_t s, const bf16* z, int P, int C, unsigned long long* acc, int* ticket, float* mean,
              float* rstd, const float* g, const float* b, int relu, bf16* y, int ldy, size_t yplane,
              unsigned long long* clear = nullptr, int clear_n = 0);
// acc <- (s1 = sum dy', s2 = sum dy' xh) (dy' = dy masked by the ReLU of the forward)
void bn_bwd_reduce(cudaStream_t s, const bf16* dy, int lddy, const bf16* z, int P, int C, const float* mean,
                   const float* rstd, const float* g, const float* b, int relu, unsigned long long* acc);
// dz = rstd g (dy' - s1/P - xh s2/P) with the pre-update g, b; then (update) the SGD WRITE
// gu -= lr s2, bu -= lr s1 (gu, bu = g, b in place; the bulk accumulator under BSP, reading
// A30); clears acc
void bn_bwd_apply(cudaStream_t s, const bf16* dy, int lddy, const bf16* z, int P, int C, const float* mean,
                  const float* rstd, const float* g, const float* b, float* gu, float* bu, float lr, int update,
                  unsigned long long* acc, int* ticket, int relu, bf16* dz, const BnWrite& prev = BnWrite());
// acc holds 2C sums + the sticky overflow flag acc[2C] (fixpoint.cuh; checked at drain)
bool bn_fix_overflow(const unsigned long long* acc, int C);
// depthwise k x k (k in {3,5,7}), stride S, dilation dil (1 or 2), pad dil*(k/2); w fp32 [C][k][k];
// H = input height = width.
// dw_fwd: x2 -> x2; dw_dgrad: bf16 (+ bf16 add); dw_wgrad reads the hi plane of x.
// stats != nullptr: also add the BatchNorm sums of the stored z to it (bn_stats fused)
void dw_fwd(cudaStream_t s, const bf16* x, const float* w, bf16* z, int B, int H, int C, int k, int S, int dil,
            unsigned long long* stats = nullptr);
// dw_fwd of y = BN(z) [+ ReLU] applied on load (BnApplyIn; x is not read)
void dw_fwd_bn(cudaStream_t s, const BnApplyIn& xin, const float* w, bf16* z, int B, int H, int C, int k, int S,
               int dil, unsigned long long* stats);
// bnb.acc != nullptr (stride 1 only): also add the BatchNorm-backward sums of the unit whose
// output gradient dx is (BnBwdFuse; bn_bwd_reduce fused)
void dw_dgrad(cudaStream_t s, const bf16* dz, const float* w, const bf16* add, bf16* dx, int B, int H, int C, int k,
              int S, int dil, const BnBwdFuse& bnb = BnBwdFuse());
int dw_wgrad_blocks(int B, int H, int C, int k, int S);
// Dense k x k conv (Table 5's Conv 3x3; reading A40) as GEMMs over explicit columns:
// cols [B*Ho*Ho][k*k*C] (column (u*k + v)*C + c = x[b, oh*S + u - k/2, ow*S + v - k/2, c],
// zero outside), x2 planes (hi plane, lo plane cplane elements later); and its adjoint
// dx[b, ih, iw, c] = sum over (u, v) in order of dcols (fp32) (+ add), rounded to bf16.
void im2col_x2(cudaStream_t s, const bf16* x, size_t xplane, int B, int H, int C, int k, int S, bf16* cols,
               size_t cplane);
void col2im(cudaStream_t s, const float* dcols, int B, int H, int C, int k, int S, const bf16* add, bf16* dx);
// weight gradient of a depthwise conv with the SGD WRITE fused: w -= lr * sum over the batch
// (acc [C*k*k + 1] and ticket zero between uses, fixpoint.cuh; w = master or BSP accumulator)
// xin != nullptr: x = the hi plane of BN(z) [+ ReLU] recomputed on load (BnApplyIn, the
// published mean/rstd and g/b snapshots); x is then not read
void dw_wgrad_sgd(cudaStream_t s, const bf16* dz, const bf16* x, unsigned long long* acc, int* ticket, float* w,
                  float lr, int B, int H, int C, int k, int S, int dil, const BnApplyIn* xin = nullptr);
// ---- NLP op families (seqconv.cu; Table 5, reading A38).  x, dy: bf16 [T = B*S, d].
// seqconv: depthwise conv along each sequence of S rows, taps w [d][k] (H == 0) or
// softmax(Wl[H][k]) shared by d/H channels (Light Conv); flip = the input gradient; out bf16 or f32.
void seqconv(cudaStream_t s, const bf16* x, const float* w, int H, int k, bool flip, bool out_f32, void* out, int T,
             int S, int d);
// weight gradient + SGD WRITE (wupd -= lr * g; Light Conv through the softmax Jacobian, wread =
// the weights the forward used); acc [d*k] fixed-point totals and ticket zero between uses,
// flag = sticky overflow flag (fixpoint.cuh)
void seqconv_wgrad_sgd(cudaStream_t s, const bf16* dy, const bf16* x, unsigned long long* acc,
                       unsigned long long* flag, int* ticket, const float* wread, float* wupd, int H, int k, float lr,
                       int T, int S, int d);
// Conv 3x1 im2col: cols [T][3d], cols[t][u*d+i] = x[t+u-1][i] inside the sequence; and its adjoint (f32)
void conv3_cols(cudaStream_t s, const bf16* x, bf16* cols, int T, int S, int d);
void conv3_cols_bwd(cudaStream_t s, const float* dcols, float* dx, int T, int S, int d);
// channel split of a stride-1 block input [P, 2Ch] (x2): out[:, i] = x[:, 2i] (ld ldo, planes
// oplane apart), xm[:, i] = x[:, 2i+1]; merge is its (plain bf16) backward
void chan_split(cudaStream_t s, const bf16* x, int P, int Ch, bf16* out, int ldo, size_t oplane, bf16* xm);
void chan_merge(cudaStream_t s, const bf16* dproj, int ldp, const bf16* dm, int P, int Ch, bf16* dx);
// frozen head pieces
void gap_pool(cudaStream_t s, const bf16* r, int B, int HW, int C, float* gap);
// logits = gap W_fc^T (fp32 tiles), then per-sample softmax CE: loss_per[b], dlogits = (p - onehot)/B
void fc_ce(cudaStream_t s, const float* gap, const float* wf, const int* labels, int B, int C, int ncls,
           float* logits, float* dlogits, float* loss_per);
void ce_mean(cudaStream_t s, const float* loss_per, int B, float* loss);
void fc_dgap(cudaStream_t s, const float* dlogits, const float* wf, int B, int C, int ncls, float* dgap);
void head_bcast(cudaStream_t s, const float* dgap, int B, int HW, int C, bf16* dr);
void synth_labels(cudaStream_t s, int* labels, int B, int ncls, uint64_t seed);

}  // namespace naspipe
