// Block families on one stage.
//   MLP (configs[0]):          y = x + tanh(x W^T + b), fp32 CUDA-core kernels (K1/K2).
//   TRANSFORMER (configs[2,3]): pre-LN MHA + GELU FFN (reading A17) on tcgen05 GEMMs with
//                              fused epilogues, mma.sync attention, CUDA-core LayerNorm.
// Backward of a stage = per block, in reverse: dgrad with the pre-update weights, then the
// wgrad GEMM whose epilogue applies SGD to the fp32 master and refreshes the bf16 shadow
// (the WRITE of Def.2 / Alg.1 line 9 "flush", reading A4); bias / LayerNorm parameters are
// updated from fixed-order partial sums.
#include <algorithm>
#include <cstring>

#include "family.h"
#include "launch.h"

namespace naspipe {

// ---------------------------------------------------------------- arena / timer
void* DevArena::raw(size_t bytes) {
  if (bytes == 0) bytes = 256;
  void* p = nullptr;
  cudaSetDevice(dev_);
  cudaError_t e = cudaMalloc(&p, bytes);
  NP_REQUIRE(e == cudaSuccess, e == cudaErrorMemoryAllocation ? NASPIPE_ENOMEM : NASPIPE_ECUDA,
             "cudaMalloc(%zu) on device %d: %s", bytes, dev_, cudaGetErrorString(e));
  ptrs_.push_back(p);
  bytes_ += bytes;
  return p;
}
DevArena::~DevArena() {
  cudaSetDevice(dev_);
  for (void* p : ptrs_) cudaFree(p);
}

void KernelTimer::begin(cudaStream_t s) {
  if (!on) return;
  if (used == pairs.size()) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    pairs.push_back({a, b});
  }
  cudaEventRecord(pairs[used].first, s);
}
void KernelTimer::end(cudaStream_t s, double f) {
  flops += f;  // algorithmic work and launches are counted with or without the events
  launches += 1;
  if (!on) return;
  cudaEventRecord(pairs[used].second, s);
  ++used;
}
void KernelTimer::collect() {
  for (size_t i = 0; i < used; ++i) {
    cudaEventSynchronize(pairs[i].second);
    float t = 0;
    cudaEventElapsedTime(&t, pairs[i].first, pairs[i].second);
    ms += t;
  }
  used = 0;
}
void Family::loss(int, const void* out, const void* target, void* dy, float* loss_dst, cudaStream_t s) {
  const size_t n = spec_base_->batch_elems();
  mse_loss(s, static_cast<const float*>(out), static_cast<const float*>(target), static_cast<float*>(dy), mse_part_,
           loss_dst, n);
  counters.launches += 2;
}

void Family::synth_target(void* dst, uint64_t seed, cudaStream_t s) {
  synth_fill(s, static_cast<float*>(dst), spec_base_->batch_elems(), seed);
}

KernelTimer::~KernelTimer() {
  for (auto& p : pairs) {
    cudaEventDestroy(p.first);
    cudaEventDestroy(p.second);
  }
}

namespace {

// ======================================================================= MLP
class MlpFamily : public Family {
 public:
  MlpFamily(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& A, cudaStream_t s)
      : spec_(spec), blocks_(blocks), W_(W), B_(spec.B()), d_(spec.raw.width), lr_(spec.raw.lr) {
    const int nb = (int)blocks.size(), n = spec.n();
    (void)s;
    const size_t act = (size_t)B_ * d_;
    params_.assign((size_t)nb * n, nullptr);
    h_.resize((size_t)W * nb);
    act_.resize((size_t)W * nb);
    xin_.assign((size_t)W * nb, nullptr);
    for (auto& p : h_) p = A.alloc<float>(act);
    for (auto& p : act_) p = A.alloc<float>(act);
    g_[0] = A.alloc<float>(act);
    g_[1] = A.alloc<float>(act);
    spec_base_ = &spec;
    n_choices_ = spec.n();
    mse_part_ = A.alloc<float>(mse_blocks(spec.batch_elems()));
  }
  void bind(int j, int c, float* w32, bf16*) override { params_[(size_t)j * spec_.n() + c] = w32; }
  size_t shadow_elems(int, int) const override { return 0; }
  float* master(int j, int c) override { return params_[(size_t)j * spec_.n() + c]; }
  void refresh_shadow(int, int, cudaStream_t) override {}

  void forward(int slot, const int32_t* ch, const void* x_in, void* x_out, cudaStream_t s) override {
    const int nb = (int)blocks_.size(), lo = rlo(), hi = rhi(nb);
    const float* x = static_cast<const float*>(x_in);
    for (int j = lo; j < hi; ++j) {
      float* P = master(j, ch[blocks_[j]]);
      float* y = (j == hi - 1) ? static_cast<float*>(x_out) : act_[(size_t)slot * nb + j + 1];
      xin_[(size_t)slot * nb + j] = x;
      mlp_fwd(s, x, P, P + (size_t)d_ * d_, y, h_[(size_t)slot * nb + j], B_, d_);
      counters.launches++;
      x = y;
    }
  }
  void backward(int slot, const int32_t* ch, const void* dy, void* dx, cudaStream_t s) override {
    const int nb = (int)blocks_.size(), lo = rlo(), hi = rhi(nb);
    const float* g = static_cast<const float*>(dy);
    for (int j = hi - 1; j >= lo; --j) {
      float* P = master(j, ch[blocks_[j]]);
      float* U = upd(j, ch[blocks_[j]]);  // SGD WRITE target (P in place; the BSP accumulator)
      float* out = (j == lo) ? static_cast<float*>(dx) : g_[j & 1];
      mlp_bwd_sgd(s, xin_[(size_t)slot * nb + j], h_[(size_t)slot * nb + j], g, out, P, U, U + (size_t)d_ * d_, lr_,
                  B_, d_);
      counters.launches++;
      g = out;
    }
  }

 private:
  const Spec& spec_;
  std::vector<int> blocks_;
  int W_, B_, d_;
  float lr_;
  std::vector<float*> params_, h_, act_;
  std::vector<const float*> xin_;
  float* g_[2];
};

// ======================================================================= Transformer
struct TfSlot {  // stash of one (slot, local block)
  const float* xin = nullptr;
  float* act = nullptr;  // block input storage when the input is produced on this stage
  bf16 *a, *qkv, *o, *a2, *z, *g;
  float *mean1, *rstd1, *lse, *x1, *mean2, *rstd2;
};

class TfFamily : public Family {
 public:
  TfFamily(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& A, cudaStream_t s)
      : spec_(spec), blocks_(blocks), W_(W), d_(spec.raw.d_model), S_(spec.raw.seq_len), B_(spec.B()),
        T_(spec.rows()), lr_(spec.raw.lr) {
    const int nb = (int)blocks.size(), n = spec.n();
    fmax_ = *std::max_element(spec.ffn.begin(), spec.ffn.end());
    hmax_ = *std::max_element(spec.heads.begin(), spec.heads.end());
    (void)s;
    w32_.assign((size_t)nb * n, nullptr);
    w16_.assign((size_t)nb * n, nullptr);
    const size_t Td = (size_t)T_ * d_;
    recompute_ = (spec.raw.flags & NASPIPE_FLAG_RECOMPUTE) != 0;
    auto alloc_acts = [&](TfSlot& t) {
      t.a = A.alloc<bf16>(Td);
      t.qkv = A.alloc<bf16>(3 * Td);
      t.o = A.alloc<bf16>(Td);
      t.a2 = A.alloc<bf16>(Td);
      t.z = A.alloc<bf16>((size_t)T_ * fmax_);
      t.g = A.alloc<bf16>((size_t)T_ * fmax_);
      t.mean1 = A.alloc<float>(T_);
      t.rstd1 = A.alloc<float>(T_);
      t.mean2 = A.alloc<float>(T_);
      t.rstd2 = A.alloc<float>(T_);
      t.lse = A.alloc<float>((size_t)B_ * hmax_ * S_);
      t.x1 = A.alloc<float>(Td);
    };
    // activation stash per (slot, block); with recomputation (reading A13) only the
    // block inputs are kept and two scratch sets (by block parity) hold a block's activations
    // while it is recomputed and back-propagated
    slots_.resize((size_t)W * nb);
    for (int sl = 0; sl < W; ++sl)
      for (int j = 0; j < nb; ++j) {
        TfSlot& t = slots_[(size_t)sl * nb + j];
        t.act = (j > 0) ? A.alloc<float>(Td) : nullptr;
        if (!recompute_) alloc_acts(t);
      }
    if (recompute_) {
      for (auto& t : rs_) alloc_acts(t);
      ry_ = A.alloc<float>(Td);
    }
    // backward workspace (tasks on a stage are serialised on its stream).  Buffers the side
    // stream reads are double buffered by block parity (see backward()).
    for (int p = 0; p < 2; ++p) {
      dy16_[p] = A.alloc<bf16>(Td);
      dz_[p] = A.alloc<bf16>((size_t)T_ * fmax_);
      dx1_16_[p] = A.alloc<bf16>(Td);
      dqkv_[p] = A.alloc<bf16>(3 * Td);
    }
    da_ = A.alloc<float>(Td);
    dx1_ = A.alloc<float>(Td);
    do16_ = A.alloc<bf16>(Td);
    gb_[0] = A.alloc<float>(Td);
    gb_[1] = A.alloc<float>(Td);
    // split-K workspace (side stream only): the largest splits * M * N of the wgrad GEMMs
    ws_elems_ = 0;
    bool any_conv3 = false, any_taps = false;
    for (int c = 0; c < n; ++c) {
      const int f = spec.ffn[c], T = T_, d = d_;
      const int shp[5][3] = {{d, f, T}, {f, d, T}, {d, d, T}, {3 * d, d, T}, {d, 3 * d, T}};
      for (auto& q : shp)
        ws_elems_ = std::max(ws_elems_, (size_t)gemm_splitk_factor(q[0], q[1], q[2]) * q[0] * q[1]);
      any_conv3 |= spec.op[c] == TF_CONV3;
      any_taps |= spec.op[c] == TF_SEPCONV7 || spec.op[c] == TF_LIGHTCONV5;
    }
    ws_ = A.alloc<float>(ws_elems_);
    // NLP op families (reading A38): Conv 3x1's column gradient, the sequence-conv weight
    // gradient partials (side stream only) and its arrival ticket
    if (any_conv3) dcols_ = A.alloc<float>(3 * Td);
    if (any_taps) {  // fixed-point totals [d * 7] + the overflow flag (reading A33)
      sc_acc_ = A.alloc<unsigned long long>((size_t)d_ * 7 + 1);
      cudaMemset(sc_acc_, 0, ((size_t)d_ * 7 + 1) * 8);
      sc_tick_ = A.alloc<int>(1);
      cudaMemset(sc_tick_, 0, sizeof(int));
    }
    csb_ = colsum_blocks(T_);
    lnb_ = ln_bwd_blocks(T_);
    for (int p = 0; p < 2; ++p) {
      p_db2_[p] = A.alloc<float>((size_t)lnb_ * d_);
      p_db1_[p] = A.alloc<float>((size_t)csb_ * fmax_);
      p_dbo_[p] = A.alloc<float>((size_t)lnb_ * d_);
      p_dbqkv_[p] = A.alloc<float>((size_t)csb_ * 3 * d_);
      p_g2_[p] = A.alloc<float>((size_t)lnb_ * d_);
      p_b2_[p] = A.alloc<float>((size_t)lnb_ * d_);
    }
    p_g1_ = A.alloc<float>((size_t)lnb_ * d_);
    p_b1_ = A.alloc<float>((size_t)lnb_ * d_);
    spec_base_ = &spec;
    n_choices_ = spec.n();
    mse_part_ = A.alloc<float>(mse_blocks(spec.batch_elems()));
    create_stream(&side_, false);
    if (side_stream_sms() > 0) gemm_set_stream_cap(side_, side_stream_sms());
    for (auto* e : {&ev_dz_, &ev_da2_, &ev_do_, &ev_da_, &ev_done_[0], &ev_done_[1], &ev_join_})
      cudaEventCreateWithFlags(e, cudaEventDisableTiming);
  }

  ~TfFamily() override {
    cudaStreamSynchronize(side_);
    for (auto e : {ev_dz_, ev_da2_, ev_do_, ev_da_, ev_done_[0], ev_done_[1], ev_join_}) cudaEventDestroy(e);
    cudaStreamDestroy(side_);
  }

  void check_after_drain() override {
    if (!sc_acc_) return;
    unsigned long long flag = 0;
    cudaMemcpy(&flag, sc_acc_ + (size_t)d_ * 7, 8, cudaMemcpyDeviceToHost);
    NP_REQUIRE(flag == 0, NASPIPE_EINTERNAL,
               "sequence-conv weight-gradient fixed-point overflow (a partial outside the 64-bit range, seqconv.cu)");
  }

  void bind(int j, int c, float* w32, bf16* w16) override {
    w32_[(size_t)j * spec_.n() + c] = w32;
    w16_[(size_t)j * spec_.n() + c] = w16;
  }
  size_t shadow_elems(int, int c) const override { return spec_.tf_offsets(c).sh_total; }
  float* master(int j, int c) override { return w32_[(size_t)j * spec_.n() + c]; }

  void refresh_shadow(int j, int c, cudaStream_t s) override {
    const TfOffsets o = spec_.tf_offsets(c);
    const size_t d = d_, f = spec_.ffn[c];
    float* p = master(j, c);
    bf16* w = w16_[(size_t)j * spec_.n() + c];
    if (o.n_Win) f32_to_bf16(s, p + o.Win, w + o.sh_Win, o.n_Win);
    f32_to_bf16(s, p + o.Wo, w + o.sh_Wo, o.n_Wo);
    f32_to_bf16(s, p + o.W1, w + o.sh_W1, f * d);
    f32_to_bf16(s, p + o.W2, w + o.sh_W2, d * f);
  }

  void forward(int slot, const int32_t* ch, const void* x_in, void* x_out, cudaStream_t s) override {
    const int nb = (int)blocks_.size(), lo = rlo(), hi = rhi(nb);
    const float* x = static_cast<const float*>(x_in);
    for (int j = lo; j < hi; ++j) {
      const int c = ch[blocks_[j]];
      TfSlot& t = slots_[(size_t)slot * nb + j];
      t.xin = x;
      float* y = (j == hi - 1) ? static_cast<float*>(x_out) : slots_[(size_t)slot * nb + j + 1].act;
      if (recompute_) {  // activations into the scratch set; only the block input is kept
        TfSlot tt = rs_[j & 1];
        tt.xin = x;
        block_fwd(j, c, tt, y, s);
      } else {
        block_fwd(j, c, t, y, s);
      }
      x = y;
    }
  }

  // Backward of the stage.  The dgrad chain (dz -> da2 -> LN2' -> do -> attention' -> da ->
  // LN1') runs on the stage stream; each weight-gradient GEMM (with its fused SGD WRITE),
  // the bias column sums and the bias/LN2 updates run on a side stream as soon as the dgrad
  // that read the pre-update weight is done (reading A4), filling the SMs the dgrad chain
  // leaves idle.  Buffers the side stream reads are double-buffered by block parity; the
  // stage stream joins the side stream before the task ends.
  void backward(int slot, const int32_t* ch, const void* dy_v, void* dx_v, cudaStream_t s) override {
    const int nb = (int)blocks_.size(), lo = rlo(), hi = rhi(nb);
    const float* dy = static_cast<const float*>(dy_v);
    float* dx = static_cast<float*>(dx_v);
    const float* g = dy;
    int db2_nblk = 0;
    for (int j = hi - 1; j >= lo; --j) {
      const int c = ch[blocks_[j]];
      const int p = j & 1;
      TfSlot& t = slots_[(size_t)slot * nb + j];
      if (j == hi - 1) {  // grad entering the stage: bf16 copy + colsum for b2
        cast_colsum(s, g, dy16_[p], p_db2_[p], T_, d_);
        counters.launches++;
        db2_nblk = lnb_;
      }
      // stage 0 needs no input gradient, but LN1's backward still runs (dgamma/dbeta):
      // its dx goes to a scratch buffer (gb_[lo & 1] is free: block lo + 1 wrote the other)
      float* out = (j == lo) ? (dx ? dx : gb_[lo & 1]) : gb_[j & 1];
      if (recompute_) {
        // recompute block j's forward from its kept input into scratch set p (bitwise the
        // forward's activations: same kernels, same input, same weights — CSP/BSP do not
        // update a candidate between F(y) and B(y)); the side stream's last reads of set p
        // (block j+2's weight gradients) end with ev_done_[p]
        TfSlot tt = rs_[p];
        tt.xin = t.xin;
        cudaStreamWaitEvent(s, ev_done_[p], 0);
        block_fwd(j, c, tt, ry_, s);
        block_bwd(j, c, tt, g, out, /*want_next=*/j > lo, db2_nblk, p, s);
      } else {
        block_bwd(j, c, t, g, out, /*want_next=*/j > lo, db2_nblk, p, s);
      }
      db2_nblk = lnb_;
      g = out;
    }
    cudaEventRecord(ev_join_, side_);
    cudaStreamWaitEvent(s, ev_join_, 0);
  }

 private:
  void gemm(cudaStream_t s, int M, int N, int K, const bf16* A, bool amn, int lda, const bf16* B, bool bmn, int ldb,
            int epi, const GemmEpiParams& ep, bool split_ok = false) {
    if (timer) timer->begin(s);
    GemmEpiParams e = ep;
    if (split_ok) {  // only the side stream owns the split-K workspace
      e.ws = ws_;
      e.ws_elems = ws_elems_;
    }
    gemm_bf16_tc(s, M, N, K, A, amn, lda, B, bmn, ldb, epi, e);
    if (timer) timer->end(s, 2.0 * M * N * K);
    counters.launches++;
  }

  void block_fwd(int j, int c, TfSlot& t, float* y, cudaStream_t s) {
    const TfOffsets o = spec_.tf_offsets(c);
    const int d = d_, f = spec_.ffn[c], h = spec_.heads[c], T = T_;
    float* P = master(j, c);
    bf16* W = w16_[(size_t)j * spec_.n() + c];
    const bf16 *Win = W + o.sh_Win, *Wo = W + o.sh_Wo, *W1 = W + o.sh_W1, *W2 = W + o.sh_W2;
    ln_fwd(s, t.xin, P + o.ln1g, P + o.ln1b, t.a, t.mean1, t.rstd1, T, d);
    // token mixer (attention, or one of Table 5's NLP convolutions, reading A38); its output
    // projection adds the bias and the residual: x1 = x + M(a)
    const bf16* mo = t.o;  // input of the output projection
    int mo_k = d;
    if (o.op == TF_ATTN) {
      GemmEpiParams e1;
      e1.bias = P + o.bin;
      e1.out = t.qkv;
      gemm(s, T, 3 * d, d, t.a, false, d, Win, false, d, EPI_BIAS_BF16, e1);
      attn_fwd(s, t.qkv, t.o, t.lse, B_, S_, d, h);
    } else if (o.op == TF_CONV3) {
      conv3_cols(s, t.a, t.qkv, T, S_, d);  // [T, 3d] columns (t.qkv holds 3 T d)
      mo = t.qkv;
      mo_k = 3 * d;
    } else if (o.op == TF_SEPCONV7) {
      seqconv(s, t.a, P + o.taps, 0, 7, false, false, t.o, T, S_, d);
    } else {  // Light Conv 5x1: v = a Wi^T + bi (in t.qkv), l = LightConv(v)
      GemmEpiParams e1;
      e1.bias = P + o.bin;
      e1.out = t.qkv;
      gemm(s, T, d, d, t.a, false, d, Win, false, d, EPI_BIAS_BF16, e1);
      seqconv(s, t.qkv, P + o.taps, h, 5, false, false, t.o, T, S_, d);
    }
    GemmEpiParams e2;
    e2.bias = P + o.bo;
    e2.resid = t.xin;
    e2.out = t.x1;
    gemm(s, T, d, mo_k, mo, false, mo_k, Wo, false, mo_k, EPI_BIAS_RESID_F32, e2);
    ln_fwd(s, t.x1, P + o.ln2g, P + o.ln2b, t.a2, t.mean2, t.rstd2, T, d);
    GemmEpiParams e3;
    e3.bias = P + o.b1;
    e3.out = t.z;
    e3.out2 = t.g;
    gemm(s, T, f, d, t.a2, false, d, W1, false, d, EPI_BIAS_GELU, e3);
    GemmEpiParams e4;
    e4.bias = P + o.b2;
    e4.resid = t.x1;
    e4.out = y;
    gemm(s, T, d, f, t.g, false, f, W2, false, f, EPI_BIAS_RESID_F32, e4);
    counters.launches += 3;
  }

  // dy: f32 grad of the block output (its bf16 copy is in dy16_[p], its column partials in
  // p_db2_[p][0..db2_nblk)); writes dx (f32); if want_next also dy16_/p_db2_[p^1] for block j-1.
  void block_bwd(int j, int c, TfSlot& t, const float* dy, float* dx, bool want_next, int db2_nblk, int p,
                 cudaStream_t s) {
    const TfOffsets o = spec_.tf_offsets(c);
    const int d = d_, f = spec_.ffn[c], h = spec_.heads[c], T = T_;
    float* P = master(j, c);
    bf16* W = w16_[(size_t)j * spec_.n() + c];
    bf16 *Win = W + o.sh_Win, *Wo = W + o.sh_Wo, *W1 = W + o.sh_W1, *W2 = W + o.sh_W2;
    float* U = upd(j, c);  // SGD WRITE target (P in place; the BSP accumulator, no shadow refresh)
    const bool inplace = in_place(j, c);
    auto sgd_ep = [&](float* w32, bf16* w16) {
      GemmEpiParams e;
      e.w32 = w32;
      e.w16 = inplace ? w16 : nullptr;
      e.lr = lr_;
      return e;
    };
    // ---- FFN half
    GemmEpiParams e;
    e.aux16 = t.z;
    e.out = dz_[p];
    gemm(s, T, f, d, dy16_[p], false, d, W2, true, f, EPI_DGELU, e);        // dz = (dy W2) * gelu'(z)
    cudaEventRecord(ev_dz_, s);
    cudaStreamWaitEvent(side_, ev_dz_, 0);
    gemm(side_, d, f, T, dy16_[p], true, d, t.g, true, f, EPI_SGD, sgd_ep(U + o.W2, W2), true);  // W2 -= lr dy^T g
    colsum_bf16(side_, dz_[p], p_db1_[p], T, f);
    e = GemmEpiParams();
    e.out = da_;
    gemm(s, T, d, f, dz_[p], false, f, W1, true, d, EPI_F32, e);             // da2 = dz W1
    cudaEventRecord(ev_da2_, s);
    cudaStreamWaitEvent(side_, ev_da2_, 0);
    gemm(side_, f, d, T, dz_[p], true, f, t.a2, true, d, EPI_SGD, sgd_ep(U + o.W1, W1), true);  // W1 -= lr dz^T a2
    ln_bwd(s, da_, t.x1, t.mean2, t.rstd2, P + o.ln2g, dy, dx1_, dx1_16_[p], p_g2_[p], p_b2_[p], p_dbo_[p], T, d);
    // ---- mixer half (da = dM/da into da_; every weight gradient on the side stream after the
    // dgrad that read the pre-update weight, reading A4)
    int nl = 0;  // non-GEMM launches of the mixer half
    if (o.op == TF_ATTN) {
      e = GemmEpiParams();
      e.out = do16_;
      gemm(s, T, d, d, dx1_16_[p], false, d, Wo, true, d, EPI_BF16, e);        // do = dx1 Wo
      cudaEventRecord(ev_do_, s);
      cudaStreamWaitEvent(side_, ev_do_, 0);
      gemm(side_, d, d, T, dx1_16_[p], true, d, t.o, true, d, EPI_SGD, sgd_ep(U + o.Wo, Wo), true);  // Wo -= lr dx1^T o
      attn_bwd(s, t.qkv, t.o, t.lse, do16_, dqkv_[p], B_, S_, d, h);
      e = GemmEpiParams();
      e.out = da_;
      gemm(s, T, d, 3 * d, dqkv_[p], false, 3 * d, Win, true, d, EPI_F32, e);  // da = dqkv Wqkv
      cudaEventRecord(ev_da_, s);
      cudaStreamWaitEvent(side_, ev_da_, 0);
      colsum_bf16(side_, dqkv_[p], p_dbqkv_[p], T, 3 * d);
      gemm(side_, 3 * d, d, T, dqkv_[p], true, 3 * d, t.a, true, d, EPI_SGD, sgd_ep(U + o.Win, Win), true);
      nl = 2;
    } else if (o.op == TF_CONV3) {
      e = GemmEpiParams();
      e.out = dcols_;
      gemm(s, T, 3 * d, d, dx1_16_[p], false, d, Wo, true, 3 * d, EPI_F32, e);  // dcols = dx1 Wc
      cudaEventRecord(ev_do_, s);
      cudaStreamWaitEvent(side_, ev_do_, 0);
      gemm(side_, d, 3 * d, T, dx1_16_[p], true, d, t.qkv, true, 3 * d, EPI_SGD, sgd_ep(U + o.Wo, Wo), true);
      conv3_cols_bwd(s, dcols_, da_, T, S_, d);                                 // da = cols'(dcols)
      nl = 1;
    } else if (o.op == TF_SEPCONV7) {
      bf16* ds = dqkv_[p];  // parity buffer: the side stream reads it
      e = GemmEpiParams();
      e.out = ds;
      gemm(s, T, d, d, dx1_16_[p], false, d, Wo, true, d, EPI_BF16, e);        // ds = dx1 Wp
      cudaEventRecord(ev_do_, s);
      cudaStreamWaitEvent(side_, ev_do_, 0);
      gemm(side_, d, d, T, dx1_16_[p], true, d, t.o, true, d, EPI_SGD, sgd_ep(U + o.Wo, Wo), true);  // Wp -= lr dx1^T s
      seqconv(s, ds, P + o.taps, 0, 7, true, true, da_, T, S_, d);              // da = DW'(ds)
      cudaEventRecord(ev_da_, s);
      cudaStreamWaitEvent(side_, ev_da_, 0);
      seqconv_wgrad_sgd(side_, ds, t.a, sc_acc_, sc_acc_ + (size_t)d * 7, sc_tick_, P + o.taps, U + o.taps, 0, 7, lr_, T, S_, d);
      nl = 2;
    } else {  // Light Conv 5x1
      bf16 *dl = dqkv_[p], *dv = dqkv_[p] + (size_t)T * d;
      e = GemmEpiParams();
      e.out = dl;
      gemm(s, T, d, d, dx1_16_[p], false, d, Wo, true, d, EPI_BF16, e);        // dl = dx1 Wo
      cudaEventRecord(ev_do_, s);
      cudaStreamWaitEvent(side_, ev_do_, 0);
      gemm(side_, d, d, T, dx1_16_[p], true, d, t.o, true, d, EPI_SGD, sgd_ep(U + o.Wo, Wo), true);  // Wo -= lr dx1^T l
      seqconv(s, dl, P + o.taps, h, 5, true, false, dv, T, S_, d);              // dv = LightConv'(dl)
      e = GemmEpiParams();
      e.out = da_;
      gemm(s, T, d, d, dv, false, d, Win, true, d, EPI_F32, e);                 // da = dv Wi
      cudaEventRecord(ev_da_, s);
      cudaStreamWaitEvent(side_, ev_da_, 0);
      seqconv_wgrad_sgd(side_, dl, t.qkv, sc_acc_, sc_acc_ + (size_t)d * 7, sc_tick_, P + o.taps, U + o.taps, h, 5, lr_, T, S_, d);
      colsum_bf16(side_, dv, p_dbqkv_[p], T, d);
      gemm(side_, d, d, T, dv, true, d, t.a, true, d, EPI_SGD, sgd_ep(U + o.Win, Win), true);  // Wi -= lr dv^T a
      nl = 3;
    }
    // bias / LN2 updates (all their partials are complete)
    SgdJobs j1{};
    j1.lr = lr_;
    j1.job[0] = {U + o.b2, p_db2_[p], db2_nblk, d};
    j1.job[1] = {U + o.b1, p_db1_[p], csb_, f};
    j1.job[2] = {U + o.bo, p_dbo_[p], lnb_, d};
    j1.job[3] = {U + o.ln2g, p_g2_[p], lnb_, d};
    j1.job[4] = {U + o.ln2b, p_b2_[p], lnb_, d};
    j1.count = 5;
    if (o.n_bin) j1.job[j1.count++] = {U + o.bin, p_dbqkv_[p], csb_, (int)o.n_bin};
    sgd_multi(side_, j1);
    cudaEventRecord(ev_done_[p], side_);
    // LN1 backward: dx = dx1 + LN1'(da); its bf16 copy / column partials feed block j-1 and
    // go to the other parity's buffers, whose last reader (block j+1's side work) must be done
    cudaStreamWaitEvent(s, ev_done_[p ^ 1], 0);
    ln_bwd(s, da_, t.xin, t.mean1, t.rstd1, P + o.ln1g, dx1_, dx, want_next ? dy16_[p ^ 1] : nullptr, p_g1_, p_b1_,
           want_next ? p_db2_[p ^ 1] : nullptr, T, d);
    SgdJobs j2{};
    j2.lr = lr_;
    j2.job[0] = {U + o.ln1g, p_g1_, lnb_, d};
    j2.job[1] = {U + o.ln1b, p_b1_, lnb_, d};
    j2.count = 2;
    sgd_multi(s, j2);
    counters.launches += 5 + nl;
  }

  const Spec& spec_;
  std::vector<int> blocks_;
  int W_, d_, S_, B_, T_, fmax_, hmax_, csb_, lnb_;
  float lr_;
  std::vector<float*> w32_;
  std::vector<bf16*> w16_;
  std::vector<TfSlot> slots_;
  bool recompute_ = false;
  TfSlot rs_[2];          // recomputation scratch activations, by block parity
  float* ry_ = nullptr;   // recomputed block output (discarded)
  bf16 *dy16_[2], *dz_[2], *dx1_16_[2], *dqkv_[2], *do16_;
  float *da_, *dx1_, *gb_[2], *ws_ = nullptr;
  float* dcols_ = nullptr;
  unsigned long long* sc_acc_ = nullptr;
  int* sc_tick_ = nullptr;
  size_t ws_elems_ = 0;
  float *p_db2_[2], *p_db1_[2], *p_dbo_[2], *p_dbqkv_[2], *p_g2_[2], *p_b2_[2], *p_g1_, *p_b1_;
  cudaStream_t side_ = nullptr;
  cudaEvent_t ev_dz_, ev_da2_, ev_do_, ev_da_, ev_done_[2], ev_join_;
};

}  // namespace

std::unique_ptr<Family> make_family(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& arena,
                                    cudaStream_t s) {
  if (spec.family() == NASPIPE_MLP) return std::make_unique<MlpFamily>(spec, blocks, W, arena, s);
  if (spec.family() == NASPIPE_SPOS_CNN) return make_spos_family(spec, blocks, W, arena);
  return std::make_unique<TfFamily>(spec, blocks, W, arena, s);
}

}  // namespace naspipe
