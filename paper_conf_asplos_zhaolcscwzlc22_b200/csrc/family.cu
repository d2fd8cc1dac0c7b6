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
  if (!on) return;
  cudaEventRecord(pairs[used].second, s);
  ++used;
  flops += f;
  launches += 1;
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
    const size_t P = spec.param_count(0, 0), act = (size_t)B_ * d_;
    params_.resize((size_t)nb * n);
    std::vector<float> host(P);
    for (int j = 0; j < nb; ++j)
      for (int c = 0; c < n; ++c) {
        float* p = A.alloc<float>(P);
        spec.init_params(blocks[j], c, host.data());
        cudaMemcpyAsync(p, host.data(), P * 4, cudaMemcpyHostToDevice, s);
        cudaStreamSynchronize(s);
        params_[(size_t)j * n + c] = p;
      }
    h_.resize((size_t)W * nb);
    act_.resize((size_t)W * nb);
    xin_.assign((size_t)W * nb, nullptr);
    for (auto& p : h_) p = A.alloc<float>(act);
    for (auto& p : act_) p = A.alloc<float>(act);
    g_[0] = A.alloc<float>(act);
    g_[1] = A.alloc<float>(act);
  }
  float* master(int j, int c) override { return params_[(size_t)j * spec_.n() + c]; }
  void refresh_shadow(int, int, cudaStream_t) override {}

  void forward(int slot, const int32_t* ch, const float* x_in, float* x_out, cudaStream_t s) override {
    const int nb = (int)blocks_.size();
    const float* x = x_in;
    for (int j = 0; j < nb; ++j) {
      float* P = master(j, ch[blocks_[j]]);
      float* y = (j == nb - 1) ? x_out : act_[(size_t)slot * nb + j + 1];
      xin_[(size_t)slot * nb + j] = x;
      mlp_fwd(s, x, P, P + (size_t)d_ * d_, y, h_[(size_t)slot * nb + j], B_, d_);
      counters.launches++;
      x = y;
    }
  }
  void backward(int slot, const int32_t* ch, const float* dy, float* dx, cudaStream_t s) override {
    const int nb = (int)blocks_.size();
    const float* g = dy;
    for (int j = nb - 1; j >= 0; --j) {
      float* P = master(j, ch[blocks_[j]]);
      float* out = (j == 0) ? dx : g_[j & 1];
      mlp_bwd_sgd(s, xin_[(size_t)slot * nb + j], h_[(size_t)slot * nb + j], g, out, P, P + (size_t)d_ * d_, lr_,
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
    w32_.resize((size_t)nb * n);
    w16_.resize((size_t)nb * n);
    for (int j = 0; j < nb; ++j)
      for (int c = 0; c < n; ++c) {
        const TfOffsets o = spec.tf_offsets(c);
        const size_t f = spec.ffn[c];
        float* p = A.alloc<float>(o.total);
        std::vector<float> host(o.total);
        spec.init_params(blocks[j], c, host.data());
        cudaMemcpyAsync(p, host.data(), o.total * 4, cudaMemcpyHostToDevice, s);
        cudaStreamSynchronize(s);
        w32_[(size_t)j * n + c] = p;
        w16_[(size_t)j * n + c] = A.alloc<bf16>(4 * (size_t)d_ * d_ + 2 * (size_t)d_ * f);
        refresh_shadow(j, c, s);
      }
    const size_t Td = (size_t)T_ * d_;
    slots_.resize((size_t)W * nb);
    for (int sl = 0; sl < W; ++sl)
      for (int j = 0; j < nb; ++j) {
        TfSlot& t = slots_[(size_t)sl * nb + j];
        t.act = (j > 0) ? A.alloc<float>(Td) : nullptr;
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
      }
    // backward workspace (tasks on a stage are serialised on its stream)
    dy16_ = A.alloc<bf16>(Td);
    dz_ = A.alloc<bf16>((size_t)T_ * fmax_);
    da_ = A.alloc<float>(Td);
    dx1_ = A.alloc<float>(Td);
    dx1_16_ = A.alloc<bf16>(Td);
    do16_ = A.alloc<bf16>(Td);
    dqkv_ = A.alloc<bf16>(3 * Td);
    gb_[0] = A.alloc<float>(Td);
    gb_[1] = A.alloc<float>(Td);
    // split-K workspace: the largest splits * M * N over this stage's GEMMs
    ws_elems_ = 0;
    for (int c = 0; c < n; ++c) {
      const int f = spec.ffn[c], T = T_, d = d_;
      const int shp[6][3] = {{d, f, T}, {f, d, T}, {d, d, T}, {3 * d, d, T}, {T, d, f}, {T, d, 3 * d}};
      for (auto& q : shp)
        ws_elems_ = std::max(ws_elems_, (size_t)gemm_splitk_factor(q[0], q[1], q[2]) * q[0] * q[1]);
    }
    ws_ = A.alloc<float>(ws_elems_);
    csb_ = colsum_blocks(T_);
    lnb_ = ln_bwd_blocks(T_);
    const int pb = std::max(csb_, lnb_);
    p_db2_ = A.alloc<float>((size_t)pb * d_);
    p_db1_ = A.alloc<float>((size_t)csb_ * fmax_);
    p_dbo_ = A.alloc<float>((size_t)lnb_ * d_);
    p_dbqkv_ = A.alloc<float>((size_t)csb_ * 3 * d_);
    p_g1_ = A.alloc<float>((size_t)lnb_ * d_);
    p_b1_ = A.alloc<float>((size_t)lnb_ * d_);
    p_g2_ = A.alloc<float>((size_t)lnb_ * d_);
    p_b2_ = A.alloc<float>((size_t)lnb_ * d_);
  }

  float* master(int j, int c) override { return w32_[(size_t)j * spec_.n() + c]; }

  void refresh_shadow(int j, int c, cudaStream_t s) override {
    const TfOffsets o = spec_.tf_offsets(c);
    const size_t d = d_, f = spec_.ffn[c];
    float* p = master(j, c);
    bf16* w = w16_[(size_t)j * spec_.n() + c];
    f32_to_bf16(s, p + o.Wqkv, w, 3 * d * d);
    f32_to_bf16(s, p + o.Wo, w + 3 * d * d, d * d);
    f32_to_bf16(s, p + o.W1, w + 4 * d * d, f * d);
    f32_to_bf16(s, p + o.W2, w + 4 * d * d + f * d, d * f);
  }

  void forward(int slot, const int32_t* ch, const float* x_in, float* x_out, cudaStream_t s) override {
    const int nb = (int)blocks_.size();
    const float* x = x_in;
    for (int j = 0; j < nb; ++j) {
      const int c = ch[blocks_[j]];
      TfSlot& t = slots_[(size_t)slot * nb + j];
      t.xin = x;
      float* y = (j == nb - 1) ? x_out : slots_[(size_t)slot * nb + j + 1].act;
      block_fwd(j, c, t, y, s);
      x = y;
    }
  }

  void backward(int slot, const int32_t* ch, const float* dy, float* dx, cudaStream_t s) override {
    const int nb = (int)blocks_.size();
    const float* g = dy;
    int db2_nblk = 0;
    for (int j = nb - 1; j >= 0; --j) {
      const int c = ch[blocks_[j]];
      TfSlot& t = slots_[(size_t)slot * nb + j];
      if (j == nb - 1) {  // grad entering the stage: bf16 copy + colsum for b2
        cast_colsum(s, g, dy16_, p_db2_, T_, d_);
        counters.launches++;
        db2_nblk = lnb_;
      }
      // stage 0 needs no input gradient, but LN1's backward still runs (dgamma/dbeta):
      // its dx goes to a scratch buffer (gb_[0] is free: block 1 wrote gb_[1])
      float* out = (j == 0) ? (dx ? dx : gb_[0]) : gb_[j & 1];
      block_bwd(j, c, t, g, out, /*want_next=*/j > 0, db2_nblk, s);
      db2_nblk = lnb_;
      g = out;
    }
  }

 private:
  void gemm(cudaStream_t s, int M, int N, int K, const bf16* A, bool amn, int lda, const bf16* B, bool bmn, int ldb,
            int epi, const GemmEpiParams& ep) {
    if (timer) timer->begin(s);
    GemmEpiParams e = ep;
    e.ws = ws_;
    e.ws_elems = ws_elems_;
    gemm_bf16_tc(s, M, N, K, A, amn, lda, B, bmn, ldb, epi, e);
    if (timer) timer->end(s, 2.0 * M * N * K);
    counters.launches++;
  }

  void block_fwd(int j, int c, TfSlot& t, float* y, cudaStream_t s) {
    const TfOffsets o = spec_.tf_offsets(c);
    const int d = d_, f = spec_.ffn[c], h = spec_.heads[c], T = T_;
    float* P = master(j, c);
    bf16* W = w16_[(size_t)j * spec_.n() + c];
    const bf16 *Wqkv = W, *Wo = W + 3 * (size_t)d * d, *W1 = W + 4 * (size_t)d * d,
               *W2 = W1 + (size_t)f * d;
    ln_fwd(s, t.xin, P + o.ln1g, P + o.ln1b, t.a, t.mean1, t.rstd1, T, d);
    GemmEpiParams e1;
    e1.bias = P + o.bqkv;
    e1.out = t.qkv;
    gemm(s, T, 3 * d, d, t.a, false, d, Wqkv, false, d, EPI_BIAS_BF16, e1);
    attn_fwd(s, t.qkv, t.o, t.lse, B_, S_, d, h);
    GemmEpiParams e2;
    e2.bias = P + o.bo;
    e2.resid = t.xin;
    e2.out = t.x1;
    gemm(s, T, d, d, t.o, false, d, Wo, false, d, EPI_BIAS_RESID_F32, e2);
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

  // dy: f32 grad of the block output (its bf16 copy is in dy16_, its column partials in
  // p_db2_[0..db2_nblk)); writes dx (f32); if want_next also dy16_/p_db2_ for block j-1.
  void block_bwd(int j, int c, TfSlot& t, const float* dy, float* dx, bool want_next, int db2_nblk,
                 cudaStream_t s) {
    const TfOffsets o = spec_.tf_offsets(c);
    const int d = d_, f = spec_.ffn[c], h = spec_.heads[c], T = T_;
    float* P = master(j, c);
    bf16* W = w16_[(size_t)j * spec_.n() + c];
    bf16 *Wqkv = W, *Wo = W + 3 * (size_t)d * d, *W1 = W + 4 * (size_t)d * d, *W2 = W1 + (size_t)f * d;
    // FFN half
    GemmEpiParams e;
    e.aux16 = t.z;
    e.out = dz_;
    gemm(s, T, f, d, dy16_, false, d, W2, true, f, EPI_DGELU, e);          // dz = (dy W2) * gelu'(z)
    e = GemmEpiParams();
    e.w32 = P + o.W2;
    e.w16 = W2;
    e.lr = lr_;
    gemm(s, d, f, T, dy16_, true, d, t.g, true, f, EPI_SGD, e);            // W2 -= lr dy^T g
    colsum_bf16(s, dz_, p_db1_, T, f);
    e = GemmEpiParams();
    e.out = da_;
    gemm(s, T, d, f, dz_, false, f, W1, true, d, EPI_F32, e);               // da2 = dz W1
    e = GemmEpiParams();
    e.w32 = P + o.W1;
    e.w16 = W1;
    e.lr = lr_;
    gemm(s, f, d, T, dz_, true, f, t.a2, true, d, EPI_SGD, e);             // W1 -= lr dz^T a2
    ln_bwd(s, da_, t.x1, t.mean2, t.rstd2, P + o.ln2g, dy, dx1_, dx1_16_, p_g2_, p_b2_, p_dbo_, T, d);
    // attention half
    e = GemmEpiParams();
    e.out = do16_;
    gemm(s, T, d, d, dx1_16_, false, d, Wo, true, d, EPI_BF16, e);          // do = dx1 Wo
    e = GemmEpiParams();
    e.w32 = P + o.Wo;
    e.w16 = Wo;
    e.lr = lr_;
    gemm(s, d, d, T, dx1_16_, true, d, t.o, true, d, EPI_SGD, e);          // Wo -= lr dx1^T o
    attn_bwd(s, t.qkv, t.o, t.lse, do16_, dqkv_, B_, S_, d, h);
    colsum_bf16(s, dqkv_, p_dbqkv_, T, 3 * d);
    e = GemmEpiParams();
    e.out = da_;
    gemm(s, T, d, 3 * d, dqkv_, false, 3 * d, Wqkv, true, d, EPI_F32, e);  // da = dqkv Wqkv
    e = GemmEpiParams();
    e.w32 = P + o.Wqkv;
    e.w16 = Wqkv;
    e.lr = lr_;
    gemm(s, 3 * d, d, T, dqkv_, true, 3 * d, t.a, true, d, EPI_SGD, e);    // Wqkv -= lr dqkv^T a
    // bias / LN2 updates (their partials are complete; LN1 partials come next)
    SgdJobs j1{};
    j1.lr = lr_;
    j1.job[0] = {P + o.b2, p_db2_, db2_nblk, d};
    j1.job[1] = {P + o.b1, p_db1_, csb_, f};
    j1.job[2] = {P + o.bo, p_dbo_, lnb_, d};
    j1.job[3] = {P + o.bqkv, p_dbqkv_, csb_, 3 * d};
    j1.job[4] = {P + o.ln2g, p_g2_, lnb_, d};
    j1.job[5] = {P + o.ln2b, p_b2_, lnb_, d};
    j1.count = 6;
    sgd_multi(s, j1);
    // LN1 backward: dx = dx1 + LN1'(da); bf16 copy / column partials feed block j-1
    ln_bwd(s, da_, t.xin, t.mean1, t.rstd1, P + o.ln1g, dx1_, dx, want_next ? dy16_ : nullptr, p_g1_, p_b1_,
           want_next ? p_db2_ : nullptr, T, d);
    SgdJobs j2{};
    j2.lr = lr_;
    j2.job[0] = {P + o.ln1g, p_g1_, lnb_, d};
    j2.job[1] = {P + o.ln1b, p_b1_, lnb_, d};
    j2.count = 2;
    sgd_multi(s, j2);
    counters.launches += 7;
  }

  const Spec& spec_;
  std::vector<int> blocks_;
  int W_, d_, S_, B_, T_, fmax_, hmax_, csb_, lnb_;
  float lr_;
  std::vector<float*> w32_;
  std::vector<bf16*> w16_;
  std::vector<TfSlot> slots_;
  bf16 *dy16_, *dz_, *dx1_16_, *do16_, *dqkv_;
  float *da_, *dx1_, *gb_[2], *ws_ = nullptr;
  size_t ws_elems_ = 0;
  float *p_db2_, *p_db1_, *p_dbo_, *p_dbqkv_, *p_g1_, *p_b1_, *p_g2_, *p_b2_;
};

}  // namespace

std::unique_ptr<Family> make_family(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& arena,
                                    cudaStream_t s) {
  if (spec.family() == NASPIPE_MLP) return std::make_unique<MlpFamily>(spec, blocks, W, arena, s);
  return std::make_unique<TfFamily>(spec, blocks, W, arena, s);
}

}  // namespace naspipe
