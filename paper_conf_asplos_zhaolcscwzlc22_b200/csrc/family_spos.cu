// SPOS CNN family (configs[1]): ShuffleNetV2-style choice blocks {Shuffle 3/5/7, Xception}
// (SURVEY §8c "C2 SPOS candidate"; oracle/spos.py), frozen stem on the first stage and frozen
// head + cross-entropy on the last stage (reading A2).
//
// Layout: NHWC activations, forward tensors bf16x2 (hi plane + lo plane, 16-bit mantissa;
// DESIGN.md A28), gradients bf16; a block's output is stored in logical channel order
// concat(proj, main) (P:L579 SPOS blocks); the stride-1 channel split (even channels pass
// through, odd channels feed the main branch) is one kernel that writes the pass-through half
// straight into the block output and the main-branch input contiguously.  Every conv -> BN
// [-> ReLU] unit keeps z (bf16) and its batch mean / rstd in the slot's stash for the
// backward; 1x1 convs run on the tcgen05 GEMM (forward: z = x W^T as the 3-pass bf16x2
// product; dgrad: dx = dz W_hi; wgrad with the fused SGD WRITE: W -= lr dz^T x_hi,
// deterministic split-K over the pixels, refreshing W's hi/lo planes), depthwise convs and
// BatchNorm on CUDA cores (spos.cu).
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "family.h"
#include "launch.h"

namespace naspipe {

namespace {

struct UnitRec {  // forward stash of one unit of (slot, block)
  const bf16* x;  // unit input (hi plane; bf16x2); nullptr when xbn.z is set
  bf16* z;        // conv output (bf16x2, contiguous)
  float *mean, *rstd;  // [C] each, then the g, b snapshots [C] each (published when the
                       // unit's bn_apply is folded into its depthwise consumer)
  BnApplyIn xbn;  // depthwise unit whose input is the previous unit's BN applied on load
};

class SposFamily : public Family {
 public:
  SposFamily(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& A)
      : spec_(spec), blocks_(blocks), W_(W), B_(spec.B()), lr_(spec.raw.lr) {
    spec_base_ = &spec;
    n_choices_ = spec.n();
    const int nb = (int)blocks.size(), n = spec.n();
    first_ = blocks.front() == 0;
    last_ = blocks.back() == spec.m() - 1;
    w32_.assign((size_t)nb * n, nullptr);
    w16_.assign((size_t)nb * n, nullptr);
    plans_.resize((size_t)nb * n);
    dims_.resize(nb);
    size_t stash_max = 0, stats_max = 0, dz_max = 0, g_max = 0, blk_max = 0, dwk_max = 0, C_max = 0, dcols_max = 0;
    ws_elems_ = 0;
    for (int j = 0; j < nb; ++j) {
      const int b = blocks[j];
      const SposDims d = spec.spos_dims(b);
      dims_[j] = d;
      blk_max = std::max({blk_max, spec.grad_bytes(b) / 2, spec.grad_bytes(b + 1) / 2});
      for (int c = 0; c < n; ++c) {
        auto& L = plans_[(size_t)j * n + c];
        L = spec.spos_convs(b, c);
        // forward stash in bf16 elements: x2 tensors take two planes
        size_t need = d.stride == 1 ? 2 * P(d.H_in) * (d.C_out / 2) : 0, st = 0;
        for (size_t i = 0; i < L.size(); ++i) {
          const SposConv& u = L[i];
          const size_t po = P(u.H_out), pi = P(u.H_in);
          need += 2 * po * u.cout * (last_of_branch(L, i) ? 1 : 2);
          if (u.dw == 2) {  // dense conv: its x2 columns stay in the stash for the weight gradient
            need += 2 * po * (size_t)u.gemm_k();
            dcols_max = std::max(dcols_max, po * (size_t)u.gemm_k());
          }
          st += 4 * (size_t)u.cout;
          dz_max = std::max(dz_max, po * u.cout);
          g_max = std::max({g_max, pi * u.cin, po * u.cout});
          C_max = std::max(C_max, (size_t)u.cout);
          if (u.dw == 1) dwk_max = std::max(dwk_max, (size_t)u.cout * u.k * u.k);
          else
            ws_elems_ = std::max(ws_elems_, (size_t)gemm_splitk_factor(u.cout, u.gemm_k(), (int)po) * u.cout *
                                                u.gemm_k());
        }
        stash_max = std::max(stash_max, need);
        stats_max = std::max(stats_max, st);
      }
    }
    const int hw0 = spec.spos_stem_hw(), hwl = spec.spos_last_hw(), C0 = spec.raw.stem_channels,
              Cl = spec.chans.back(), Ch = spec.raw.head_channels, ncls = spec.raw.num_classes;
    if (last_) C_max = std::max(C_max, (size_t)Ch);
    if (first_) C_max = std::max(C_max, (size_t)C0);
    stash_.resize((size_t)W * nb);
    stats_.resize((size_t)W * nb);
    act_.assign((size_t)W * nb, nullptr);
    recs_.resize((size_t)W * nb);
    xin_.assign((size_t)W * nb, nullptr);
    for (int sl = 0; sl < W; ++sl)
      for (int j = 0; j < nb; ++j) {
        const size_t k = (size_t)sl * nb + j;
        stash_[k] = A.alloc<bf16>(stash_max);
        stats_[k] = A.alloc<float>(stats_max);
        if (j < nb - 1) act_[k] = A.alloc<bf16>(spec.act_bytes(blocks[j] + 1) / 2);
      }
    for (auto& d : dz_) d = A.alloc<bf16>(dz_max);
    create_stream(&side_, false);
    if (side_stream_sms() > 0) gemm_set_stream_cap(side_, side_stream_sms());
    for (int i = 0; i < kRing; ++i) {
      cudaEventCreateWithFlags(&ev_dg_[i], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&ev_wg_[i], cudaEventDisableTiming);
    }
    cudaEventCreateWithFlags(&ev_join_, cudaEventDisableTiming);
    g_[0] = A.alloc<bf16>(g_max);
    g_[1] = A.alloc<bf16>(g_max);
    gb_[0] = A.alloc<bf16>(blk_max);
    gb_[1] = A.alloc<bf16>(blk_max);
    gfirst_ = A.alloc<bf16>(g_max);
    // fixed-point BatchNorm accumulators + arrival tickets (zero between uses; spos.cu)
    // per channel count C of a use, acc[2C] is that use's overflow flag: size 2 C_max + 1
    // and zero everywhere, so every flag position starts (and, flags aside, stays) zero
    acc_f_ = A.alloc<unsigned long long>(2 * C_max + 1);
    acc_b_ = A.alloc<unsigned long long>(2 * C_max + 1);
    acc_f2_ = A.alloc<unsigned long long>(2 * C_max + 1);
    // bn_apply, bn_bwd_apply, dw weight gradient (side stream), depthwise conv with BN on load
    tick_ = A.alloc<int>(4);
    cudaMemset(acc_f_, 0, (2 * C_max + 1) * 8);
    cudaMemset(acc_b_, 0, (2 * C_max + 1) * 8);
    cudaMemset(acc_f2_, 0, (2 * C_max + 1) * 8);
    // ticket-free BatchNorm (kernels.h BnWrite note): rings of 3 accumulators per direction;
    // the fused-producer experiments keep the ticket path
    tfree_ = !fuse_bna_ && !fuse_bnb_ && !fuse_bnb_gemm_ && !getenv("NASPIPE_BN_TICKETS");  // A/B knob
    if (tfree_)
      for (int i = 0; i < 3; ++i) {
        ringF_[i] = A.alloc<unsigned long long>(2 * C_max + 1);
        ringB_[i] = A.alloc<unsigned long long>(2 * C_max + 1);
        cudaMemset(ringF_[i], 0, (2 * C_max + 1) * 8);
        cudaMemset(ringB_[i], 0, (2 * C_max + 1) * 8);
      }
    if (tfree_) {
      acc_f_ = ringF_[0];
      acc_b_ = ringB_[0];
    }
    C_max_ = (int)C_max;
    cudaMemset(tick_, 0, 4 * sizeof(int));
    dwk_max_ = dwk_max;
    acc_w_ = A.alloc<unsigned long long>(dwk_max + 1);
    cudaMemset(acc_w_, 0, (dwk_max + 1) * 8);
    ws_ = A.alloc<float>(std::max<size_t>(ws_elems_, 4));
    if (dcols_max) dcols_ = A.alloc<float>(dcols_max);  // dense conv input-gradient columns (fp32)
    if (first_) {
      std::vector<float> h(spec.frozen_count(0));
      spec.init_frozen(0, h.data());
      w_stem_ = A.alloc<float>(h.size());
      cudaMemcpy(w_stem_, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
      stem_z_ = A.alloc<bf16>(2 * P(hw0) * C0);
      stem_mean_ = A.alloc<float>(C0);
      stem_rstd_ = A.alloc<float>(C0);
      stem_y_.resize(W);
      for (auto& p : stem_y_) p = A.alloc<bf16>(2 * P(hw0) * C0);
      std::vector<float> ones(C0, 1.0f), zeros(C0, 0.0f);
      ones_s_ = A.alloc<float>(C0);
      zeros_s_ = A.alloc<float>(C0);
      cudaMemcpy(ones_s_, ones.data(), C0 * 4, cudaMemcpyHostToDevice);
      cudaMemcpy(zeros_s_, zeros.data(), C0 * 4, cudaMemcpyHostToDevice);
    }
    if (last_) {
      std::vector<float> h(spec.frozen_count(1));
      spec.init_frozen(1, h.data());
      std::vector<bf16> h16(2 * h.size());  // hi plane, lo plane
      for (size_t i = 0; i < h.size(); ++i) {
        h16[i] = __float2bfloat16_rn(h[i]);
        h16[h.size() + i] = __float2bfloat16_rn(h[i] - __bfloat162float(h16[i]));
      }
      wh16_ = A.alloc<bf16>(h16.size());
      cudaMemcpy(wh16_, h16.data(), h16.size() * 2, cudaMemcpyHostToDevice);
      std::vector<float> f(spec.frozen_count(2));
      spec.init_frozen(2, f.data());
      wf_ = A.alloc<float>(f.size());
      cudaMemcpy(wf_, f.data(), f.size() * 4, cudaMemcpyHostToDevice);
      std::vector<float> ones(Ch, 1.0f), zeros(Ch, 0.0f);
      ones_ = A.alloc<float>(Ch);
      zeros_ = A.alloc<float>(Ch);
      cudaMemcpy(ones_, ones.data(), Ch * 4, cudaMemcpyHostToDevice);
      cudaMemcpy(zeros_, zeros.data(), Ch * 4, cudaMemcpyHostToDevice);
      const size_t PL = P(hwl);
      zh_ = A.alloc<bf16>(2 * PL * Ch);
      rh_ = A.alloc<bf16>(2 * PL * Ch);
      dzh_ = A.alloc<bf16>(PL * Ch);
      hmean_ = A.alloc<float>(Ch);
      hrstd_ = A.alloc<float>(Ch);
      gap_ = A.alloc<float>((size_t)B_ * Ch);
      dgap_ = A.alloc<float>((size_t)B_ * Ch);
      dlogits_ = A.alloc<float>((size_t)B_ * ncls);
      logits_ = A.alloc<float>((size_t)B_ * ncls);
      loss_per_ = A.alloc<float>(B_);
    }
    (void)Cl;
  }

  void bind(int j, int c, float* w32, bf16* w16) override {
    w32_[(size_t)j * spec_.n() + c] = w32;
    w16_[(size_t)j * spec_.n() + c] = w16;
  }
  size_t shadow_elems(int j, int c) const override { return spec_.spos_shadow_elems(blocks_[j], c); }
  float* master(int j, int c) override { return w32_[(size_t)j * spec_.n() + c]; }
  void refresh_shadow(int j, int c, cudaStream_t s) override {
    float* p = master(j, c);
    bf16* w = w16_[(size_t)j * spec_.n() + c];
    const size_t half = shadow_elems(j, c) / 2;
    for (const SposConv& u : plans_[(size_t)j * spec_.n() + c])
      if (u.dw != 1) f32_to_bf16x2(s, p + u.off_w, w + u.off_w16, w + half + u.off_w16, u.weights());
  }

  void forward(int slot, const int32_t* ch, const void* x_in, void* x_out, cudaStream_t s) override {
    const int nb = (int)blocks_.size(), lo = rlo(), hi = rhi(nb);
    const bf16* x = static_cast<const bf16*>(x_in);
    if (first_ && lo == 0) {  // frozen stem: conv3x3 s2 -> BN(1, 0) batch statistics -> ReLU
      const int H = spec_.raw.image_hw, C0 = spec_.raw.stem_channels;
      const int Po = (int)P(H / 2);
      spos_stem_conv(s, static_cast<const float*>(x_in), w_stem_, stem_z_, B_, H, C0);
      counters.bytes += 4.0 * 3 * (double)P(H) + 4.0 * Po * C0;  // fp32 image in, z x2 out
      t_bn_stats(s, stem_z_, Po, C0, stem_mean_, stem_rstd_);
      t_bn_apply(s, stem_z_, Po, C0, stem_mean_, stem_rstd_, ones_s_, zeros_s_, 1, stem_y_[slot], C0, (size_t)Po * C0,
                 acc_f_);
      counters.launches += 3;
      x = stem_y_[slot];
    }
    for (int j = lo; j < hi; ++j) {
      const int c = ch[blocks_[j]];
      const size_t k = (size_t)slot * nb + j;
      bf16* out = (j == hi - 1) ? static_cast<bf16*>(x_out) : act_[k];
      xin_[k] = x;
      block_fwd(j, c, k, x, out, s);
      x = out;
    }
  }

  void backward(int slot, const int32_t* ch, const void* dy, void* dx, cudaStream_t s) override {
    const int nb = (int)blocks_.size(), lo = rlo(), hi = rhi(nb);
    const bf16* g = static_cast<const bf16*>(dy);
    for (int j = hi - 1; j >= lo; --j) {
      const int c = ch[blocks_[j]];
      const size_t k = (size_t)slot * nb + j;
      const bool need_dx = j > lo || dx != nullptr;
      bf16* out = (j == lo) ? static_cast<bf16*>(dx) : gb_[j & 1];
      block_bwd(j, c, k, g, out, need_dx, s);
      g = out;
    }
    if (tfree_ && bpend_.acc != nullptr) {  // the task's last deferred gamma / beta WRITE
      bn_write_flush(s, bpend_);
      bpend_ = BnWrite();
      counters.launches++;
    }
    // the task ends when its weight updates have landed (the next task may read them)
    cudaEventRecord(ev_join_, side_);
    cudaStreamWaitEvent(s, ev_join_, 0);
  }

  ~SposFamily() override {
    cudaStreamSynchronize(side_);
    for (int i = 0; i < kRing; ++i) {
      cudaEventDestroy(ev_dg_[i]);
      cudaEventDestroy(ev_wg_[i]);
    }
    cudaEventDestroy(ev_join_);
    cudaStreamDestroy(side_);
  }

  // Frozen head: pw Clast->Ch (tcgen05) -> BN(1,0) -> ReLU -> GAP -> FC (fp32) -> mean CE,
  // then its backward down to dL/d(stage output) (no parameter is updated, reading A2).
  void loss(int, const void* out, const void* target, void* dy, float* loss_dst, cudaStream_t s) override {
    const int hw = spec_.spos_last_hw(), HW = hw * hw, Cl = spec_.chans.back(), Ch = spec_.raw.head_channels,
              ncls = spec_.raw.num_classes;
    const int PL = (int)P(hw);
    GemmEpiParams e;
    e.out = zh_;
    e.out2 = zh_ + (size_t)PL * Ch;
    const bf16* xo = static_cast<const bf16*>(out);
    e.stats = acc_f_;  // fused bn_stats
    gemm_x2(s, PL, Ch, Cl, xo, xo + (size_t)PL * Cl, Cl, wh16_, wh16_ + (size_t)Ch * Cl, Cl, e);
    counters.bytes += 4.0 * PL * Cl + 4.0 * PL * Ch;
    t_bn_apply(s, zh_, PL, Ch, hmean_, hrstd_, ones_, zeros_, 1, rh_, Ch, (size_t)PL * Ch, acc_f_);
    gap_pool(s, rh_, B_, HW, Ch, gap_);
    counters.bytes += 4.0 * PL * Ch;
    fc_ce(s, gap_, wf_, static_cast<const int*>(target), B_, Ch, ncls, logits_, dlogits_, loss_per_);
    ce_mean(s, loss_per_, B_, loss_dst);
    fc_dgap(s, dlogits_, wf_, B_, Ch, ncls, dgap_);
    head_bcast(s, dgap_, B_, HW, Ch, rh_);  // dr overwrites r (the mask is recomputed from z)
    counters.bytes += 2.0 * PL * Ch;
    t_bn_bwd_reduce(s, rh_, Ch, zh_, PL, Ch, hmean_, hrstd_, ones_, zeros_, 1);
    t_bn_bwd_apply(s, rh_, Ch, zh_, PL, Ch, hmean_, hrstd_, ones_, zeros_, ones_, zeros_, 0, 1, dzh_);
    e = GemmEpiParams();
    e.out = dy;
    gemm(s, PL, Cl, Ch, dzh_, false, Ch, wh16_, true, Cl, EPI_BF16, e);
    counters.bytes += 2.0 * PL * Ch + 2.0 * PL * Cl;
    counters.launches += 9;
  }

  void check_after_drain() override {
    bool bad = false;  // a flag at acc[2C] of any use; the accumulators are zero elsewhere after a drain
    std::vector<unsigned long long> h(2 * (size_t)C_max_ + 1);
    std::vector<unsigned long long*> accs = {acc_f_, acc_b_, acc_f2_};
    if (tfree_) {
      // the last forward use's slot is cleared by the next use's apply: check its flag, clear it here
      unsigned long long* last = ringF_[(fu_ + 2) % 3];
      unsigned long long flag = 0;
      cudaMemcpy(&flag, last + fprev_n_, 8, cudaMemcpyDeviceToHost);
      bad |= flag != 0;
      cudaMemset(last, 0, ((size_t)fprev_n_ + 1) * 8);
      fprev_n_ = 0;
      accs = {ringF_[0], ringF_[1], ringF_[2], ringB_[0], ringB_[1], ringB_[2], acc_f2_};
    }
    for (const unsigned long long* a : accs) {
      cudaMemcpy(h.data(), a, h.size() * 8, cudaMemcpyDeviceToHost);
      for (auto v : h) bad |= v != 0;
    }
    h.resize(dwk_max_ + 1);
    cudaMemcpy(h.data(), acc_w_, h.size() * 8, cudaMemcpyDeviceToHost);
    for (auto v : h) bad |= v != 0;
    NP_REQUIRE(!bad, NASPIPE_EINTERNAL,
               "BatchNorm fixed-point accumulator overflow (a partial sum outside the 64-bit range, spos.cu)");
  }

  void synth_target(void* dst, uint64_t seed, cudaStream_t s) override {
    synth_labels(s, static_cast<int*>(dst), B_, spec_.raw.num_classes, seed);
  }

 private:
  size_t P(int hw) const { return (size_t)B_ * hw * hw; }
  static bool last_of_branch(const std::vector<SposConv>& L, size_t i) {
    return i + 1 == L.size() || L[i + 1].branch != L[i].branch;
  }
  // forward 1x1 conv: 3-pass bf16x2 product into z's hi/lo planes
  void gemm_x2(cudaStream_t s, int M, int N, int K, const bf16* Ahi, const bf16* Alo, int lda, const bf16* Bhi,
               const bf16* Blo, int ldb, const GemmEpiParams& ep) {
    gemm_bf16x2_tc(s, M, N, K, Ahi, Alo, lda, Bhi, Blo, ldb, EPI_X2, ep);
    counters.launches++;
  }

  void gemm(cudaStream_t s, int M, int N, int K, const bf16* A, bool amn, int lda, const bf16* B, bool bmn, int ldb,
            int epi, const GemmEpiParams& ep, bool split_ok = false) {
    GemmEpiParams e = ep;
    if (split_ok) {
      e.ws = ws_;
      e.ws_elems = ws_elems_;
    }
    gemm_bf16_tc(s, M, N, K, A, amn, lda, B, bmn, ldb, epi, e);
    counters.launches += (epi == EPI_SGD && gemm_splitk_factor(M, N, K) > 1) ? 2 : 1;
  }

  // BatchNorm kernels, the step's dominant kernel family (bench.py roofline):
  // with FLAG_TIMING each call is bracketed by CUDA events on its stream and credited with
  // its algorithmic HBM bytes (bf16x2 forward tensors 4 B/element, bf16 gradients 2 B).
  void t_bn_stats(cudaStream_t s, const bf16* z, int Pp, int C, float*, float*) {
    if (timer) timer->begin(s);
    bn_stats(s, z, Pp, C, acc_f_);
    if (timer) timer->end(s, 4.0 * Pp * C);
    counters.bytes += 4.0 * Pp * C;
  }
  void t_bn_apply(cudaStream_t s, const bf16* z, int Pp, int C, float* mean, float* rstd, const float* g,
                  const float* b, int relu, bf16* y, int ldy, size_t yplane, unsigned long long* acc) {
    if (timer) timer->begin(s);
    if (tfree_) {  // acc == ringF_[fu_ % 3]; zero the previous use's slot
      bn_apply(s, z, Pp, C, acc, nullptr, mean, rstd, g, b, relu, y, ldy, yplane, ringF_[(fu_ + 2) % 3], fprev_n_);
      fprev_n_ = 2 * C;
      acc_f_ = ringF_[++fu_ % 3];
    } else {
      bn_apply(s, z, Pp, C, acc, tick_, mean, rstd, g, b, relu, y, ldy, yplane);
    }
    if (timer) timer->end(s, 8.0 * Pp * C);
    counters.bytes += 8.0 * Pp * C;
  }
  void t_bn_bwd_reduce(cudaStream_t s, const bf16* dy, int lddy, const bf16* z, int Pp, int C, const float* mean,
                       const float* rstd, const float* g, const float* b, int relu) {
    if (timer) timer->begin(s);
    bn_bwd_reduce(s, dy, lddy, z, Pp, C, mean, rstd, g, b, relu, acc_b_);
    if (timer) timer->end(s, 6.0 * Pp * C);
    counters.bytes += 6.0 * Pp * C;
  }
  void t_bn_bwd_apply(cudaStream_t s, const bf16* dy, int lddy, const bf16* z, int Pp, int C, const float* mean,
                      const float* rstd, const float* g, const float* b, float* gu, float* bu, int update, int relu,
                      bf16* dz) {
    if (timer) timer->begin(s);
    if (tfree_) {  // acc_b_ == ringB_[bu_ % 3]; the previous use's WRITE is performed by this launch
      bn_bwd_apply(s, dy, lddy, z, Pp, C, mean, rstd, g, b, gu, bu, lr_, update, acc_b_, nullptr, relu, dz, bpend_);
      bpend_.gu = gu;
      bpend_.bu = bu;
      bpend_.g = g;
      bpend_.b = b;
      bpend_.acc = acc_b_;
      bpend_.C = C;
      bpend_.update = update;
      bpend_.lr = lr_;
      acc_b_ = ringB_[++bu_ % 3];
    } else {
      bn_bwd_apply(s, dy, lddy, z, Pp, C, mean, rstd, g, b, gu, bu, lr_, update, acc_b_, tick_ + 1, relu, dz);
    }
    if (timer) timer->end(s, 8.0 * Pp * C);
    counters.bytes += 8.0 * Pp * C;
  }

  void block_fwd(int j, int c, size_t k, const bf16* x, bf16* out, cudaStream_t s) {
    const SposDims& d = dims_[j];
    const auto& L = plans_[(size_t)j * spec_.n() + c];
    float* Pm = master(j, c);
    const bf16* W16 = w16_[(size_t)j * spec_.n() + c];
    bf16* cv = stash_[k];
    float* st = stats_[k];
    auto& recs = recs_[k];
    recs.clear();
    const size_t half = shadow_elems(j, c) / 2;  // lo planes of the 1x1 weights
    const size_t oplane = P(d.H_out) * d.C_out;   // planes of the block output
    const bf16* main_in = x;
    size_t main_plane = P(d.H_in) * d.C_in, x_plane = main_plane;
    int main_col = d.inp;  // column of the main branch in the block output
    if (d.stride == 1) {
      bf16* xm = cv;
      main_plane = P(d.H_in) * (d.C_out / 2);
      cv += 2 * main_plane;
      chan_split(s, x, (int)P(d.H_in), d.C_out / 2, out, d.C_out, oplane, xm);
      counters.bytes += 8.0 * P(d.H_in) * d.C_out;
      counters.launches++;
      main_in = xm;
      main_col = d.C_out / 2;
    }
    const bf16* h = nullptr;
    size_t hplane = 0;
    BnApplyIn pend;  // the previous unit's BN, folded into this depthwise conv's input load
    for (size_t i = 0; i < L.size(); ++i) {
      const SposConv& u = L[i];
      if (i == 0 || L[i - 1].branch != u.branch) {
        h = (u.branch == 0) ? x : main_in;
        hplane = (u.branch == 0) ? x_plane : main_plane;
      }
      const int Po = (int)P(u.H_out);
      const size_t zplane = (size_t)Po * u.cout;
      UnitRec r{h, cv, st, st + u.cout, BnApplyIn()};
      cv += 2 * zplane;
      st += 4 * u.cout;
      // the depthwise conv adds the BatchNorm sums of its output itself (fused bn_stats); with
      // its input's BN applied on load it reads acc_f_ and so adds its own sums to acc_f2_
      unsigned long long* zacc = acc_f_;
      if (u.dw == 1 && pend.z != nullptr) {
        r.x = nullptr;
        r.xbn = pend;
        zacc = acc_f2_;
        dw_fwd_bn(s, pend, Pm + u.off_w, r.z, B_, u.H_in, u.cin, u.k, u.stride, u.dil, zacc);
        counters.bytes += 4.0 * P(u.H_in) * u.cin + 4.0 * Po * u.cout;
        counters.launches++;
        pend = BnApplyIn();
      } else if (u.dw == 1) {
        dw_fwd(s, h, Pm + u.off_w, r.z, B_, u.H_in, u.cin, u.k, u.stride, u.dil, zacc);
        counters.bytes += 4.0 * P(u.H_in) * u.cin + 4.0 * Po * u.cout;
        counters.launches++;
      } else if (u.dw == 2) {  // dense k x k (reading A40): x2 columns, 3-pass GEMM over K = k k cin
        const int gk = u.gemm_k();
        const size_t cplane = (size_t)Po * gk;
        bf16* cols = cv;
        cv += 2 * cplane;
        im2col_x2(s, h, hplane, B_, u.H_in, u.cin, u.k, u.stride, cols, cplane);
        counters.bytes += 4.0 * P(u.H_in) * u.cin + 4.0 * (double)cplane;
        counters.launches++;
        r.x = cols;  // the weight gradient reads the columns' hi plane
        GemmEpiParams e;  // the GEMM epilogue adds the BatchNorm sums of z (fused bn_stats)
        e.out = r.z;
        e.out2 = r.z + zplane;
        e.stats = acc_f_;
        gemm_x2(s, Po, u.cout, gk, cols, cols + cplane, gk, W16 + u.off_w16, W16 + half + u.off_w16, gk, e);
        counters.bytes += 4.0 * (double)cplane + 4.0 * Po * u.cout;
      } else {
        GemmEpiParams e;  // the GEMM epilogue adds the BatchNorm sums of z (fused bn_stats)
        e.out = r.z;
        e.out2 = r.z + zplane;
        e.stats = acc_f_;
        gemm_x2(s, Po, u.cout, u.cin, h, h + hplane, u.cin, W16 + u.off_w16, W16 + half + u.off_w16, u.cin, e);
        counters.bytes += 4.0 * Po * u.cin + 4.0 * Po * u.cout;
      }
      if (fuse_bna_ && u.dw == 0 && !last_of_branch(L, i) && L[i + 1].dw == 1) {
        // conv -> BN -> ReLU -> depthwise: no bn_apply; the depthwise conv applies it on load
        // (and its last CTA publishes this unit's mean / rstd and the g / b it used)
        pend.z = r.z;
        pend.zplane = zplane;
        pend.P = Po;
        pend.acc = acc_f_;
        pend.ticket = tick_ + 3;
        pend.mean = r.mean;
        pend.rstd = r.rstd;
        pend.g = Pm + u.off_g;
        pend.b = Pm + u.off_b;
        pend.gsnap = r.rstd + u.cout;
        pend.bsnap = r.rstd + 2 * u.cout;
        pend.relu = u.relu;
        recs.push_back(r);
        h = nullptr;
        continue;
      }
      bf16* y;
      int ldy;
      size_t yplane;
      if (last_of_branch(L, i)) {
        y = out + (u.branch == 0 ? 0 : main_col);
        ldy = d.C_out;
        yplane = oplane;
      } else {
        y = cv;
        yplane = zplane;
        cv += 2 * zplane;
        ldy = u.cout;
      }
      t_bn_apply(s, r.z, Po, u.cout, r.mean, r.rstd, Pm + u.off_g, Pm + u.off_b, u.relu, y, ldy, yplane, zacc);
      hplane = yplane;
      counters.launches += 1;
      recs.push_back(r);
      h = y;
    }
  }

  // One unit's BN backward (+ the WRITE of its gamma/beta), leaves dz in the next ring
  // buffer dz_[ring_] (whose previous reader, a weight-gradient on the side stream, is done).
  // reduced: the producer of dy already added the reduction's sums (BnBwdFuse), so only the
  // apply runs.
  void unit_bn_bwd(const SposConv& u, const UnitRec& r, float* Pm, float* Um, const bf16* dy, int lddy, bool reduced,
                   cudaStream_t s) {
    const int Po = (int)P(u.H_out);
    ring_ = (ring_ + 1) % kRing;
    if (ring_used_[ring_]) cudaStreamWaitEvent(s, ev_wg_[ring_], 0);
    if (!reduced) {
      t_bn_bwd_reduce(s, dy, lddy, r.z, Po, u.cout, r.mean, r.rstd, Pm + u.off_g, Pm + u.off_b, u.relu);
      counters.launches += 1;
    }
    t_bn_bwd_apply(s, dy, lddy, r.z, Po, u.cout, r.mean, r.rstd, Pm + u.off_g, Pm + u.off_b, Um + u.off_g, Um + u.off_b,
                   1, u.relu, dz_[ring_]);
    counters.launches += 1;
  }
  // the fused BatchNorm-backward reduction of unit `v` (record r) for the kernel producing its
  // output gradient: stride-1 depthwise input gradients and 1x1-conv input gradients (GEMM
  // epilogue EPI_BNBWD); the pre-update g, b (reading A4), as bn_bwd_reduce reads them
  bool fusable_producer(const SposConv& u) const {
    return u.dw == 1 ? fuse_bnb_ : (u.dw == 0 ? fuse_bnb_gemm_ : false);
  }
  BnBwdFuse bnb_of(const SposConv& v, const UnitRec& r, const float* Pm) const {
    BnBwdFuse f;
    f.z = r.z;
    f.zplane = P(v.H_out) * (size_t)v.cout;
    f.mean = r.mean;
    f.rstd = r.rstd;
    f.g = Pm + v.off_g;
    f.b = Pm + v.off_b;
    f.relu = v.relu;
    f.acc = acc_b_;
    return f;
  }

  // conv backward of one unit from dz: the input gradient into dst (+ add) with the
  // pre-update weights on the stage stream (skipped if dst == nullptr); then, on the side
  // stream once that has been issued, the weight gradient with the SGD WRITE (reading A4),
  // overlapping the rest of the input-gradient chain.
  void unit_conv_bwd(const SposConv& u, const UnitRec& r, float* Pm, float* Um, bool inplace, bf16* W16, size_t half,
                     bf16* dst, const bf16* add, cudaStream_t s, const BnBwdFuse* fuse = nullptr) {
    const int Po = (int)P(u.H_out);
    const bf16* dz = dz_[ring_];
    if (dst) {
      if (u.dw == 1) {
        dw_dgrad(s, dz, Pm + u.off_w, add, dst, B_, u.H_in, u.cin, u.k, u.stride, u.dil, fuse ? *fuse : BnBwdFuse());
        counters.bytes += 2.0 * Po * u.cout + 2.0 * P(u.H_in) * u.cin * (add ? 2 : 1);
        counters.launches++;
      } else if (u.dw == 2) {  // dense: dcols = dz W (fp32), then the fixed-order column adjoint
        GemmEpiParams e;
        e.out = dcols_;
        gemm(s, Po, u.gemm_k(), u.cout, dz, false, u.cout, W16 + u.off_w16, true, u.gemm_k(), EPI_F32, e);
        col2im(s, dcols_, B_, u.H_in, u.cin, u.k, u.stride, add, dst);
        counters.bytes += 2.0 * Po * u.cout + 8.0 * Po * u.gemm_k() + 2.0 * P(u.H_in) * u.cin * (add ? 2 : 1);
        counters.launches++;
      } else {
        NP_REQUIRE(add == nullptr, NASPIPE_EINTERNAL, "pw dgrad with an addend");
        GemmEpiParams e;
        e.out = dst;
        if (fuse) e.bnb = *fuse;
        gemm(s, Po, u.cin, u.cout, dz, false, u.cout, W16 + u.off_w16, true, u.cin, fuse ? EPI_BNBWD : EPI_BF16, e);
        counters.bytes += 2.0 * Po * u.cout + 2.0 * Po * u.cin;
      }
    }
    cudaEventRecord(ev_dg_[ring_], s);
    cudaStreamWaitEvent(side_, ev_dg_[ring_], 0);
    if (u.dw == 1) {
      counters.bytes += 2.0 * Po * u.cout + (r.xbn.z ? 4.0 : 2.0) * P(u.H_in) * u.cin;
      dw_wgrad_sgd(side_, dz, r.x, acc_w_, tick_ + 2, Um + u.off_w, lr_, B_, u.H_in, u.cin, u.k, u.stride, u.dil,
                   r.xbn.z ? &r.xbn : nullptr);
      counters.launches += 1;
    } else {
      GemmEpiParams e;
      e.w32 = Um + u.off_w;  // the BSP accumulator has no shadow (refreshed at the flush)
      e.w16 = inplace ? W16 + u.off_w16 : nullptr;
      e.w16lo = inplace ? W16 + half + u.off_w16 : nullptr;
      e.lr = lr_;
      counters.bytes += 2.0 * Po * u.cout + 2.0 * Po * u.gemm_k();
      gemm(side_, u.cout, u.gemm_k(), Po, dz, true, u.cout, r.x, true, u.gemm_k(), EPI_SGD, e, true);
    }
    cudaEventRecord(ev_wg_[ring_], side_);
    ring_used_[ring_] = true;
  }

  void block_bwd(int j, int c, size_t k, const bf16* dyb, bf16* dxb, bool need_dx, cudaStream_t s) {
    const SposDims& d = dims_[j];
    const auto& L = plans_[(size_t)j * spec_.n() + c];
    float* Pm = master(j, c);
    float* Um = upd(j, c);
    const bool inplace = in_place(j, c);
    bf16* W16 = w16_[(size_t)j * spec_.n() + c];
    const size_t half = shadow_elems(j, c) / 2;
    const auto& recs = recs_[k];
    const int main_col = d.stride == 1 ? d.C_out / 2 : d.inp;
    size_t m0 = 0;  // first main-branch unit
    while (m0 < L.size() && L[m0].branch == 0) ++m0;
    // ---- main branch, last unit first
    const bf16* h = dyb + main_col;
    int ldh = d.C_out;
    int pp = 0;
    bool reduced = false;  // the producer of h added unit i's BatchNorm-backward sums
    for (size_t i = L.size(); i-- > m0;) {
      const SposConv& u = L[i];
      unit_bn_bwd(u, recs[i], Pm, Um, h, ldh, reduced, s);
      bf16* dst;
      if (i > m0) dst = g_[pp ^= 1];
      else dst = need_dx ? (d.stride == 1 ? g_[pp ^ 1] : gfirst_) : nullptr;
      reduced = i > m0 && fusable_producer(u);
      BnBwdFuse f;
      if (reduced) f = bnb_of(L[i - 1], recs[i - 1], Pm);
      unit_conv_bwd(u, recs[i], Pm, Um, inplace, W16, half, dst, nullptr, s, reduced ? &f : nullptr);
      h = dst;
      ldh = u.cin;
    }
    if (d.stride == 1) {
      if (need_dx) {
        chan_merge(s, dyb, d.C_out, h, (int)P(d.H_in), d.C_out / 2, dxb);
        counters.bytes += 4.0 * P(d.H_in) * d.C_out;
        counters.launches++;
      }
      return;
    }
    // ---- stride 2: proj branch (dw s2 -> BN -> pw -> BN -> ReLU); its input gradient adds
    // the main branch's (both branches read the block input)
    const bf16* hp = dyb;
    int ldp = d.C_out;
    reduced = false;
    for (size_t i = m0; i-- > 0;) {
      const SposConv& u = L[i];
      unit_bn_bwd(u, recs[i], Pm, Um, hp, ldp, reduced, s);
      bf16* dst = i > 0 ? g_[pp ^= 1] : (need_dx ? dxb : nullptr);
      reduced = i > 0 && fusable_producer(u);
      BnBwdFuse f;
      if (reduced) f = bnb_of(L[i - 1], recs[i - 1], Pm);
      unit_conv_bwd(u, recs[i], Pm, Um, inplace, W16, half, dst, (i == 0 && need_dx) ? gfirst_ : nullptr, s,
                    reduced ? &f : nullptr);
      hp = dst;
      ldp = u.cin;
    }
  }

  const Spec& spec_;
  std::vector<int> blocks_;
  int W_, B_;
  float lr_;
  bool first_ = false, last_ = false;
  std::vector<float*> w32_;
  std::vector<bf16*> w16_;
  std::vector<std::vector<SposConv>> plans_;
  std::vector<SposDims> dims_;
  std::vector<bf16*> stash_, act_;
  std::vector<float*> stats_;
  std::vector<std::vector<UnitRec>> recs_;
  std::vector<const bf16*> xin_;
  static constexpr int kRing = 3;  // dz buffers shared by the stage stream and the side stream
  bf16 *dz_[kRing], *g_[2], *gb_[2], *gfirst_;
  int ring_ = 0;
  bool ring_used_[kRing] = {false, false, false};
  cudaStream_t side_ = nullptr;  // weight gradients + SGD of the backward
  cudaEvent_t ev_dg_[kRing], ev_wg_[kRing], ev_join_;
  float* ws_;
  float* dcols_ = nullptr;  // dense conv: fp32 input-gradient columns (stage stream)
  unsigned long long *acc_f_, *acc_b_;  // BatchNorm fixed-point accumulators (forward / backward)
  unsigned long long* acc_f2_;          // forward sums of a depthwise conv that reads acc_f_ (BN on load)
  // ticket-free mode: acc_f_ / acc_b_ point at ring slot fu_ % 3 / bu_ % 3 of the next use
  bool tfree_ = false;
  unsigned long long *ringF_[3] = {}, *ringB_[3] = {};
  int64_t fu_ = 0, bu_ = 0;
  int fprev_n_ = 0;  // 2 C of the previous forward use (its slot is zeroed by the next apply)
  BnWrite bpend_;    // the backward WRITE deferred to the next apply (or the task's flush)
  unsigned long long* acc_w_ = nullptr; // depthwise weight gradient accumulator (side stream)
  size_t dwk_max_ = 0;
  int* tick_;                           // [2] arrival tickets of bn_apply / bn_bwd_apply
  int C_max_ = 0;
  size_t ws_elems_ = 0;
  // BatchNorm-backward reductions fused into the depthwise producers of dy
  // (NASPIPE_SPOS_FUSE_BNB=1; off by default: measured slower)
  const bool fuse_bnb_ = [] {
    const char* e = getenv("NASPIPE_SPOS_FUSE_BNB");
    return e && e[0] == '1';
  }();
  // ... and into the 1x1-conv input-gradient GEMM's epilogue (EPI_BNBWD): off by default --
  // measured slower (the epilogue's extra z reads and per-tile sums cost more than the
  // reduce launch they remove: +0.7 ms per configs[1] step); NASPIPE_SPOS_FUSE_BNB_GEMM=1
  const bool fuse_bnb_gemm_ = [] {
    const char* e = getenv("NASPIPE_SPOS_FUSE_BNB_GEMM");
    return e && e[0] == '1';
  }();
  // bn_apply of a conv -> BN -> ReLU unit folded into its depthwise consumer's load
  // (NASPIPE_SPOS_FUSE_BNA=1; off by default: measured neutral to slower)
  const bool fuse_bna_ = [] {
    const char* e = getenv("NASPIPE_SPOS_FUSE_BNA");
    return e && e[0] == '1';
  }();
  // stem
  float* w_stem_ = nullptr;
  bf16* stem_z_ = nullptr;
  float *stem_mean_ = nullptr, *stem_rstd_ = nullptr, *ones_s_ = nullptr, *zeros_s_ = nullptr;
  std::vector<bf16*> stem_y_;
  // head
  bf16 *wh16_ = nullptr, *zh_ = nullptr, *rh_ = nullptr, *dzh_ = nullptr;
  float *wf_ = nullptr, *ones_ = nullptr, *zeros_ = nullptr, *hmean_ = nullptr, *hrstd_ = nullptr, *gap_ = nullptr,
        *dgap_ = nullptr, *dlogits_ = nullptr, *logits_ = nullptr, *loss_per_ = nullptr;
};

}  // namespace

std::unique_ptr<Family> make_spos_family(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& arena) {
  return std::make_unique<SposFamily>(spec, blocks, W, arena);
}

}  // namespace naspipe
