// Supernet specification: validated deep copy of naspipe_supernet_spec, parameter layouts,
// the analytic cost table, the balanced partition and the counter-hash initialiser.
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>

#include "common.h"

namespace naspipe {

// contiguous partition of per-block weights into D stages minimising the max stage weight,
// ties -> lexicographically smallest split points (reading A12)
std::vector<int32_t> balanced_partition(const std::vector<int64_t>& w, int D);

// One tensor of a candidate's packed parameter vector.
struct Segment {
  size_t offset, size;
  int kind;      // 0 = uniform(+-1/sqrt(fan_in)), 1 = ones, 2 = zeros
  int fan_in;
};

// Offsets (in floats) of the transformer candidate tensors in the packed vector
// (packing order of include/naspipe.h).
// Transformer-family candidate (oracle/transformer.py layout).  The token mixer (reading A38)
// is op: 0 attention (Win = Wqkv [3d,d], bin = bqkv, Wo [d,d], bo), 1 Conv 3x1 (Wo = Wc [d,3d],
// bo = bc), 2 Sep Conv 7x1 (taps = Wd [d,7], Wo = Wp [d,d], bo = bp), 3 Light Conv 5x1 (Win = Wi
// [d,d], bin = bi, taps = Wl [H,5], Wo [d,d], bo).  Unused roles have size 0 (offset = next).
// The bf16 shadow holds Win at sh_Win, Wo at sh_Wo, then W1, W2 (sh_total elements).
enum TfOp { TF_ATTN = 0, TF_CONV3 = 1, TF_SEPCONV7 = 2, TF_LIGHTCONV5 = 3 };
struct TfOffsets {
  int op;
  size_t Win, bin, taps, Wo, bo, ln1g, ln1b, W1, b1, W2, b2, ln2g, ln2b, total;
  size_t n_Win, n_bin, n_taps, n_Wo;  // element counts of the mixer matrices / bias / taps
  int taps_k, taps_rows;       // taps: [taps_rows][taps_k]
  int wo_in;                   // Wo's input width (d, or 3d for Conv 3x1)
  size_t sh_Win, sh_Wo, sh_W1, sh_W2, sh_total;
};

// SPOS block geometry (SURVEY §8c "C2 SPOS candidate"; oracle/spos.py block_dims).
struct SposDims {
  int stride, inp, mid, outm, C_in, C_out, H_in, H_out;
};
// One conv -> BN [-> ReLU] unit of a SPOS candidate, in packing order.
struct SposConv {
  int branch;   // 0 = proj (stride-2 blocks), 1 = main
  int dw;       // 1 = depthwise k x k, 0 = pointwise, 2 = dense k x k (Table 5's Conv 3x3; reading A40)
  int cin, cout, k, stride;
  int dil;      // dw: dilation (1, or 2 for Table 5's Dil Conv; reading A36)
  int relu;     // ReLU after the BN
  int H_in, H_out;
  size_t off_w, off_g, off_b;  // offsets in the packed fp32 vector
  size_t off_w16;              // pw / dense: offset of the bf16 GEMM operand in the shadow
  // GEMM K of a pointwise / dense unit (dense: over the k x k x cin columns) and weight count
  int gemm_k() const { return dw == 2 ? k * k * cin : cin; }
  size_t weights() const {
    return dw == 1 ? (size_t)cout * k * k : (dw == 2 ? (size_t)cout * k * k * cin : (size_t)cout * cin);
  }
};

struct Spec {
  naspipe_supernet_spec raw{};  // scalar fields; pointer fields re-pointed into vectors below
  std::vector<int32_t> heads, ffn, op, stage_of_block, cost_fwd, cost_bwd;
  std::vector<int32_t> reps, chans, kern, xcep, dil;  // SPOS
  bool has_partition = false, has_costs = false;

  explicit Spec(const naspipe_supernet_spec* s);
  Spec(const Spec& o);
  void repoint();  // raw's pointer fields -> the owned vectors

  int family() const { return raw.family; }
  int m() const { return raw.n_blocks; }
  int n() const { return raw.n_choices; }
  int B() const { return raw.batch; }
  // SERIAL ("w/o scheduler"): one subnet in flight, W = 1 (reading A32)
  int window(int D) const {
    return raw.sync_policy == NASPIPE_SYNC_SERIAL ? 1 : raw.window > 0 ? raw.window : 4 * D;
  }
  int bulk(int D) const { return raw.bulk_size > 0 ? raw.bulk_size : 4 * D; }
  int lookahead() const { return raw.lookahead > 0 ? raw.lookahead : 2; }
  int64_t residency_horizon() const { return raw.residency_horizon == 0 ? 64 : raw.residency_horizon; }
  // elements of one sample of input / output (the residual stream width per batch row)
  size_t sample_elems() const;
  size_t batch_elems() const { return (size_t)B() * sample_elems(); }
  // Boundary tensors: bytes of the activation entering block b (b == m: the last block's
  // output), of the batch input and of the target.  MLP/TRANSFORMER: fp32 [B, sample];
  // SPOS: bf16x2 NHWC activations (hi + lo planes, A28), fp32 NHWC image, int32
  // labels.
  size_t act_bytes(int b) const;
  size_t grad_bytes(int b) const;  // gradient w.r.t. that activation (SPOS: plain bf16)
  size_t input_bytes() const;
  size_t target_bytes() const;
  // SPOS geometry
  SposDims spos_dims(int b) const;
  std::vector<SposConv> spos_convs(int b, int c) const;
  size_t spos_shadow_elems(int b, int c) const;
  int spos_stem_hw() const { return raw.image_hw / 2; }
  int spos_last_hw() const;
  // frozen SPOS parameters (reading A2): part 0 = stem [C0,3,3,3], 1 = head [Ch, Clast],
  // 2 = fc [classes, Ch]; counter hash with uid m*n + part
  size_t frozen_count(int part) const;
  void init_frozen(int part, float* dst) const;
  int rows() const;  // GEMM rows T: B (MLP) or B*S (transformer)
  int d() const { return family() == NASPIPE_MLP ? raw.width : raw.d_model; }

  std::vector<Segment> segments(int b, int c) const;
  size_t param_count(int b, int c) const;
  TfOffsets tf_offsets(int c) const;
  void init_params(int b, int c, float* dst) const;

  void default_costs(int32_t* cf, int32_t* cb) const;
  // cost tables actually used by the planner (spec's or default), [m*n]
  void costs(std::vector<int32_t>& cf, std::vector<int32_t>& cb) const;
  std::vector<int32_t> partition(int D) const;
  void validate_stages(int D) const;
};

// splitmix64 counter hash (reading A21)
uint64_t splitmix64(uint64_t x);

}  // namespace naspipe
