// Spec validation, layouts, analytic costs, balanced partition (reading A12) and the
// counter-hash initialiser (reading A21).
#include "spec.h"

#include <algorithm>
#include <cmath>
#include <cstring>
#include <limits>

namespace naspipe {

std::string strfmt(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  return buf;
}

uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

Spec::Spec(const naspipe_supernet_spec* s) {
  NP_REQUIRE(s != nullptr, NASPIPE_EINVAL, "spec is NULL");
  NP_REQUIRE(s->abi_version == NASPIPE_ABI_VERSION, NASPIPE_EINVAL, "abi_version %d != %d",
             s->abi_version, NASPIPE_ABI_VERSION);
  raw = *s;
  NP_REQUIRE(raw.family == NASPIPE_MLP || raw.family == NASPIPE_TRANSFORMER || raw.family == NASPIPE_SPOS_CNN,
             NASPIPE_EINVAL, "unsupported family %d", raw.family);
  NP_REQUIRE(raw.n_blocks >= 1 && raw.n_blocks <= 4096, NASPIPE_EINVAL, "n_blocks %d", raw.n_blocks);
  NP_REQUIRE(raw.n_choices >= 1 && raw.n_choices <= 4096, NASPIPE_EINVAL, "n_choices %d",
             raw.n_choices);
  NP_REQUIRE(raw.batch >= 1, NASPIPE_EINVAL, "batch %d", raw.batch);
  NP_REQUIRE(std::isfinite(raw.lr), NASPIPE_EINVAL, "lr not finite");
  NP_REQUIRE(raw.window >= 0 && raw.lookahead >= 0 && raw.bwd_policy >= 0 && raw.bwd_policy <= 1 &&
                 raw.link_latency >= 0 && raw.hbm_weight_budget_bytes >= 0,
             NASPIPE_EINVAL, "bad window/lookahead/policy/latency/budget");
  NP_REQUIRE(raw.sync_policy >= NASPIPE_SYNC_CSP && raw.sync_policy <= NASPIPE_SYNC_SERIAL && raw.bulk_size >= 0,
             NASPIPE_EINVAL, "bad sync_policy %d / bulk_size %d", raw.sync_policy, raw.bulk_size);
  NP_REQUIRE(!(raw.flags & NASPIPE_FLAG_RECOMPUTE) ||
                 (raw.family == NASPIPE_TRANSFORMER && raw.sync_policy != NASPIPE_SYNC_ASP),
             NASPIPE_EINVAL, "activation recomputation: transformer family, not under ASP (reading A13)");
  const int n = raw.n_choices, m = raw.n_blocks;
  if (raw.family == NASPIPE_MLP) {
    NP_REQUIRE(raw.width >= 1 && raw.width <= 1024, NASPIPE_EINVAL, "width %d", raw.width);
    NP_REQUIRE(raw.compute_dtype == NASPIPE_FP32, NASPIPE_EINVAL, "MLP computes in fp32");
  } else if (raw.family == NASPIPE_TRANSFORMER) {
    NP_REQUIRE(raw.compute_dtype == NASPIPE_BF16, NASPIPE_EINVAL, "transformer computes in bf16");
    NP_REQUIRE(raw.d_model >= 16 && raw.d_model % 16 == 0, NASPIPE_EINVAL,
               "d_model %d must be a positive multiple of 16", raw.d_model);
    NP_REQUIRE(raw.seq_len >= 1 && raw.seq_len <= 128, NASPIPE_EINVAL, "seq_len %d (1..128)",
               raw.seq_len);
    NP_REQUIRE(raw.choice_heads && raw.choice_ffn, NASPIPE_EINVAL, "choice_heads/choice_ffn NULL");
    heads.assign(raw.choice_heads, raw.choice_heads + n);
    ffn.assign(raw.choice_ffn, raw.choice_ffn + n);
    if (raw.choice_op) op.assign(raw.choice_op, raw.choice_op + n);
    else op.assign(n, TF_ATTN);
    for (int c = 0; c < n; ++c) {
      NP_REQUIRE(op[c] >= TF_ATTN && op[c] <= TF_LIGHTCONV5, NASPIPE_EINVAL, "choice_op[%d]=%d (0..3)", c, op[c]);
      NP_REQUIRE(heads[c] >= 1 && raw.d_model % heads[c] == 0, NASPIPE_EINVAL,
                 "heads[%d]=%d must divide d_model", c, heads[c]);
      const int hd = raw.d_model / heads[c];
      NP_REQUIRE(op[c] != TF_ATTN || (hd % 16 == 0 && hd <= 128), NASPIPE_EINVAL,
                 "head dim %d must be 16..128, %%16", hd);
      NP_REQUIRE(ffn[c] >= 16 && ffn[c] % 16 == 0, NASPIPE_EINVAL, "ffn[%d]=%d must be a multiple of 16",
                 c, ffn[c]);
    }
  } else {
    NP_REQUIRE(raw.compute_dtype == NASPIPE_BF16, NASPIPE_EINVAL, "SPOS CNN computes in bf16");
    NP_REQUIRE(raw.n_cnn_stages >= 1 && raw.n_cnn_stages <= 8 && raw.stage_repeats && raw.stage_channels &&
                   raw.choice_kernel && raw.choice_xception,
               NASPIPE_EINVAL, "SPOS: n_cnn_stages / stage_repeats / stage_channels / choice_* missing");
    reps.assign(raw.stage_repeats, raw.stage_repeats + raw.n_cnn_stages);
    chans.assign(raw.stage_channels, raw.stage_channels + raw.n_cnn_stages);
    kern.assign(raw.choice_kernel, raw.choice_kernel + n);
    xcep.assign(raw.choice_xception, raw.choice_xception + n);
    if (raw.choice_dilation) dil.assign(raw.choice_dilation, raw.choice_dilation + n);
    else dil.assign(n, 1);
    int total = 0, prev = raw.stem_channels;
    NP_REQUIRE(raw.stem_channels >= 16 && raw.stem_channels % 16 == 0, NASPIPE_EINVAL, "stem_channels %d (%%16)",
               raw.stem_channels);
    for (int i = 0; i < raw.n_cnn_stages; ++i) {
      NP_REQUIRE(reps[i] >= 1, NASPIPE_EINVAL, "stage_repeats[%d]=%d", i, reps[i]);
      NP_REQUIRE(chans[i] % 32 == 0 && chans[i] > prev && (chans[i] - prev) % 16 == 0, NASPIPE_EINVAL,
                 "stage_channels[%d]=%d must be %%32, > previous (%d), difference %%16", i, chans[i], prev);
      total += reps[i];
      prev = chans[i];
    }
    NP_REQUIRE(total == m, NASPIPE_EINVAL, "sum(stage_repeats)=%d != n_blocks=%d", total, m);
    NP_REQUIRE(raw.image_hw >= 32 && raw.image_hw % (2 << raw.n_cnn_stages) == 0, NASPIPE_EINVAL,
               "image_hw %d must be a multiple of 2^(1+n_cnn_stages)", raw.image_hw);
    NP_REQUIRE(raw.num_classes >= 2 && raw.head_channels >= 16 && raw.head_channels % 16 == 0, NASPIPE_EINVAL,
               "num_classes %d / head_channels %d (%%16)", raw.num_classes, raw.head_channels);
    for (int c = 0; c < n; ++c)
      NP_REQUIRE((kern[c] == 3 || kern[c] == 5 || kern[c] == 7) && (xcep[c] >= 0 && xcep[c] <= 2) &&
                     (dil[c] == 1 || dil[c] == 2) && (xcep[c] != 2 || (kern[c] == 3 && dil[c] == 1)),
                 NASPIPE_EINVAL,
                 "choice %d: kernel %d xception %d dilation %d (k in {3,5,7}, dilation 1 or 2; the dense "
                 "Conv 3x3 (xception 2) takes k 3, dilation 1)",
                 c, kern[c], xcep[c], dil[c]);
  }
  if (raw.stage_of_block) {
    stage_of_block.assign(raw.stage_of_block, raw.stage_of_block + m);
    has_partition = true;
  }
  NP_REQUIRE((raw.cost_fwd == nullptr) == (raw.cost_bwd == nullptr), NASPIPE_EINVAL,
             "cost_fwd and cost_bwd must both be given or both NULL");
  if (raw.cost_fwd) {
    cost_fwd.assign(raw.cost_fwd, raw.cost_fwd + (size_t)m * n);
    cost_bwd.assign(raw.cost_bwd, raw.cost_bwd + (size_t)m * n);
    for (size_t i = 0; i < cost_fwd.size(); ++i)
      NP_REQUIRE(cost_fwd[i] >= 0 && cost_bwd[i] >= 0, NASPIPE_EINVAL, "negative cost");
    has_costs = true;
  }
  repoint();
}

Spec::Spec(const Spec& o)
    : raw(o.raw), heads(o.heads), ffn(o.ffn), op(o.op), stage_of_block(o.stage_of_block),
      cost_fwd(o.cost_fwd), cost_bwd(o.cost_bwd), reps(o.reps), chans(o.chans), kern(o.kern),
      xcep(o.xcep), dil(o.dil), has_partition(o.has_partition), has_costs(o.has_costs) {
  repoint();
}

void Spec::repoint() {
  raw.choice_heads = heads.empty() ? nullptr : heads.data();
  raw.choice_ffn = ffn.empty() ? nullptr : ffn.data();
  raw.choice_op = op.empty() ? nullptr : op.data();
  raw.stage_of_block = has_partition ? stage_of_block.data() : nullptr;
  raw.cost_fwd = has_costs ? cost_fwd.data() : nullptr;
  raw.cost_bwd = has_costs ? cost_bwd.data() : nullptr;
  raw.stage_repeats = reps.empty() ? nullptr : reps.data();
  raw.stage_channels = chans.empty() ? nullptr : chans.data();
  raw.choice_kernel = kern.empty() ? nullptr : kern.data();
  raw.choice_xception = xcep.empty() ? nullptr : xcep.data();
  raw.choice_dilation = dil.empty() ? nullptr : dil.data();
}

size_t Spec::sample_elems() const {
  if (family() == NASPIPE_SPOS_CNN) return (size_t)raw.image_hw * raw.image_hw * 3;
  return family() == NASPIPE_MLP ? (size_t)raw.width : (size_t)raw.seq_len * raw.d_model;
}

size_t Spec::input_bytes() const { return 4 * batch_elems(); }
size_t Spec::target_bytes() const {
  return family() == NASPIPE_SPOS_CNN ? 4 * (size_t)B() : 4 * batch_elems();
}
size_t Spec::grad_bytes(int b) const {
  if (family() != NASPIPE_SPOS_CNN) return 4 * batch_elems();
  if (b < m()) {
    const SposDims d = spos_dims(b);
    return 2 * (size_t)B() * d.H_in * d.H_in * d.C_in;
  }
  const int hw = spos_last_hw();
  return 2 * (size_t)B() * hw * hw * chans.back();
}
size_t Spec::act_bytes(int b) const {
  return family() == NASPIPE_SPOS_CNN ? 2 * grad_bytes(b) : grad_bytes(b);
}

// oracle/spos.py block_dims: the stem halves image_hw; the first block of every CNN stage
// has stride 2 (inp = C_prev, mid = C/2, out = C - C_prev), the others stride 1 with the
// channel split (inp = mid = out = C/2).
SposDims Spec::spos_dims(int b) const {
  NP_REQUIRE(family() == NASPIPE_SPOS_CNN && b >= 0 && b < m(), NASPIPE_EINVAL, "spos_dims(%d)", b);
  int c_prev = raw.stem_channels, H = raw.image_hw / 2, k = 0;
  for (size_t st = 0; st < reps.size(); ++st) {
    const int co = chans[st];
    for (int i = 0; i < reps[st]; ++i, ++k) {
      if (k == b) {
        if (i == 0) return {2, c_prev, co / 2, co - c_prev, c_prev, co, H, H / 2};
        return {1, co / 2, co / 2, co / 2, co, co, H, H};
      }
      if (i == 0) H /= 2;
    }
    c_prev = co;
  }
  return {};
}

int Spec::spos_last_hw() const { return raw.image_hw >> (1 + (int)reps.size()); }

std::vector<SposConv> Spec::spos_convs(int b, int c) const {
  const SposDims d = spos_dims(b);
  const int k = kern[c], dl = dil[c];
  std::vector<SposConv> L;
  // (branch, dw, cin, cout, k, stride, relu, H_in, H_out)
  auto add = [&](int br, int dw, int ci, int co, int kk, int s, int relu, int hin) {
    SposConv u{};
    u.branch = br; u.dw = dw; u.cin = ci; u.cout = co; u.k = kk; u.stride = s; u.relu = relu;
    u.dil = dw == 1 ? dl : 1;
    u.H_in = hin; u.H_out = hin / s;
    L.push_back(u);
  };
  const int H = d.H_in, s = d.stride, Ho = d.H_out;
  if (s == 2) {
    add(0, 1, d.inp, d.inp, k, 2, 0, H);
    add(0, 0, d.inp, d.inp, 1, 1, 1, Ho);
  }
  if (xcep[c] == 2) {  // dense Conv 3x3 in place of the depthwise conv (reading A40)
    add(1, 0, d.inp, d.mid, 1, 1, 1, H);
    add(1, 2, d.mid, d.mid, k, s, 0, H);
    add(1, 0, d.mid, d.outm, 1, 1, 1, Ho);
  } else if (!xcep[c]) {
    add(1, 0, d.inp, d.mid, 1, 1, 1, H);
    add(1, 1, d.mid, d.mid, k, s, 0, H);
    add(1, 0, d.mid, d.outm, 1, 1, 1, Ho);
  } else {
    add(1, 1, d.inp, d.inp, k, s, 0, H);
    add(1, 0, d.inp, d.mid, 1, 1, 1, Ho);
    add(1, 1, d.mid, d.mid, k, 1, 0, Ho);
    add(1, 0, d.mid, d.mid, 1, 1, 1, Ho);
    add(1, 1, d.mid, d.mid, k, 1, 0, Ho);
    add(1, 0, d.mid, d.outm, 1, 1, 1, Ho);
  }
  size_t off = 0, off16 = 0;
  for (auto& u : L) {
    u.off_w = off;
    const size_t nw = u.weights();
    off += nw;
    u.off_g = off;
    off += u.cout;
    u.off_b = off;
    off += u.cout;
    u.off_w16 = off16;
    if (u.dw != 1) off16 += nw;
  }
  return L;
}

// bf16x2 shadow: hi planes of every 1x1 weight, then the lo planes (same offsets + half)
size_t Spec::spos_shadow_elems(int b, int c) const {
  size_t t = 0;
  for (auto& u : spos_convs(b, c))
    if (u.dw != 1) t += u.weights();
  return 2 * t;
}

size_t Spec::frozen_count(int part) const {
  if (part == 0) return (size_t)raw.stem_channels * 27;
  if (part == 1) return (size_t)raw.head_channels * chans.back();
  return (size_t)raw.num_classes * raw.head_channels;
}

void Spec::init_frozen(int part, float* dst) const {
  const int fan = part == 0 ? 27 : part == 1 ? chans.back() : raw.head_channels;
  const uint64_t uid = (uint64_t)m() * (uint64_t)n() + (uint64_t)part;
  const float bound = 1.0f / std::sqrt((float)fan);
  const size_t cnt = frozen_count(part);
  for (size_t i = 0; i < cnt; ++i) {
    const uint64_t z = splitmix64(raw.init_seed ^ (uid * 0x9E3779B97F4A7C15ull + i));
    dst[i] = bound * (2.0f * ((float)(z >> 40) * 5.9604644775390625e-08f) - 1.0f);
  }
}

int Spec::rows() const { return family() == NASPIPE_MLP ? raw.batch : raw.batch * raw.seq_len; }

TfOffsets Spec::tf_offsets(int c) const {
  const size_t d = raw.d_model, f = ffn[c], H = heads[c];
  TfOffsets o{};
  o.op = op[c];
  size_t off = 0;
  auto take = [&](size_t n) { size_t r = off; off += n; return r; };
  switch (o.op) {  // packing order of oracle/transformer.py mixer_layout
    case TF_ATTN:
      o.n_Win = 3 * d * d; o.Win = take(o.n_Win); o.n_bin = 3 * d; o.bin = take(o.n_bin);
      o.taps = off;
      o.n_Wo = d * d; o.wo_in = (int)d; o.Wo = take(o.n_Wo); o.bo = take(d);
      break;
    case TF_CONV3:
      o.Win = o.bin = o.taps = off;
      o.n_Wo = 3 * d * d; o.wo_in = 3 * (int)d; o.Wo = take(o.n_Wo); o.bo = take(d);
      break;
    case TF_SEPCONV7:
      o.Win = o.bin = off;
      o.taps_rows = (int)d; o.taps_k = 7; o.n_taps = 7 * d; o.taps = take(o.n_taps);
      o.n_Wo = d * d; o.wo_in = (int)d; o.Wo = take(o.n_Wo); o.bo = take(d);
      break;
    default:  // TF_LIGHTCONV5
      o.n_Win = d * d; o.Win = take(o.n_Win); o.n_bin = d; o.bin = take(o.n_bin);
      o.taps_rows = (int)H; o.taps_k = 5; o.n_taps = 5 * H; o.taps = take(o.n_taps);
      o.n_Wo = d * d; o.wo_in = (int)d; o.Wo = take(o.n_Wo); o.bo = take(d);
      break;
  }
  o.ln1g = take(d); o.ln1b = take(d);
  o.W1 = take(f * d); o.b1 = take(f);
  o.W2 = take(d * f); o.b2 = take(d);
  o.ln2g = take(d); o.ln2b = take(d);
  o.total = off;
  o.sh_Win = 0;
  o.sh_Wo = o.n_Win;
  o.sh_W1 = o.sh_Wo + o.n_Wo;
  o.sh_W2 = o.sh_W1 + f * d;
  o.sh_total = o.sh_W2 + d * f;
  return o;
}

std::vector<Segment> Spec::segments(int b, int c) const {
  std::vector<Segment> s;
  if (family() == NASPIPE_SPOS_CNN) {
    for (auto& u : spos_convs(b, c)) {
      s.push_back({u.off_w, u.off_g - u.off_w, 0, u.dw == 1 ? u.k * u.k : u.gemm_k()});
      s.push_back({u.off_g, (size_t)u.cout, 1, 0});
      s.push_back({u.off_b, (size_t)u.cout, 2, 0});
    }
    return s;
  }
  if (family() == NASPIPE_MLP) {
    const size_t d = raw.width;
    s.push_back({0, d * d, 0, (int)d});
    s.push_back({d * d, d, 0, (int)d});
    return s;
  }
  const TfOffsets o = tf_offsets(c);
  const size_t d = raw.d_model, f = ffn[c];
  if (o.n_Win) {
    s.push_back({o.Win, o.n_Win, 0, (int)d});
    s.push_back({o.bin, o.n_bin, 0, (int)d});
  }
  if (o.n_taps) s.push_back({o.taps, o.n_taps, 0, o.taps_k});
  s.push_back({o.Wo, o.n_Wo, 0, o.wo_in});
  s.push_back({o.bo, d, 0, o.wo_in});
  s.push_back({o.ln1g, d, 1, 0});
  s.push_back({o.ln1b, d, 2, 0});
  s.push_back({o.W1, f * d, 0, (int)d});
  s.push_back({o.b1, f, 0, (int)d});
  s.push_back({o.W2, d * f, 0, (int)f});
  s.push_back({o.b2, d, 0, (int)f});
  s.push_back({o.ln2g, d, 1, 0});
  s.push_back({o.ln2b, d, 2, 0});
  return s;
}

size_t Spec::param_count(int b, int c) const {
  size_t t = 0;
  for (auto& s : segments(b, c)) t += s.size;
  return t;
}

void Spec::init_params(int b, int c, float* dst) const {
  const uint64_t uid = (uint64_t)b * (uint64_t)n() + (uint64_t)c;
  for (auto& s : segments(b, c)) {
    if (s.kind == 1) { std::fill(dst + s.offset, dst + s.offset + s.size, 1.0f); continue; }
    if (s.kind == 2) { std::fill(dst + s.offset, dst + s.offset + s.size, 0.0f); continue; }
    const float bound = 1.0f / std::sqrt((float)s.fan_in);
    for (size_t k = 0; k < s.size; ++k) {
      const uint64_t i = s.offset + k;
      const uint64_t z = splitmix64(raw.init_seed ^ (uid * 0x9E3779B97F4A7C15ull + i));
      const float u = (float)(z >> 40) * 5.9604644775390625e-08f;  // 2^-24
      const float two_u_m1 = 2.0f * u - 1.0f;                       // exact
      dst[s.offset + k] = bound * two_u_m1;
    }
  }
}

// Analytic per-(block, choice) tick table (1 tick = 1 us), SURVEY §8c "Cost tables":
// cf = ceil(max(flops / (0.6 * 1378e12), bytes / (0.8 * 6544e9))), cb = ceil(2 * tf + update).
void Spec::default_costs(int32_t* cf, int32_t* cb) const {
  const double peak = 0.6 * 1378e12, bw = 0.8 * 6544e9;
  for (int b = 0; b < m(); ++b)
    for (int c = 0; c < n(); ++c) {
      double flops, bytes;
      const double P = (double)param_count(b, c);
      if (family() == NASPIPE_MLP) {
        const double d = raw.width, T = raw.batch;
        flops = 2.0 * T * d * d;
        bytes = 4.0 * (3.0 * T * d + d * d + d);
      } else if (family() == NASPIPE_SPOS_CNN) {
        // per conv -> BN unit: conv reads x, writes z; BN stats read z; apply reads z, writes y
        flops = bytes = 0;
        for (auto& u : spos_convs(b, c)) {
          const double Pin = (double)B() * u.H_in * u.H_in, Pout = (double)B() * u.H_out * u.H_out;
          flops += u.dw == 1 ? 2.0 * Pout * u.cout * u.k * u.k : 2.0 * Pout * u.gemm_k() * u.cout;
          bytes += 2.0 * (Pin * u.cin + 4.0 * Pout * u.cout);
        }
      } else {
        const double d = raw.d_model, f = ffn[c], T = (double)raw.batch * raw.seq_len,
                     S = raw.seq_len;
        const int opc = op[c];
        const double mix = opc == TF_ATTN ? 4.0 * d * d : opc == TF_CONV3 ? 3.0 * d * d
                         : opc == TF_SEPCONV7 ? d * d + 7.0 * d : 2.0 * d * d + 5.0 * d;
        flops = 2.0 * T * (mix + 2.0 * d * f) + (opc == TF_ATTN ? 4.0 * T * S * d : 0.0);
        bytes = 2.0 * T * (12.0 * d + 3.0 * f) + 2.0 * P;
      }
      const double tf = std::max(flops / peak, bytes / bw) * 1e6;
      const double tb = 2.0 * tf + 10.0 * P / bw * 1e6;
      cf[b * n() + c] = (int32_t)std::max(1.0, std::ceil(tf));
      cb[b * n() + c] = (int32_t)std::max(1.0, std::ceil(tb));
    }
}

void Spec::costs(std::vector<int32_t>& cf, std::vector<int32_t>& cb) const {
  if (has_costs) { cf = cost_fwd; cb = cost_bwd; return; }
  cf.assign((size_t)m() * n(), 0);
  cb.assign((size_t)m() * n(), 0);
  default_costs(cf.data(), cb.data());
}

void Spec::validate_stages(int D) const {
  NP_REQUIRE(D >= 1 && D <= m(), NASPIPE_EINVAL, "n_stages %d not in 1..n_blocks=%d", D, m());
  if (!has_partition) return;
  NP_REQUIRE(stage_of_block[0] == 0 && stage_of_block[m() - 1] == D - 1, NASPIPE_EINVAL,
             "stage_of_block must start at 0 and end at n_stages-1");
  for (int b = 1; b < m(); ++b)
    NP_REQUIRE(stage_of_block[b] == stage_of_block[b - 1] || stage_of_block[b] == stage_of_block[b - 1] + 1,
               NASPIPE_EINVAL, "stage_of_block must be contiguous and non-decreasing");
}

// Balanced contiguous partition of per-block weights w into D non-empty stages: minimise the
// max stage weight; ties -> lexicographically smallest split points (reading A12).  Exact
// integer DP.
std::vector<int32_t> balanced_partition(const std::vector<int64_t>& w, int D) {
  const int M = (int)w.size();
  NP_REQUIRE(D >= 1 && D <= M, NASPIPE_EINVAL, "partition of %d blocks into %d stages", M, D);
  std::vector<int64_t> pre(M + 1, 0);
  for (int b = 0; b < M; ++b) pre[b + 1] = pre[b] + w[b];
  auto seg = [&](int i, int e) { return pre[e] - pre[i]; };
  const int64_t INF = std::numeric_limits<int64_t>::max();
  // g[k][i]: min over splits of blocks [i, M) into k non-empty stages of the max weight
  std::vector<std::vector<int64_t>> g(D + 1, std::vector<int64_t>(M + 1, INF));
  for (int i = 0; i < M; ++i) g[1][i] = seg(i, M);
  for (int k = 2; k <= D; ++k)
    for (int i = 0; i + k <= M; ++i)
      for (int e = i + 1; e + (k - 1) <= M; ++e)
        g[k][i] = std::min(g[k][i], std::max(seg(i, e), g[k - 1][e]));
  const int64_t best = g[D][0];
  std::vector<int32_t> sob(M, 0);
  int start = 0;
  for (int k = 0; k < D - 1; ++k) {
    const int r = D - k;  // stages left including this one
    int e = start + 1;
    for (; e + (r - 1) <= M; ++e)
      if (seg(start, e) <= best && g[r - 1][e] <= best) break;
    for (int b = start; b < e; ++b) sob[b] = k;
    start = e;
  }
  for (int b = start; b < M; ++b) sob[b] = D - 1;
  return sob;
}

// The supernet partition: the spec's, else balanced over weight(b) = sum_c (cf + cb).
std::vector<int32_t> Spec::partition(int D) const {
  validate_stages(D);
  if (has_partition) return stage_of_block;
  std::vector<int32_t> cf, cb;
  costs(cf, cb);
  std::vector<int64_t> w(m(), 0);
  for (int b = 0; b < m(); ++b)
    for (int c = 0; c < n(); ++c) w[b] += (int64_t)cf[b * n() + c] + cb[b * n() + c];
  return balanced_partition(w, D);
}

}  // namespace naspipe
