// CSP planner and Belady residency planner (see planner.h).
#include "planner.h"

#include <algorithm>
#include <limits>
#include <map>

namespace naspipe {

Planner::Planner(const Spec& spec, int D)
    : D_(D), m_(spec.m()), n_(spec.n()), W_(spec.window(D)), policy_(spec.raw.bwd_policy),
      lambda_(spec.raw.link_latency), sync_(spec.raw.sync_policy), G_(spec.bulk(D)) {
  sob_ = spec.partition(D);
  blocks_.assign(D, {});
  for (int b = 0; b < m_; ++b) blocks_[sob_[b]].push_back(b);
  spec.costs(cf_tab_, cb_tab_);
  last_user_.assign((size_t)m_ * n_, -1);
  use_count_.assign((size_t)m_ * n_, 0);
  inF_.assign(D, {});
  inB_.assign(D, {});
  fin_.assign(D, {});
  fin_wm_.assign(D, 0);
  busy_.assign(D, {});
  last_kind_.assign(D, -1);
  stage_tasks_.assign(D, {});
  stall_.assign(D, 0);
  bubble_.assign(D, 0);
}

int64_t Planner::add_subnet(const int32_t* choice) {
  NP_REQUIRE(!finalized_, NASPIPE_ESTATE, "stream already finalised (drained)");
  for (int b = 0; b < m_; ++b)
    NP_REQUIRE(choice[b] >= 0 && choice[b] < n_, NASPIPE_EINVAL,
               "choice[%d]=%d outside [0,%d)", b, choice[b], n_);
  const int64_t y = n_subnets();
  for (int b = 0; b < m_; ++b) {
    const size_t key = (size_t)b * n_ + choice[b];
    choices_.push_back(choice[b]);
    dep_.push_back(last_user_[key]);      // dependency table (D8)
    ver_.push_back(use_count_[key]);
    last_user_[key] = y;
    use_count_[key] += 1;
  }
  for (int K = 0; K < D_; ++K) fin_[K].push_back(0);
  return y;
}

void Planner::reopen() {
  NP_REQUIRE(done_, NASPIPE_ESTATE, "reopen before the plan finished");
  finalized_ = false;
  done_ = false;
  phase_ = 0;
}

std::vector<int64_t> Planner::deps(int64_t y, int K) const {
  std::vector<int64_t> out;
  for (int b : blocks_[K]) {
    const int64_t d = dep(y, b);
    if (d >= 0) out.push_back(d);
  }
  std::sort(out.begin(), out.end());
  out.erase(std::unique(out.begin(), out.end()), out.end());
  return out;
}

int64_t Planner::cost(int K, int64_t y, int kind) const {
  int64_t s = 0;
  const auto& tab = kind == 0 ? cf_tab_ : cb_tab_;
  for (int b : blocks_[K]) s += tab[(size_t)b * n_ + choice(y, b)];
  return std::max<int64_t>(1, s);
}

bool Planner::admissible(int K, int64_t y) const {
  if (sync_ == NASPIPE_SYNC_ASP || sync_ == NASPIPE_SYNC_BSP) return true;  // dependencies ignored
  for (int b : blocks_[K]) {
    const int64_t d = dep(y, b);
    if (d >= 0 && !fin_[K][d]) return false;
  }
  return true;
}

void Planner::start(int K, int kind, int64_t y) {
  busy_[K] = {true, t_ + cost(K, y, kind), kind, y};
  last_kind_[K] = kind;
  stage_tasks_[K].push_back((int64_t)tasks_.size());
  tasks_.push_back({t_, K, kind, y});
}

void Planner::advance() {
  while (!done_) {
    if (phase_ == 0) {
      // (1) completions at t, then deliveries with time <= t
      for (int K = 0; K < D_; ++K) {
        Busy& bz = busy_[K];
        if (!bz.on || bz.end != t_) continue;
        bz.on = false;
        if (bz.kind == 0) {
          if (K < D_ - 1) deliveries_.push_back({t_ + lambda_, 0, K + 1, bz.y});
          else inB_[K].insert(bz.y);
        } else {
          fin_[K][bz.y] = 1;
          while (fin_wm_[K] < (int64_t)fin_[K].size() && fin_[K][fin_wm_[K]]) ++fin_wm_[K];
          if (K > 0) deliveries_.push_back({t_ + lambda_, 1, K - 1, bz.y});
          else ++done0_;
        }
      }
      std::vector<Delivery> keep;
      for (auto& dv : deliveries_) {
        if (dv.time <= t_) (dv.to_B ? inB_ : inF_)[dv.K].insert(dv.y);
        else keep.push_back(dv);
      }
      deliveries_.swap(keep);
      phase_ = 1;
    }
    // the stream may have been finalised while suspended at this tick
    if (finalized_ && done0_ == n_subnets()) {
      done_ = true;
      makespan_ = t_;
      return;
    }
    // (2) stage-0 source under the window: y < wm0 + W (reading A7); BSP: the current bulk,
    // which opens once every subnet of the previous bulk finished on stage 0 (the flush)
    const int64_t N = n_subnets();
    const int64_t wm0 = fin_wm_[0];
    const int64_t hi = sync_ == NASPIPE_SYNC_BSP ? (wm0 / G_ + 1) * G_ : wm0 + W_;
    if (!finalized_ && N < hi) return;  // streaming rule: wait for more subnets
    const int64_t lim = std::min(hi, N);
    for (; src_next_ < lim; ++src_next_) inF_[0].insert(src_next_);
    // (3) decisions on idle stages
    for (int K = 0; K < D_; ++K) {
      if (busy_[K].on) continue;
      int64_t first = -1;
      if (sync_ == NASPIPE_SYNC_INORDER) {             // w/o scheduler: only the head may go
        if (!inF_[K].empty() && admissible(K, *inF_[K].begin())) first = *inF_[K].begin();
      } else {
        for (int64_t y : inF_[K])
          if (admissible(K, y)) { first = y; break; }  // ascending id (reading A6)
      }
      if (sync_ == NASPIPE_SYNC_BSP && first >= 0) {  // GPipe: a bulk's forwards before its backwards
        inF_[K].erase(first);
        start(K, 0, first);
      } else if (policy_ == 1 && last_kind_[K] == 1 && first >= 0) {
        inF_[K].erase(first);
        start(K, 0, first);
      } else if (!inB_[K].empty()) {                  // backward first, lowest id (A5)
        const int64_t y = *inB_[K].begin();
        inB_[K].erase(inB_[K].begin());
        start(K, 1, y);
      } else if (first >= 0) {
        inF_[K].erase(first);
        start(K, 0, first);
      }
    }
    // (4) advance time
    int64_t nxt = std::numeric_limits<int64_t>::max();
    for (auto& bz : busy_) if (bz.on) nxt = std::min(nxt, bz.end);
    for (auto& dv : deliveries_) nxt = std::min(nxt, dv.time);
    NP_REQUIRE(nxt != std::numeric_limits<int64_t>::max(), NASPIPE_EINTERNAL,
               "CSP planner stalled at tick %lld", (long long)t_);
    for (int K = 0; K < D_; ++K)
      if (!busy_[K].on) (inF_[K].empty() ? bubble_ : stall_)[K] += nxt - t_;
    t_ = nxt;
    phase_ = 0;
  }
}

bool BeladyResidency::can_decide() const {
  if (next_ >= known()) return false;
  if (final_) return true;
  if (H_ <= 0) return false;
  return known() >= next_ + std::max<int64_t>(L_, H_);
}

int64_t BeladyResidency::next_use(int64_t u, int64_t i) const {
  const int64_t end = H_ > 0 ? std::min(known(), i + H_) : known();
  for (int64_t j = i; j < end; ++j)
    if (std::binary_search(uses_[j].begin(), uses_[j].end(), u)) return j;
  return std::numeric_limits<int64_t>::max();
}

int64_t BeladyResidency::size_of(const std::set<int64_t>& s) const {
  int64_t t = 0;
  for (int64_t u : s) t += bytes_[u];
  return t;
}

void BeladyResidency::decide_next(std::vector<ResidencyEvent>& events,
                                  std::vector<std::pair<int64_t, int64_t>>& writebacks) {
  const int64_t i = next_;
  const int64_t T = known();
  std::set<int64_t> need(uses_[i].begin(), uses_[i].end());
  NP_REQUIRE(size_of(need) <= budget_, NASPIPE_EBUDGET, "stage %d task %lld needs %lld bytes > budget %lld", K_,
             (long long)i, (long long)size_of(need), (long long)budget_);
  for (int depth = 2; depth <= L_; ++depth) {  // prefetch depth L' <= L that fits the budget
    if (i + depth - 1 >= T) break;
    std::set<int64_t> cand = need;
    cand.insert(uses_[i + depth - 1].begin(), uses_[i + depth - 1].end());
    if (size_of(cand) > budget_) break;
    need.swap(cand);
  }
  for (;;) {
    std::set<int64_t> uni = resident_;
    uni.insert(need.begin(), need.end());
    if (size_of(uni) <= budget_) break;
    int64_t victim = -1, far = -1;
    for (int64_t u : resident_) {  // ascending uid: ties keep the lowest
      if (need.count(u)) continue;
      const int64_t nu = next_use(u, i);
      if (nu > far) { far = nu; victim = u; }
    }
    resident_.erase(victim);
    events.push_back({K_, i, 1, victim});
    if (dirty_.count(victim)) {
      writebacks.push_back({i, victim});
      dirty_.erase(victim);
    }
  }
  std::vector<std::pair<int64_t, int64_t>> loads;
  for (int64_t u : need)
    if (!resident_.count(u)) loads.push_back({next_use(u, i), u});
  std::sort(loads.begin(), loads.end());
  for (auto& lu : loads) {
    resident_.insert(lu.second);
    events.push_back({K_, i, 0, lu.second});
  }
  if (kinds_[i] == 1) dirty_.insert(uses_[i].begin(), uses_[i].end());
  ++next_;
}

ResidencyPlan plan_residency(int K, const std::vector<std::vector<int64_t>>& uses,
                             const std::vector<int>& kinds, const std::vector<int64_t>& bytes,
                             int64_t budget, int L, int64_t horizon) {
  ResidencyPlan out;
  BeladyResidency r(K, bytes, budget, L, horizon);
  for (size_t i = 0; i < uses.size(); ++i) r.push_task(uses[i], kinds[i]);
  r.set_final();
  while (r.can_decide()) r.decide_next(out.events, out.writebacks);
  return out;
}

}  // namespace naspipe
