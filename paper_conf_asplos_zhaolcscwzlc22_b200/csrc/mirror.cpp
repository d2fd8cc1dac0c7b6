// Per-subnet balanced partitions with layer mirroring (PAPER.md P:L166
// "The partition is a D-partition ... of a subnet's sequential list of layers, with each
// partition having roughly the same execution time", "Layer Mirroring ... the new
// parameters are actively pushed to all the other mirrored ones"; reading A31).
// Planning only: the executor runs the fixed supernet partition (reading A12).
//
// Subnet y gets its own balanced contiguous partition of its chosen candidates' costs, so a
// candidate (b, c) may run on different stages for different subnets.  CSP (Def.2)
// then reads: F(y, K) may start at tick t only if, for every block b that y runs on K, the
// previous user x = dep[y][b] of (b, c_y[b]) has finished the backward that WROTE it —
// B(x, stage_x(b)) — by t, plus `mirror_latency` ticks when that stage differs from K (the
// push to the mirror).  Everything else is the O2 event model of planner.cpp: strict
// backward-first, lowest id first, the stage-0 window W, link latency lambda, completions
// and deliveries before decisions.  With every subnet on the supernet partition and
// mirror_latency 0 the plan equals the Planner's.
#include <algorithm>
#include <limits>
#include <set>
#include <vector>

#include "mirror.h"

namespace naspipe {

MirrorPlan plan_mirrored(const Spec& spec, int D, const int32_t* choices, int64_t N, int64_t mirror_latency) {
  NP_REQUIRE(N >= 0 && (N == 0 || choices), NASPIPE_EINVAL, "choices");
  NP_REQUIRE(mirror_latency >= 0, NASPIPE_EINVAL, "mirror_latency %lld", (long long)mirror_latency);
  NP_REQUIRE(spec.raw.sync_policy == NASPIPE_SYNC_CSP && spec.raw.bwd_policy == 0, NASPIPE_EINVAL,
             "mirrored planning supports the CSP policy with strict backward-first only");
  spec.validate_stages(D);
  const int m = spec.m(), n = spec.n(), W = spec.window(D);
  const int64_t lam = spec.raw.link_latency;
  for (int64_t i = 0; i < N * m; ++i)
    NP_REQUIRE(choices[i] >= 0 && choices[i] < n, NASPIPE_EINVAL, "choice %d out of range", choices[i]);
  std::vector<int32_t> cf, cb;
  spec.costs(cf, cb);
  auto C = [&](int64_t y, int b) { return choices[y * m + b]; };

  MirrorPlan P;
  P.sob.assign((size_t)N * m, 0);
  std::vector<int64_t> tf((size_t)N * D, 0), tb((size_t)N * D, 0);  // task costs [y][K]
  for (int64_t y = 0; y < N; ++y) {
    std::vector<int64_t> w(m);
    for (int b = 0; b < m; ++b) w[b] = (int64_t)cf[b * n + C(y, b)] + cb[b * n + C(y, b)];
    const std::vector<int32_t> s = balanced_partition(w, D);
    std::copy(s.begin(), s.end(), P.sob.begin() + y * m);
    for (int b = 0; b < m; ++b) {
      tf[y * D + s[b]] += cf[b * n + C(y, b)];
      tb[y * D + s[b]] += cb[b * n + C(y, b)];
    }
    for (int K = 0; K < D; ++K) {
      tf[y * D + K] = std::max<int64_t>(1, tf[y * D + K]);
      tb[y * D + K] = std::max<int64_t>(1, tb[y * D + K]);
    }
  }
  auto stage_of = [&](int64_t y, int b) { return P.sob[y * m + b]; };
  // dependency table: latest earlier user of the same candidate
  std::vector<int64_t> dep((size_t)N * m, -1), last((size_t)m * n, -1);
  for (int64_t y = 0; y < N; ++y)
    for (int b = 0; b < m; ++b) {
      dep[y * m + b] = last[b * n + C(y, b)];
      last[b * n + C(y, b)] = y;
    }

  const int64_t NONE = std::numeric_limits<int64_t>::max();
  std::vector<int64_t> bend((size_t)N * D, NONE);  // end tick of B(y, K) once started
  std::vector<std::set<int64_t>> inF(D), inB(D);
  std::vector<char> fin0(N, 0), started0(N, 0);
  struct Busy { bool on = false; int64_t end = 0; int kind = 0; int64_t y = 0; };
  struct Delivery { int64_t time; int toB; int K; int64_t y; };
  std::vector<Busy> busy(D);
  std::vector<Delivery> deliv;
  P.stall.assign(D, 0);
  P.bubble.assign(D, 0);
  int64_t t = 0, done0 = 0, wm0 = 0;

  // earliest tick F(y, K)'s writes-before-reads allow; NONE while a WRITE has not started
  auto ready_at = [&](int64_t y, int K) {
    int64_t r = 0;
    for (int b = 0; b < m; ++b) {
      if (stage_of(y, b) != K) continue;
      const int64_t x = dep[y * m + b];
      if (x < 0) continue;
      const int Kx = stage_of(x, b);
      const int64_t e = bend[x * D + Kx];
      if (e == NONE || e > t) return NONE;
      r = std::max(r, e + (Kx != K ? mirror_latency : 0));
    }
    return r;
  };

  while (true) {
    for (int K = 0; K < D; ++K) {
      Busy& bz = busy[K];
      if (!bz.on || bz.end != t) continue;
      bz.on = false;
      if (bz.kind == 0) {
        if (K < D - 1) deliv.push_back({t + lam, 0, K + 1, bz.y});
        else inB[K].insert(bz.y);
      } else if (K > 0) {
        deliv.push_back({t + lam, 1, K - 1, bz.y});
      } else {
        fin0[bz.y] = 1;
        ++done0;
      }
    }
    std::vector<Delivery> keep;
    for (const Delivery& d : deliv) {
      if (d.time <= t) (d.toB ? inB : inF)[d.K].insert(d.y);
      else keep.push_back(d);
    }
    deliv.swap(keep);
    if (done0 == N) break;
    while (wm0 < N && fin0[wm0]) ++wm0;
    for (int64_t y = wm0; y < std::min<int64_t>(N, wm0 + W); ++y)
      if (!started0[y]) inF[0].insert(y);
    std::vector<int64_t> wake;
    for (int K = 0; K < D; ++K) {
      if (busy[K].on) continue;
      int kind = -1;
      int64_t y = -1;
      if (!inB[K].empty()) {
        kind = 1;
        y = *inB[K].begin();
      } else {
        for (int64_t q : inF[K]) {
          const int64_t r = ready_at(q, K);
          if (r == NONE) continue;
          if (r <= t) {
            kind = 0;
            y = q;
            break;
          }
          wake.push_back(r);
        }
      }
      if (kind < 0) continue;
      int64_t cost;
      if (kind == 0) {
        inF[K].erase(y);
        if (K == 0) started0[y] = 1;
        cost = tf[y * D + K];
      } else {
        inB[K].erase(y);
        cost = tb[y * D + K];
        bend[y * D + K] = t + cost;
      }
      busy[K] = {true, t + cost, kind, y};
      P.trace.push_back({t, K, kind, y});
    }
    int64_t nxt = NONE;
    for (const Busy& bz : busy)
      if (bz.on) nxt = std::min(nxt, bz.end);
    for (const Delivery& d : deliv) nxt = std::min(nxt, d.time);
    for (int64_t w : wake)
      if (w > t) nxt = std::min(nxt, w);
    NP_REQUIRE(nxt != NONE, NASPIPE_EINTERNAL, "mirrored plan stalled at tick %lld", (long long)t);
    for (int K = 0; K < D; ++K)
      if (!busy[K].on) (inF[K].empty() ? P.bubble[K] : P.stall[K]) += nxt - t;
    t = nxt;
  }
  P.makespan = t;
  return P;
}

}  // namespace naspipe
