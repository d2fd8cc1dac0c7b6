// Deterministic CSP planner: dependency table over (block, choice) keyed by chronological
// subnet order, and a logical-time discrete-event schedule of Alg.1 + Alg.2 (PAPER.md
// P:L170-221) under readings A5-A8.  Streaming: subnets are appended one at a
// time; a stage-0 decision at tick t is taken only once every y < wm0 + W has been
// submitted or the stream has been finalised, so the plan never depends on submit pace.
#pragma once
#include <cstdint>
#include <deque>
#include <set>
#include <vector>

#include "spec.h"

namespace naspipe {

struct Task {
  int64_t t;    // start tick
  int32_t K;    // stage
  int32_t kind; // 0 = F, 1 = B
  int64_t y;    // subnet sequence id
};

class Planner {
 public:
  Planner(const Spec& spec, int D);

  int D() const { return D_; }
  const std::vector<int32_t>& stage_of_block() const { return sob_; }
  const std::vector<int>& blocks_of(int K) const { return blocks_[K]; }

  // Append subnet (choice vector of length m).  Returns its id.
  int64_t add_subnet(const int32_t* choice);
  // Fix N = number of added subnets.
  void finalize() { finalized_ = true; }
  // After done(): accept more subnets; the continuation starts at the previous makespan with
  // every earlier subnet finished (a drain is a pipeline flush).
  void reopen();
  // Advance the simulation as far as allowed; newly planned tasks are appended to tasks().
  void advance();
  bool done() const { return done_; }
  int64_t makespan() const { return makespan_; }
  int64_t n_subnets() const { return (int64_t)choices_.size() / m_; }

  const std::vector<Task>& tasks() const { return tasks_; }
  // per-stage planned order: indices into tasks()
  const std::vector<std::vector<int64_t>>& stage_tasks() const { return stage_tasks_; }

  int32_t choice(int64_t y, int b) const { return choices_[(size_t)y * m_ + b]; }
  const int32_t* choice_row(int64_t y) const { return choices_.data() + (size_t)y * m_; }
  // dependency table: dep[y][b] = latest x < y with c_x[b] == c_y[b], else -1
  int64_t dep(int64_t y, int b) const { return dep_[(size_t)y * m_ + b]; }
  // version of candidate (b, c_y[b]) seen by subnet y = #{x < y : c_x[b] == c_y[b]}
  int64_t version(int64_t y, int b) const { return ver_[(size_t)y * m_ + b]; }
  std::vector<int64_t> deps(int64_t y, int K) const;
  int64_t cost(int K, int64_t y, int kind) const;
  // idle ticks per stage: stalled (a queued forward is blocked by a dependency) / bubble
  // (nothing queued) — SURVEY §8d C5
  const std::vector<int64_t>& stall_ticks() const { return stall_; }
  const std::vector<int64_t>& bubble_ticks() const { return bubble_; }

 private:
  bool admissible(int K, int64_t y) const;
  void start(int K, int kind, int64_t y);

  int D_, m_, n_, W_, policy_, lambda_, sync_, G_;
  std::vector<int32_t> sob_;
  std::vector<std::vector<int>> blocks_;
  std::vector<int32_t> cf_tab_, cb_tab_;  // [m*n]

  std::vector<int32_t> choices_;   // [N*m]
  std::vector<int64_t> dep_, ver_; // [N*m]
  std::vector<int64_t> last_user_, use_count_;  // [m*n]

  // simulation state
  struct Busy { bool on = false; int64_t end = 0; int kind = 0; int64_t y = 0; };
  struct Delivery { int64_t time; int to_B; int K; int64_t y; };
  std::vector<std::set<int64_t>> inF_, inB_;
  std::vector<std::vector<uint8_t>> fin_;  // fin_[K][y]
  std::vector<int64_t> fin_wm_;            // all y < fin_wm_[K] finished on K
  std::vector<Busy> busy_;
  std::vector<int> last_kind_;
  std::vector<Delivery> deliveries_;
  std::vector<int64_t> stall_, bubble_;
  int64_t t_ = 0, src_next_ = 0, done0_ = 0, makespan_ = -1;
  int phase_ = 0;
  bool finalized_ = false, done_ = false;

  std::vector<Task> tasks_;
  std::vector<std::vector<int64_t>> stage_tasks_;
};

// Point-to-point operations rank `rank` performs for global task t in multi-process mode
// (one process per stage), in the order the executor walks the plan: it posts the receive
// of an activation when the upstream F(y, rank-1) starts and of a gradient when the
// downstream B(y, rank+1) starts, and sends after its own F (to rank+1) and B (to rank-1).
// Each channel therefore carries y in the sender's plan order, which is exactly the
// receiver's posting order (test: tests/test_dist_gloo.py).
enum CommOp { SEND_ACT = 0, RECV_ACT = 1, SEND_GRAD = 2, RECV_GRAD = 3 };
struct CommStep {
  int op, peer;
  int64_t y;
};
inline int comm_ops(const Task& t, int rank, int D, CommStep out[2]) {
  int n = 0;
  if (t.kind == 0 && t.K == rank - 1) out[n++] = {RECV_ACT, rank - 1, t.y};
  if (t.kind == 1 && t.K == rank + 1) out[n++] = {RECV_GRAD, rank + 1, t.y};
  if (t.K == rank && t.kind == 0 && rank < D - 1) out[n++] = {SEND_ACT, rank + 1, t.y};
  if (t.K == rank && t.kind == 1 && rank > 0) out[n++] = {SEND_GRAD, rank - 1, t.y};
  return n;
}

// Belady residency over one stage's planned order (reading A9).
struct ResidencyEvent { int32_t K; int64_t i; int32_t op; int64_t uid; };  // op 0 LOAD 1 EVICT
struct ResidencyPlan {
  std::vector<ResidencyEvent> events;
  std::vector<std::pair<int64_t, int64_t>> writebacks;  // (task index, uid)
};
// Incremental Belady residency of one stage (SURVEY §8c O6 with the next-use horizon of
// reading A26).  Tasks are appended as the plan grows; the decision before task i is taken
// once tasks [i, i + max(L, H)) are known or the plan is final, so it never depends on how
// far the planner happened to be.  horizon <= 0: unbounded (needs the final plan).
class BeladyResidency {
 public:
  BeladyResidency(int K, std::vector<int64_t> bytes, int64_t budget, int L, int64_t horizon)
      : K_(K), bytes_(std::move(bytes)), budget_(budget), L_(L), H_(horizon) {}
  void push_task(std::vector<int64_t> sorted_uids, int kind) {
    uses_.push_back(std::move(sorted_uids));
    kinds_.push_back(kind);
  }
  void set_final() { final_ = true; }
  bool can_decide() const;
  // Decide the next task: appends its LOAD/EVICT events and write-backs.  Throws EBUDGET.
  void decide_next(std::vector<ResidencyEvent>& events, std::vector<std::pair<int64_t, int64_t>>& writebacks);
  int64_t decided() const { return next_; }
  int64_t known() const { return (int64_t)uses_.size(); }
  const std::vector<int64_t>& uses(int64_t i) const { return uses_[i]; }
  int kind(int64_t i) const { return kinds_[i]; }

 private:
  int64_t next_use(int64_t u, int64_t i) const;
  int64_t size_of(const std::set<int64_t>& s) const;
  int K_;
  std::vector<int64_t> bytes_;
  int64_t budget_;
  int L_;
  int64_t H_;
  bool final_ = false;
  int64_t next_ = 0;
  std::vector<std::vector<int64_t>> uses_;
  std::vector<int> kinds_;
  std::set<int64_t> resident_, dirty_;
};

// Whole-plan convenience wrapper (host planner API).
ResidencyPlan plan_residency(int K, const std::vector<std::vector<int64_t>>& uses,
                             const std::vector<int>& kinds, const std::vector<int64_t>& bytes,
                             int64_t budget, int L, int64_t horizon);

}  // namespace naspipe
