// extern "C" boundary (include/naspipe.h).  Converts exceptions into status codes and the
// thread-local last-error message; no computation happens here.
#include <algorithm>
#include <cstring>
#include <memory>

#include "engine.h"
#include "launch.h"
#include "mirror.h"
#include "planner.h"

using namespace naspipe;

namespace naspipe {
static thread_local std::string g_last_error;
void set_last_error(const std::string& msg) { g_last_error = msg; }
}  // namespace naspipe

template <class F>
static int guarded(F&& f) {
  try {
    f();
    return NASPIPE_OK;
  } catch (const Error& e) {
    set_last_error(e.what());
    return e.code;
  } catch (const std::bad_alloc&) {
    set_last_error("host allocation failed");
    return NASPIPE_ENOMEM;
  } catch (const std::exception& e) {
    set_last_error(e.what());
    return NASPIPE_EINTERNAL;
  }
}

struct naspipe_plan_handle {
  std::unique_ptr<Spec> spec;
  std::unique_ptr<Planner> planner;
};

extern "C" {

const char* naspipe_last_error(void) { return g_last_error.c_str(); }
int naspipe_abi_version(void) { return NASPIPE_ABI_VERSION; }

int naspipe_param_count(const naspipe_supernet_spec* spec, int32_t block, int32_t choice,
                        size_t* n_floats) {
  return guarded([&] {
    Spec s(spec);
    NP_REQUIRE(block >= 0 && block < s.m() && choice >= 0 && choice < s.n(), NASPIPE_EINVAL,
               "candidate (%d,%d) out of range", block, choice);
    NP_REQUIRE(n_floats, NASPIPE_EINVAL, "n_floats NULL");
    *n_floats = s.param_count(block, choice);
  });
}

int naspipe_default_costs(const naspipe_supernet_spec* spec, int32_t* cost_fwd, int32_t* cost_bwd) {
  return guarded([&] {
    Spec s(spec);
    NP_REQUIRE(cost_fwd && cost_bwd, NASPIPE_EINVAL, "NULL output");
    s.default_costs(cost_fwd, cost_bwd);
  });
}

int naspipe_partition(const naspipe_supernet_spec* spec, int32_t n_stages, int32_t* stage_of_block) {
  return guarded([&] {
    Spec s(spec);
    NP_REQUIRE(stage_of_block, NASPIPE_EINVAL, "NULL output");
    auto sob = s.partition(n_stages);
    std::memcpy(stage_of_block, sob.data(), sob.size() * sizeof(int32_t));
  });
}

int naspipe_plan_mirrored(const naspipe_supernet_spec* spec, int32_t n_stages, const int32_t* choices,
                          int64_t n_subnets, int32_t mirror_latency, int32_t* stage_of_block, int64_t* trace,
                          size_t cap_tasks, size_t* n_tasks, int64_t* makespan, int64_t* stall, int64_t* bubble) {
  return guarded([&] {
    Spec s(spec);
    NP_REQUIRE(n_tasks && makespan, NASPIPE_EINVAL, "NULL output");
    const MirrorPlan P = plan_mirrored(s, n_stages, choices, n_subnets, mirror_latency);
    if (stage_of_block) std::memcpy(stage_of_block, P.sob.data(), P.sob.size() * sizeof(int32_t));
    *n_tasks = P.trace.size();
    for (size_t i = 0; i < P.trace.size() && i < cap_tasks && trace; ++i) {
      trace[4 * i] = P.trace[i].t;
      trace[4 * i + 1] = P.trace[i].K;
      trace[4 * i + 2] = P.trace[i].kind;
      trace[4 * i + 3] = P.trace[i].y;
    }
    *makespan = P.makespan;
    for (int K = 0; K < n_stages; ++K) {
      if (stall) stall[K] = P.stall[K];
      if (bubble) bubble[K] = P.bubble[K];
    }
  });
}

int naspipe_init_params(const naspipe_supernet_spec* spec, int32_t block, int32_t choice,
                        float* dst, size_t n_floats) {
  return guarded([&] {
    Spec s(spec);
    NP_REQUIRE(block >= 0 && block < s.m() && choice >= 0 && choice < s.n(), NASPIPE_EINVAL,
               "candidate (%d,%d) out of range", block, choice);
    NP_REQUIRE(dst && n_floats == s.param_count(block, choice), NASPIPE_EINVAL,
               "n_floats %zu != %zu", n_floats, s.param_count(block, choice));
    s.init_params(block, choice, dst);
  });
}

int naspipe_init_frozen(const naspipe_supernet_spec* spec, int32_t part, float* dst, size_t n_floats) {
  return guarded([&] {
    Spec s(spec);
    NP_REQUIRE(s.family() == NASPIPE_SPOS_CNN && part >= 0 && part <= 2, NASPIPE_EINVAL,
               "frozen part %d (SPOS only: 0 stem, 1 head, 2 fc)", part);
    NP_REQUIRE(dst && n_floats == s.frozen_count(part), NASPIPE_EINVAL, "n_floats %zu != %zu", n_floats,
               s.frozen_count(part));
    s.init_frozen(part, dst);
  });
}

int naspipe_plan_create(const naspipe_supernet_spec* spec, int32_t n_stages, const int32_t* choices,
                        int64_t n_subnets, naspipe_plan_t** out) {
  return guarded([&] {
    NP_REQUIRE(out && (choices || n_subnets == 0) && n_subnets >= 0, NASPIPE_EINVAL, "bad args");
    auto p = std::make_unique<naspipe_plan_handle>();
    p->spec = std::make_unique<Spec>(spec);
    p->planner = std::make_unique<Planner>(*p->spec, n_stages);
    const int m = p->spec->m();
    for (int64_t y = 0; y < n_subnets; ++y) {
      p->planner->add_subnet(choices + y * m);
      p->planner->advance();
    }
    p->planner->finalize();
    p->planner->advance();
    *out = p.release();
  });
}

int naspipe_plan_trace(const naspipe_plan_t* p, int64_t* dst, size_t cap_tasks, size_t* n_tasks) {
  return guarded([&] {
    NP_REQUIRE(p && n_tasks, NASPIPE_EINVAL, "bad args");
    const auto& t = p->planner->tasks();
    *n_tasks = t.size();
    for (size_t i = 0; i < t.size() && i < cap_tasks && dst; ++i) {
      dst[4 * i] = t[i].t;
      dst[4 * i + 1] = t[i].K;
      dst[4 * i + 2] = t[i].kind;
      dst[4 * i + 3] = t[i].y;
    }
  });
}

int naspipe_plan_makespan(const naspipe_plan_t* p, int64_t* makespan) {
  return guarded([&] {
    NP_REQUIRE(p && makespan, NASPIPE_EINVAL, "bad args");
    *makespan = p->planner->makespan();
  });
}

int naspipe_plan_deps(const naspipe_plan_t* p, int64_t y, int32_t stage, int64_t* dst, size_t cap,
                      size_t* n) {
  return guarded([&] {
    NP_REQUIRE(p && n && y >= 0 && y < p->planner->n_subnets() && stage >= 0 &&
                   stage < p->planner->D(),
               NASPIPE_EINVAL, "bad args");
    auto d = p->planner->deps(y, stage);
    *n = d.size();
    for (size_t i = 0; i < d.size() && i < cap && dst; ++i) dst[i] = d[i];
  });
}

int naspipe_plan_residency(const naspipe_plan_t* p, int32_t stage, int64_t budget_bytes, int32_t depth,
                           int32_t horizon, int64_t* dst, size_t cap, size_t* n, int64_t* n_writebacks) {
  return guarded([&] {
    NP_REQUIRE(p && n && stage >= 0 && stage < p->planner->D() && budget_bytes >= 0 && depth >= 0,
               NASPIPE_EINVAL, "bad args");
    const Planner& pl = *p->planner;
    const Spec& s = *p->spec;
    std::vector<std::vector<int64_t>> uses;
    std::vector<int> kinds;
    for (int64_t ti : pl.stage_tasks()[stage]) {
      const Task& t = pl.tasks()[ti];
      std::vector<int64_t> u;
      for (int b : pl.blocks_of(stage)) u.push_back((int64_t)b * s.n() + pl.choice(t.y, b));
      std::sort(u.begin(), u.end());
      uses.push_back(u);
      kinds.push_back(t.kind);
    }
    std::vector<int64_t> bytes((size_t)s.m() * s.n());
    for (int b = 0; b < s.m(); ++b)
      for (int c = 0; c < s.n(); ++c) bytes[(size_t)b * s.n() + c] = 4 * (int64_t)s.param_count(b, c);
    ResidencyPlan rp;
    if (budget_bytes > 0)
      rp = plan_residency(stage, uses, kinds, bytes, budget_bytes, depth > 0 ? depth : s.lookahead(),
                          horizon == 0 ? s.residency_horizon() : horizon);
    *n = rp.events.size();
    if (n_writebacks) *n_writebacks = (int64_t)rp.writebacks.size();
    for (size_t i = 0; i < rp.events.size() && i < cap && dst; ++i) {
      dst[4 * i] = rp.events[i].K;
      dst[4 * i + 1] = rp.events[i].i;
      dst[4 * i + 2] = rp.events[i].op;
      dst[4 * i + 3] = rp.events[i].uid;
    }
  });
}

int naspipe_plan_idle(const naspipe_plan_t* p, int64_t* stall, int64_t* bubble) {
  return guarded([&] {
    NP_REQUIRE(p && stall && bubble, NASPIPE_EINVAL, "bad args");
    for (int K = 0; K < p->planner->D(); ++K) {
      stall[K] = p->planner->stall_ticks()[K];
      bubble[K] = p->planner->bubble_ticks()[K];
    }
  });
}

int naspipe_plan_comm_schedule(const naspipe_plan_t* p, int32_t rank, int64_t* dst, size_t cap, size_t* n) {
  return guarded([&] {
    NP_REQUIRE(p && n && rank >= 0 && rank < p->planner->D(), NASPIPE_EINVAL, "bad args");
    size_t k = 0;
    for (const Task& t : p->planner->tasks()) {
      CommStep ops[2];
      const int m = comm_ops(t, rank, p->planner->D(), ops);
      for (int i = 0; i < m; ++i, ++k)
        if (dst && k < cap) {
          dst[3 * k] = ops[i].op;
          dst[3 * k + 1] = ops[i].peer;
          dst[3 * k + 2] = ops[i].y;
        }
    }
    *n = k;
  });
}

void naspipe_plan_destroy(naspipe_plan_t* p) { delete p; }

int naspipe_set_pdl(int enabled) {
  return guarded([&] { pdl_runtime_off().store(enabled ? 0 : 1); });
}

int naspipe_nccl_unique_id(void* out128) {
  return guarded([&] {
    NP_REQUIRE(out128, NASPIPE_EINVAL, "out NULL");
    nccl_unique_id(out128);
  });
}

// ---------------------------------------------------------------------------------------
// Engine
// ---------------------------------------------------------------------------------------
struct naspipe_handle {
  std::unique_ptr<Engine> eng;
};

int naspipe_create(const naspipe_supernet_spec* spec, int32_t n_stages, naspipe_t** out) {
  return guarded([&] {
    NP_REQUIRE(out, NASPIPE_EINVAL, "out NULL");
    const Spec sp(spec);
    NP_REQUIRE(sp.raw.sync_policy != NASPIPE_SYNC_BSP || sp.raw.hbm_weight_budget_bytes == 0, NASPIPE_EINVAL,
               "BSP runs with every candidate resident (hbm_weight_budget_bytes = 0)");
    auto h = std::make_unique<naspipe_handle>();
    h->eng = Engine::create_local(sp, n_stages);
    *out = h.release();
  });
}

int naspipe_create_rank(const naspipe_supernet_spec* spec, int32_t n_stages, int32_t stage_rank,
                        int32_t device, const void* nccl_ids, naspipe_t** out) {
  return guarded([&] {
    NP_REQUIRE(out, NASPIPE_EINVAL, "out NULL");
    const Spec sp(spec);
    NP_REQUIRE(sp.raw.sync_policy != NASPIPE_SYNC_BSP || sp.raw.hbm_weight_budget_bytes == 0, NASPIPE_EINVAL,
               "BSP runs with every candidate resident (hbm_weight_budget_bytes = 0)");
    auto h = std::make_unique<naspipe_handle>();
    h->eng = Engine::create_rank(sp, n_stages, stage_rank, device, nccl_ids);
    *out = h.release();
  });
}

int naspipe_create_rank_peer(const naspipe_supernet_spec* spec, int32_t n_stages, int32_t stage_rank,
                             int32_t device, naspipe_t** out) {
  return guarded([&] {
    NP_REQUIRE(out, NASPIPE_EINVAL, "out NULL");
    const Spec sp(spec);
    NP_REQUIRE(sp.raw.sync_policy != NASPIPE_SYNC_BSP || sp.raw.hbm_weight_budget_bytes == 0, NASPIPE_EINVAL,
               "BSP runs with every candidate resident (hbm_weight_budget_bytes = 0)");
    auto h = std::make_unique<naspipe_handle>();
    h->eng = Engine::create_rank_peer(sp, n_stages, stage_rank, device);
    *out = h.release();
  });
}

#define ENGINE_CALL(h, body)                                         \
  guarded([&] {                                                       \
    NP_REQUIRE((h) != nullptr, NASPIPE_EINVAL, "handle NULL");       \
    Engine& e = *(h)->eng;                                            \
    e.check_sticky();                                                 \
    try {                                                             \
      body;                                                           \
    } catch (const Error& err) {                                      \
      if (err.code == NASPIPE_ECUDA || err.code == NASPIPE_ENCCL ||   \
          err.code == NASPIPE_EINTERNAL)                              \
        e.set_sticky(err.code, err.what());                           \
      throw;                                                          \
    }                                                                 \
  })

int naspipe_submit(naspipe_t* h, const int32_t* choice, const naspipe_batch* batch, int64_t* seq_id_out) {
  return ENGINE_CALL(h, {
    const int64_t y = e.submit(choice, batch);
    if (seq_id_out) *seq_id_out = y;
  });
}

int naspipe_drain(naspipe_t* h) { return ENGINE_CALL(h, e.drain()); }

int naspipe_peer_export(naspipe_t* h, void* dst, size_t cap, size_t* n) {
  return ENGINE_CALL(h, e.peer_export(dst, cap, n));
}

int naspipe_peer_connect(naspipe_t* h, const void* prev_blob, size_t prev_n, const void* next_blob, size_t next_n) {
  return ENGINE_CALL(h, e.peer_connect(prev_blob, prev_n, next_blob, next_n));
}

int naspipe_get_params(naspipe_t* h, int32_t block, int32_t choice, float* dst, size_t n_floats) {
  return ENGINE_CALL(h, e.get_params(block, choice, dst, n_floats));
}

int naspipe_set_params(naspipe_t* h, int32_t block, int32_t choice, const float* src, size_t n_floats) {
  return ENGINE_CALL(h, e.set_params(block, choice, src, n_floats));
}

int naspipe_get_losses(naspipe_t* h, float* dst, int64_t n) { return ENGINE_CALL(h, e.get_losses(dst, n)); }

int naspipe_get_trace(naspipe_t* h, int64_t* dst, size_t cap_tasks, size_t* n_tasks) {
  return ENGINE_CALL(h, e.get_trace(dst, cap_tasks, n_tasks));
}

int naspipe_get_stats(naspipe_t* h, double* dst16) { return ENGINE_CALL(h, e.get_stats(dst16)); }

int naspipe_set_timing(naspipe_t* h, int on) { return ENGINE_CALL(h, e.set_timing(on != 0)); }

int naspipe_get_timed_stats(naspipe_t* h, double* dst6) { return ENGINE_CALL(h, e.get_timed_stats(dst6)); }

int naspipe_get_residency_trace(naspipe_t* h, int64_t* dst, size_t cap, size_t* n) {
  return ENGINE_CALL(h, e.get_residency_trace(dst, cap, n));
}

void naspipe_destroy(naspipe_t* h) {
  if (!h) return;
  try {
    h->eng->shutdown();
  } catch (...) {
  }
  delete h;
}

}  // extern "C"
