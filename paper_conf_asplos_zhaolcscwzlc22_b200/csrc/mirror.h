// Per-subnet balanced partitions with layer mirroring: a planning-only CSP schedule
// (reading A31; see mirror.cpp).
#pragma once
#include <cstdint>
#include <vector>

#include "planner.h"
#include "spec.h"

namespace naspipe {

struct MirrorPlan {
  std::vector<int32_t> sob;  // [N][m] stage of block b in subnet y
  std::vector<Task> trace;   // task starts in decision order
  int64_t makespan = 0;
  std::vector<int64_t> stall, bubble;  // idle ticks per stage (blocked forward / nothing queued)
};

MirrorPlan plan_mirrored(const Spec& spec, int D, const int32_t* choices, int64_t N, int64_t mirror_latency);

}  // namespace naspipe
