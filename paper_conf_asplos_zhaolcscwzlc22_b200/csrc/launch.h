// Kernel launch with programmatic dependent launch (PDL) enabled: the launch of a kernel
// overlaps the tail of the previous kernel in the stream; the kernel itself waits
// (ptx::pdl_wait) before reading its predecessors' outputs.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdlib>

#include "common.h"

namespace naspipe {

// Engines alive in this process that launch without PDL:
// * context-switching engines (hbm_weight_budget_bytes > 0): the compute stream's kernels
//   follow cross-stream event waits (a candidate's load / shadow refresh is ready).  Round 1
//   saw a 14-subnet configs[3] run deadlock with PDL.  Round 2 moved the GEMMs' TMEM
//   allocation after griddepcontrol.wait (an early-launched CTA no longer holds TMEM while
//   it waits); with that, the reproduction (tools/c4_probe.py --no-drain, NASPIPE_FORCE_PDL=1)
//   passed 3 of 3 runs and tests/test_gpu_context.py passed, but the bench's configs[3] run
//   (submit/drain cycles, HOST batches) still hung with PDL (killed by its 600 s timeout).
//   Root cause not found: PDL stays off for these engines (DESIGN.md §5 "PDL").
// * multi-process rank engines: their compute streams wait on transport streams / peer
//   flags between kernels (the same cross-stream pattern).
// The CTA-pair GEMM's early triggers (NASPIPE_PAIR_TRIGGER=1) also still hang
// tools/hangtest.sh and stay off.
// Stream priorities (NASPIPE_STREAM_PRIO=1; OFF by default): a stage's compute stream (the
// task's critical chain) at the highest priority, the families' side streams (weight
// gradients) at the lowest.  Measured neutral on configs[1] / configs[2]
// (profiles/r2_ab2/), and with it the configs[3] context-switching bench HUNG (killed after
// 900 s; 86 s without, same box) -- root cause not found, so the default stays off.
inline bool stream_prio_on() {
  static const bool v = [] {
    const char* e = getenv("NASPIPE_STREAM_PRIO");
    return e && e[0] == '1';
  }();
  return v;
}
inline cudaError_t create_stream(cudaStream_t* s, bool critical) {
  int lo = 0, hi = 0;
  if (!stream_prio_on() || cudaDeviceGetStreamPriorityRange(&lo, &hi) != cudaSuccess)
    return cudaStreamCreateWithFlags(s, cudaStreamNonBlocking);
  return cudaStreamCreateWithPriority(s, cudaStreamNonBlocking, critical ? hi : lo);
}

inline std::atomic<int>& pdl_suppressors() {
  static std::atomic<int> n{0};
  return n;
}

// NASPIPE_NO_PDL=1 launches without the PDL attribute; NASPIPE_FORCE_PDL=1 keeps it even
// while a suppressing engine lives (diagnostics: the deadlock reproductions).
// naspipe_set_pdl(0): process-wide switch for measurement runs (bench.py times each kernel's
// own execution with CUPTI: with PDL a kernel's recorded interval starts while it still waits
// in griddepcontrol.wait for its predecessor, so summed durations double-count the overlap)
inline std::atomic<int>& pdl_runtime_off() {
  static std::atomic<int> v{0};
  return v;
}
inline bool pdl_enabled() {
  if (pdl_runtime_off().load(std::memory_order_relaxed)) return false;
  static const int v = [] {
    const char* e = getenv("NASPIPE_NO_PDL");
    const char* f = getenv("NASPIPE_FORCE_PDL");
    return (e && e[0] == '1') ? 0 : (f && f[0] == '1') ? 2 : 1;
  }();
  return v == 2 || (v == 1 && pdl_suppressors().load(std::memory_order_relaxed) == 0);
}

template <typename... KArgs, typename... Args>
inline void launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                       Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  const cudaError_t e = cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
  if (e != cudaSuccess) cudaGetLastError();  // consume it: a launch-configuration error is not sticky
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "kernel launch: %s", cudaGetErrorString(e));
}

}  // namespace naspipe
