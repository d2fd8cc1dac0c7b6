// Candidate storage of one stage and the context switch (PAPER.md P:L156,
// P:L160-162; readings A9, A26).
//
// Budget 0: every candidate of the stage is resident in HBM for the whole run.
// Budget > 0: all candidates live in a pinned host stash (fp32 masters, "by default,
// the supernet's operators all reside in CPU storage"); before each task the Belady plan
// (BeladyResidency: farthest next use within the horizon, depth-L prefetch that fits the
// budget) issues EVICTs (D2H write-back only if updated since load) and LOADs (H2D + bf16
// shadow refresh) on the stage's copy stream; an eviction copies a dirty candidate into a
// device staging slot and frees it at once, the D2H from the slot and the shadow kernels run
// on their own streams, so both PCIe directions stay busy; the compute stream waits only for the
// candidates of the task it is about to run, so prefetches for later tasks overlap compute.
// Numerics are unaffected by residency: a candidate's bytes are the same wherever it lives.
#pragma once
#include <cuda_runtime.h>

#include <memory>
#include <vector>

#include "family.h"
#include "planner.h"

namespace naspipe {

class CandidateStore {
 public:
  // blocks: the blocks this stage holds candidates of (the planner's partition, or every
  // block under layer mirroring)
  CandidateStore(const Spec& spec, const Planner& planner, int K, int dev, Family* fam, DevArena* arena,
                 int64_t budget, const std::vector<int>& blocks);
  ~CandidateStore();
  bool managed() const { return budget_ > 0; }

  // plan feed (host thread)
  void push_task(const Task& t);
  void set_final();
  bool ready() const;  // the next stage task's residency can be decided

  // issue hooks, in the stage's plan order
  void before_task(const Task& t, cudaStream_t comp, cudaStream_t copy);
  void after_task(const Task& t, cudaStream_t comp);

  void sync();  // wait for outstanding write-backs

  // BSP (reading A30; all candidates resident): an fp32 accumulator per candidate takes the
  // SGD WRITEs of a bulk (Family::bind_update) while the bulk reads the masters; after_task
  // marks a backward's candidates dirty, bsp_flush copies the dirty accumulators into the
  // masters and refreshes their bf16 shadows on stream s.
  void enable_bsp(DevArena* arena);
  void bsp_flush(cudaStream_t s);
  // device copy of candidate (b, c) (resident mode): fp32 master, bf16 shadow and their sizes
  float* dev_master(int b, int c) { return cands_[uid_of(b, c)].w32; }
  bf16* dev_shadow(int b, int c) { return cands_[uid_of(b, c)].w16; }
  size_t n32(int b, int c) const { return cands_[uid_of(b, c)].n32; }
  size_t n16(int b, int c) const { return cands_[uid_of(b, c)].n16; }
  // read-out (streams idle)
  void get(int b, int c, float* dst);
  void set(int b, int c, const float* src, cudaStream_t s);

  uint64_t loads = 0, evicts = 0, writebacks = 0;
  double h2d_bytes = 0, d2h_bytes = 0;
  std::vector<ResidencyEvent> log;

 private:
  cudaMemPool_t pool_ = nullptr;  // private pool of the managed candidates (context switching)
  struct Cand {
    int j = -1, c = -1;  // local block, choice
    size_t n32 = 0, n16 = 0;
    float* stash = nullptr;  // pinned host fp32 master (managed mode)
    float* w32 = nullptr;    // device, when resident
    bf16* w16 = nullptr;
    cudaEvent_t ready = nullptr, last_use = nullptr, wb_done = nullptr, h2d_done = nullptr;
    float* acc = nullptr;  // BSP accumulator
    bool dirty = false;
  };
  int uid_of(int b, int c) const { return b * n_ + c; }
  std::vector<int64_t> task_uids(const Task& t) const;
  void load(Cand& cd, cudaStream_t copy);
  void evict(Cand& cd, bool writeback, cudaStream_t copy);

  const Spec& spec_;
  const Planner& planner_;
  int K_, dev_, n_;
  Family* fam_;
  int64_t budget_;
  std::vector<Cand> cands_;  // indexed by uid (only this stage's blocks are populated)
  cudaStream_t evict_ = nullptr;   // evictions: D2D into a staging slot, then the free
  cudaStream_t shadow_ = nullptr;  // bf16 shadow refresh of loaded candidates (a kernel)
  cudaStream_t wb_ = nullptr;      // D2H of staged write-backs
  static constexpr int kStage = 2;  // write-back staging slots (max candidate fp32 bytes each)
  float* stage_[kStage] = {nullptr, nullptr};
  cudaEvent_t stage_free_[kStage] = {nullptr, nullptr}, staged_[kStage] = {nullptr, nullptr};
  bool stage_used_[kStage] = {false, false};
  uint64_t stage_next_ = 0;
  std::unique_ptr<BeladyResidency> belady_;
  bool bsp_ = false;
};

}  // namespace naspipe
