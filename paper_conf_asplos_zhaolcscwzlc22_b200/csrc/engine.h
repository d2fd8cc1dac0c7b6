// Stage executor: turns the CSP plan into device work.  Each stage owns one compute stream
// (tasks in plan order), an input-copy stream, per-slot boundary buffers and events.  Slots
// are indexed y mod W: every in-flight subnet lies in [wm0, wm0 + W) (reading A7), so slot
// reuse is ordered by the plan itself.
#pragma once
#include <cuda_runtime.h>

#include <memory>
#include <string>
#include <vector>

#include "context.h"
#include "family.h"
#include "peer.h"
#include "planner.h"

namespace naspipe {

struct Transport;  // NCCL channels (multi-process mode)
int nccl_unique_id(void* out128);

struct StageRt {
  int K = 0, dev = 0;
  bool local = false;
  int64_t bulk = 0;  // BSP: bulk of the last task issued on this stage
  cudaStream_t comp = nullptr, copy = nullptr;
  std::unique_ptr<DevArena> arena;
  std::unique_ptr<Family> fam;
  std::unique_ptr<CandidateStore> store;  // candidate parameters (resident or context-switched)
  size_t pushed = 0;                      // stage tasks fed to the store
  // boundary buffers per slot (device, on dev); opaque bytes (Spec::act_bytes)
  size_t in_bytes = 0, out_bytes = 0;    // stage input (batch input at K = 0) / output
  size_t in_gbytes = 0, out_gbytes = 0;  // gradients w.r.t. them
  std::vector<void*> in, out, gin, gout, target;
  std::vector<cudaEvent_t> ev_f, ev_b, ev_in, ev_tgt;
  float* loss = nullptr;  // [loss_cap] on the last stage
};

struct BatchRec {
  naspipe_batch b;
};

class Engine {
 public:
  static std::unique_ptr<Engine> create_local(const Spec& spec, int D);
  static std::unique_ptr<Engine> create_rank(const Spec& spec, int D, int rank, int device, const void* nccl_ids);
  // one process per GPU, peer-memory transport (peer.h): create, export the blob, exchange
  // blobs out of band, connect to the neighbours' blobs, then submit as usual
  static std::unique_ptr<Engine> create_rank_peer(const Spec& spec, int D, int rank, int device);
  void peer_export(void* dst, size_t cap, size_t* n);
  void peer_connect(const void* prev, size_t prev_n, const void* next, size_t next_n);
  ~Engine();

  int64_t submit(const int32_t* choice, const naspipe_batch* batch);
  void drain();
  void get_params(int block, int choice, float* dst, size_t n);
  void set_params(int block, int choice, const float* src, size_t n);
  void get_losses(float* dst, int64_t n);
  void get_trace(int64_t* dst, size_t cap, size_t* n);
  void get_stats(double* dst16);
  void get_timed_stats(double* dst6);
  void set_timing(bool on);
  void get_residency_trace(int64_t* dst, size_t cap, size_t* n);
  void shutdown();

  void check_sticky() const;
  void set_sticky(int code, const std::string& msg);

 private:
  bool suppress_pdl_ = false;  // context switching or multi-process: PDL off while it lives
  void suppress_pdl();
  Engine(const Spec& spec, int D);
  void stage_sizes();
  void setup_stage(int K, int dev, bool local);
  void link_local_buffers();
  void feed_stores();
  void issue_planned();
  void issue(const Task& t);
  void issue_forward(StageRt& st, int64_t y, int slot);
  void drain_mirrored();
  void drain_timed();
  void issue_mirrored(const Task& t);
  void issue_backward(StageRt& st, int64_t y, int slot);
  void version_check(const Task& t);
  void cuda_check(const char* what);

  Spec spec_;
  int D_, W_;
  int rank_ = -1;  // -1: single process, all stages local
  Planner planner_;
  std::vector<StageRt> st_;
  std::unique_ptr<Transport> tx_;   // NCCL channels (create_rank)
  std::unique_ptr<PeerLink> peer_;  // peer-memory transport (create_rank_peer)
  // layer mirroring (NASPIPE_FLAG_MIRROR): per-subnet partitions, mirror copies, pushes
  bool mirror_ = false;
  std::vector<int32_t> msob_;          // [N][m] stage of block b for subnet y
  int64_t mbase_ = 0, mticks_ = 0;     // first subnet of the undrained batch; ticks so far
  std::vector<int> mwriter_;           // per candidate: stage of its last WRITE (-1: none)
  std::vector<cudaEvent_t> ev_push_;   // per candidate: its last push to the other stages
  std::vector<cudaStream_t> push_;     // per stage
  std::vector<cudaEvent_t> ev_wrote_;  // per stage: the backward whose WRITEs are pushed
  // timing-driven execution (NASPIPE_FLAG_TIMED): one running task per stage, observed
  // through ev_run_[K]; subnets [tbase_, N) run at the next drain
  bool timed_ = false;
  int64_t tbase_ = 0;
  std::vector<cudaEvent_t> ev_run_;
  double tstat_[6] = {0, 0, 0, 0, 0, 0};
  std::vector<BatchRec> batches_;
  std::vector<int32_t> stage_choice_;  // scratch
  size_t issued_ = 0;
  bool drained_ = false;
  int64_t loss_cap_ = 1 << 20;
  int sticky_code_ = 0;
  std::string sticky_msg_;
  // version counters per candidate (host mirror, VERSION_CHECK)
  std::vector<int64_t> version_;
  uint64_t version_checks_ = 0;
  // stats
  double h2d_bytes_ = 0, d2h_bytes_ = 0, p2p_bytes_ = 0;
  uint64_t engine_launches_ = 0;  // kernels launched by the engine itself (loss, synthetic data)
  std::vector<Task> trace_;
  KernelTimer timer_;
};

}  // namespace naspipe
