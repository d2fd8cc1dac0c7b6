// Per-stage model state of one block family: candidate parameters (fp32 masters, bf16
// shadows), the per-slot activation stash kept between F(y,K) and B(y,K), and the per-stage
// backward workspace.  forward()/backward() enqueue the stage's kernels on one stream.
#pragma once
#include <cuda_runtime.h>

#include <memory>
#include <vector>

#include "kernels.h"
#include "spec.h"

namespace naspipe {

// Device allocations of one stage (freed together).
class DevArena {
 public:
  explicit DevArena(int dev) : dev_(dev) {}
  ~DevArena();
  template <class T>
  T* alloc(size_t n) { return static_cast<T*>(raw(n * sizeof(T))); }
  size_t bytes() const { return bytes_; }

 private:
  void* raw(size_t bytes);
  int dev_;
  size_t bytes_ = 0;
  std::vector<void*> ptrs_;
};

// Optional CUDA-event timing of the dominant kernel (the tcgen05 GEMM).
struct KernelTimer {
  bool on = false;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> pairs;
  size_t used = 0;
  double flops = 0, launches = 0, ms = 0;
  void begin(cudaStream_t s);
  void end(cudaStream_t s, double f);
  void collect();  // synchronises the recorded events, accumulates ms
  ~KernelTimer();
};

struct FamilyCounters {
  uint64_t launches = 0;
  // algorithmic HBM bytes of every kernel the family launched (SPOS: each tensor read and
  // written once per launch at its stored width; stats [15], the whole-step roofline)
  double bytes = 0;
};

class Family {
 public:
  virtual ~Family() = default;
  // blocks: the stage's blocks (global ids), W slots.  Boundary tensors are opaque here:
  // fp32 [B, sample] for MLP/TRANSFORMER, bf16 NHWC for SPOS (the stage-0 input is the
  // batch input itself, see Spec::act_bytes / input_bytes).
  virtual void forward(int slot, const int32_t* choice_of_block, const void* x_in, void* x_out,
                       cudaStream_t s) = 0;
  // dy: grad w.r.t. the stage output; dx: grad w.r.t. the stage input (nullptr: not needed)
  virtual void backward(int slot, const int32_t* choice_of_block, const void* dy, void* dx,
                        cudaStream_t s) = 0;
  // Last stage only: loss of the stage output against the target -> *loss_dst (device) and
  // the seed gradient dy (same layout as the output).  MSE (reading A18) unless overridden.
  virtual void loss(int slot, const void* out, const void* target, void* dy, float* loss_dst,
                    cudaStream_t s);
  // synthetic target (perf runs): N(0,1)-like fp32 by default, labels for SPOS
  virtual void synth_target(void* dst, uint64_t seed, cudaStream_t s);
  // Candidate (local block j, choice c) parameters live in buffers the engine owns (resident
  // for the whole run, or loaded/evicted by the context switch); bind() points the family at
  // them (nullptr = not resident).  master() is the packed fp32 vector, the bf16 shadow holds
  // the GEMM operands (shadow_elems(j, c) elements; 0 for fp32 families).
  virtual void bind(int local_block, int c, float* w32, bf16* w16) = 0;
  virtual size_t shadow_elems(int local_block, int c) const = 0;
  virtual float* master(int local_block, int c) = 0;
  virtual void refresh_shadow(int local_block, int c, cudaStream_t s) = 0;  // bf16 <- fp32
  // BSP (reading A30): inside a bulk every forward and input gradient reads the bulk-start
  // weights (master + shadow) while the SGD WRITEs accumulate into a separate fp32 copy
  // bound here (nullptr = update in place, every other policy); the engine copies it back
  // into the master (and refreshes the shadow) at the bulk's flush.
  void bind_update(int local_block, int c, float* acc) {
    const size_t k = (size_t)local_block * n_choices_ + c;
    if (upd_.size() <= k) upd_.resize(k + 1, nullptr);
    upd_[k] = acc;
  }
  float* upd(int local_block, int c) {
    const size_t k = (size_t)local_block * n_choices_ + c;
    return (k < upd_.size() && upd_[k]) ? upd_[k] : master(local_block, c);
  }
  bool in_place(int local_block, int c) const {
    const size_t k = (size_t)local_block * n_choices_ + c;
    return k >= upd_.size() || upd_[k] == nullptr;
  }
  // Layer mirroring (NASPIPE_FLAG_MIRROR, reading A31): a stage's family holds every block and
  // a task runs the contiguous local range [lo, hi) its subnet's partition assigns to the
  // stage; the fixed partition runs [0, #blocks).  Set by the engine before forward/backward.
  void set_range(int lo, int hi) {
    lo_ = lo;
    hi_ = hi;
  }
  int rlo() const { return lo_; }
  int rhi(int nb) const { return hi_ < nb ? hi_ : nb; }
  // called by the engine after a drain's synchronisation (device-side sticky checks)
  virtual void check_after_drain() {}
  FamilyCounters counters;
  KernelTimer* timer = nullptr;

 protected:
  const Spec* spec_base_ = nullptr;
  int n_choices_ = 1;            // set by the families (bind_update's key)
  std::vector<float*> upd_;      // BSP accumulators, [local_block * n + c]
  float* mse_part_ = nullptr;  // MSE workspace (last stage)
  int lo_ = 0, hi_ = 1 << 30;  // task block range (set_range)
};

std::unique_ptr<Family> make_family(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& arena,
                                    cudaStream_t s);
std::unique_ptr<Family> make_spos_family(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& arena);

}  // namespace naspipe
