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
};

class Family {
 public:
  virtual ~Family() = default;
  // blocks: the stage's blocks (global ids), W slots
  virtual void forward(int slot, const int32_t* choice_of_block, const float* x_in, float* x_out,
                       cudaStream_t s) = 0;
  // dy: grad w.r.t. the stage output; dx: grad w.r.t. the stage input (nullptr: not needed)
  virtual void backward(int slot, const int32_t* choice_of_block, const float* dy, float* dx,
                        cudaStream_t s) = 0;
  // Candidate (local block j, choice c) parameters live in buffers the engine owns (resident
  // for the whole run, or loaded/evicted by the context switch); bind() points the family at
  // them (nullptr = not resident).  master() is the packed fp32 vector, the bf16 shadow holds
  // the GEMM operands (shadow_elems(c) elements; 0 for fp32 families).
  virtual void bind(int local_block, int c, float* w32, bf16* w16) = 0;
  virtual size_t shadow_elems(int c) const = 0;
  virtual float* master(int local_block, int c) = 0;
  virtual void refresh_shadow(int local_block, int c, cudaStream_t s) = 0;  // bf16 <- fp32
  FamilyCounters counters;
  KernelTimer* timer = nullptr;
};

std::unique_ptr<Family> make_family(const Spec& spec, const std::vector<int>& blocks, int W, DevArena& arena,
                                    cudaStream_t s);

}  // namespace naspipe
