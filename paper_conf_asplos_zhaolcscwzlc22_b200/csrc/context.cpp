// Candidate storage and the context switch (see context.h).
#include "context.h"

#include <algorithm>
#include <atomic>
#include <cstring>
#include <thread>

namespace naspipe {

#define CU(call)                                                                               \
  do {                                                                                         \
    cudaError_t e_ = (call);                                                                   \
    NP_REQUIRE(e_ == cudaSuccess, NASPIPE_ECUDA, "%s: %s", #call, cudaGetErrorString(e_));     \
  } while (0)

CandidateStore::CandidateStore(const Spec& spec, const Planner& planner, int K, int dev, Family* fam,
                               DevArena* arena, int64_t budget, const std::vector<int>& blocks)
    : spec_(spec), planner_(planner), K_(K), dev_(dev), n_(spec.n()), fam_(fam), budget_(budget) {
  cands_.resize((size_t)spec.m() * n_);
  std::vector<int> uids;
  for (size_t j = 0; j < blocks.size(); ++j)
    for (int c = 0; c < n_; ++c) {
      Cand& cd = cands_[uid_of(blocks[j], c)];
      cd.j = (int)j;
      cd.c = c;
      cd.n32 = spec.param_count(blocks[j], c);
      cd.n16 = fam->shadow_elems(j, c);
      uids.push_back(uid_of(blocks[j], c));
    }
  CU(cudaSetDevice(dev));
  if (managed()) {
    // EBUDGET: the largest possible task need (the biggest candidate of every block) must fit
    int64_t worst = 0;
    for (int b : blocks) {
      int64_t mx = 0;
      for (int c = 0; c < n_; ++c) mx = std::max<int64_t>(mx, 4 * (int64_t)spec.param_count(b, c));
      worst += mx;
    }
    NP_REQUIRE(worst <= budget_, NASPIPE_EBUDGET,
               "stage %d: HBM weight budget %lld bytes cannot hold one task's candidates (%lld bytes)", K,
               (long long)budget_, (long long)worst);
    std::vector<int64_t> bytes(cands_.size(), 0);
    for (int u : uids) bytes[u] = 4 * (int64_t)cands_[u].n32;
    belady_ = std::make_unique<BeladyResidency>(K, bytes, budget_, spec.lookahead(), spec.residency_horizon());
    for (int u : uids) {
      CU(cudaHostAlloc(reinterpret_cast<void**>(&cands_[u].stash), cands_[u].n32 * 4, cudaHostAllocDefault));
      CU(cudaEventCreateWithFlags(&cands_[u].ready, cudaEventDisableTiming));
      CU(cudaEventCreateWithFlags(&cands_[u].last_use, cudaEventDisableTiming));
      CU(cudaEventCreateWithFlags(&cands_[u].wb_done, cudaEventDisableTiming));
      CU(cudaEventCreateWithFlags(&cands_[u].h2d_done, cudaEventDisableTiming));
    }
    CU(cudaStreamCreateWithFlags(&evict_, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&shadow_, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&wb_, cudaStreamNonBlocking));
    // write-back staging ring: an evicted dirty candidate is copied device-to-device into a
    // staging slot (HBM speed) and its memory freed at once; the D2H from the slot runs on
    // wb_.  A load that reuses the freed memory therefore waits only for the D2D copy, not for
    // the PCIe write-back, so both PCIe directions stream concurrently.
    size_t max_n32 = 0;
    for (int u : uids) max_n32 = std::max(max_n32, cands_[u].n32);
    for (int i = 0; i < kStage; ++i) {
      CU(cudaMalloc(reinterpret_cast<void**>(&stage_[i]), max_n32 * 4));
      CU(cudaEventCreateWithFlags(&stage_free_[i], cudaEventDisableTiming));
      CU(cudaEventCreateWithFlags(&staged_[i], cudaEventDisableTiming));
    }
    // a private stream-ordered pool (the device's default pool and stream 0 are
    // left alone) that keeps freed blocks: loads reuse evicted memory
    cudaMemPoolProps props{};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    CU(cudaMemPoolCreate(&pool_, &props));
    uint64_t thr = UINT64_MAX;
    CU(cudaMemPoolSetAttribute(pool_, cudaMemPoolAttrReleaseThreshold, &thr));
    // reserve the pool up front (fp32 masters + bf16 shadows of a full budget, plus the
    // in-flight loads/evictions) so no load pays for growing the pool mid-run
    void* reserve = nullptr;
    const size_t rbytes = (size_t)(2.0 * (double)budget_);
    if (cudaMallocFromPoolAsync(&reserve, rbytes, pool_, evict_) == cudaSuccess) {
      cudaFreeAsync(reserve, evict_);
      cudaStreamSynchronize(evict_);
    } else {
      cudaGetLastError();  // not fatal: the pool grows on demand
    }
  } else {
    for (int u : uids) {
      cands_[u].w32 = arena->alloc<float>(cands_[u].n32);
      cands_[u].w16 = cands_[u].n16 ? arena->alloc<bf16>(cands_[u].n16) : nullptr;
      fam->bind(cands_[u].j, cands_[u].c, cands_[u].w32, cands_[u].w16);
    }
  }
  // counter-hash initialisation (reading A21), candidates spread over host threads
  std::atomic<size_t> next{0};
  std::atomic<int> failed{0};
  const unsigned nt = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
  auto worker = [&] {
    cudaSetDevice(dev);
    std::vector<float> host;
    for (size_t k; (k = next.fetch_add(1)) < uids.size();) {
      Cand& cd = cands_[uids[k]];
      const int b = uids[k] / n_;
      if (managed()) {
        spec.init_params(b, cd.c, cd.stash);
      } else {
        host.resize(cd.n32);
        spec.init_params(b, cd.c, host.data());
        if (cudaMemcpy(cd.w32, host.data(), cd.n32 * 4, cudaMemcpyHostToDevice) != cudaSuccess) failed = 1;
      }
    }
  };
  std::vector<std::thread> threads;
  for (unsigned i = 0; i < nt; ++i) threads.emplace_back(worker);
  for (auto& t : threads) t.join();
  NP_REQUIRE(!failed, NASPIPE_ECUDA, "initial parameter upload failed");
  if (!managed()) {
    for (int u : uids) fam->refresh_shadow(cands_[u].j, cands_[u].c, 0);
    CU(cudaDeviceSynchronize());
  }
}

CandidateStore::~CandidateStore() {
  cudaSetDevice(dev_);
  if (evict_) cudaStreamSynchronize(evict_);
  if (wb_) cudaStreamSynchronize(wb_);  // write-backs into the stash have landed
  for (auto& cd : cands_) {
    if (cd.stash) cudaFreeHost(cd.stash);
    if (managed() && cd.w32) cudaFreeAsync(cd.w32, evict_);
    if (managed() && cd.w16) cudaFreeAsync(cd.w16, evict_);
    if (cd.ready) cudaEventDestroy(cd.ready);
    if (cd.last_use) cudaEventDestroy(cd.last_use);
    if (cd.wb_done) cudaEventDestroy(cd.wb_done);
    if (cd.h2d_done) cudaEventDestroy(cd.h2d_done);
  }
  if (evict_) {
    cudaStreamSynchronize(evict_);
    cudaStreamDestroy(evict_);
  }
  if (pool_) cudaMemPoolDestroy(pool_);
  if (shadow_) {
    cudaStreamSynchronize(shadow_);
    cudaStreamDestroy(shadow_);
  }
  if (wb_) {
    cudaStreamSynchronize(wb_);
    cudaStreamDestroy(wb_);
  }
  for (int i = 0; i < kStage; ++i) {
    if (stage_[i]) cudaFree(stage_[i]);
    if (stage_free_[i]) cudaEventDestroy(stage_free_[i]);
    if (staged_[i]) cudaEventDestroy(staged_[i]);
  }
}

std::vector<int64_t> CandidateStore::task_uids(const Task& t) const {
  std::vector<int64_t> u;
  for (int b : planner_.blocks_of(K_)) u.push_back(uid_of(b, planner_.choice(t.y, b)));
  std::sort(u.begin(), u.end());
  return u;
}

void CandidateStore::push_task(const Task& t) {
  if (managed()) belady_->push_task(task_uids(t), t.kind);
}
void CandidateStore::set_final() {
  if (managed()) belady_->set_final();
}
bool CandidateStore::ready() const { return !managed() || belady_->can_decide(); }

void CandidateStore::load(Cand& cd, cudaStream_t copy) {
  CU(cudaStreamWaitEvent(copy, cd.wb_done, 0));  // a reload reads the written-back stash
  CU(cudaMallocFromPoolAsync(reinterpret_cast<void**>(&cd.w32), cd.n32 * 4, pool_, copy));
  if (cd.n16) CU(cudaMallocFromPoolAsync(reinterpret_cast<void**>(&cd.w16), cd.n16 * 2, pool_, copy));
  CU(cudaMemcpyAsync(cd.w32, cd.stash, cd.n32 * 4, cudaMemcpyHostToDevice, copy));
  fam_->bind(cd.j, cd.c, cd.w32, cd.w16);
  // the bf16 shadow is a kernel: on its own stream, so the copy stream's next H2D does not
  // queue behind it while the compute stream holds the SMs
  CU(cudaEventRecord(cd.h2d_done, copy));
  CU(cudaStreamWaitEvent(shadow_, cd.h2d_done, 0));
  fam_->refresh_shadow(cd.j, cd.c, shadow_);
  CU(cudaEventRecord(cd.ready, shadow_));
  h2d_bytes += 4.0 * cd.n32;
  ++loads;
}

void CandidateStore::evict(Cand& cd, bool writeback, cudaStream_t) {
  CU(cudaStreamWaitEvent(evict_, cd.last_use, 0));  // the last task reading/updating it is done
  CU(cudaStreamWaitEvent(evict_, cd.ready, 0));     // (and its load finished)
  if (writeback) {
    const int k = stage_next_++ % kStage;
    if (stage_used_[k]) CU(cudaStreamWaitEvent(evict_, stage_free_[k], 0));  // slot's previous D2H done
    CU(cudaMemcpyAsync(stage_[k], cd.w32, cd.n32 * 4, cudaMemcpyDeviceToDevice, evict_));
    CU(cudaEventRecord(staged_[k], evict_));
    CU(cudaStreamWaitEvent(wb_, staged_[k], 0));
    CU(cudaMemcpyAsync(cd.stash, stage_[k], cd.n32 * 4, cudaMemcpyDeviceToHost, wb_));
    CU(cudaEventRecord(stage_free_[k], wb_));
    CU(cudaEventRecord(cd.wb_done, wb_));
    stage_used_[k] = true;
    d2h_bytes += 4.0 * cd.n32;
    ++writebacks;
  } else {
    CU(cudaEventRecord(cd.wb_done, evict_));
  }
  CU(cudaFreeAsync(cd.w32, evict_));
  if (cd.w16) CU(cudaFreeAsync(cd.w16, evict_));
  cd.w32 = nullptr;
  cd.w16 = nullptr;
  fam_->bind(cd.j, cd.c, nullptr, nullptr);
  ++evicts;
}

void CandidateStore::before_task(const Task& t, cudaStream_t comp, cudaStream_t copy) {
  if (!managed()) return;
  std::vector<ResidencyEvent> ev;
  std::vector<std::pair<int64_t, int64_t>> wb;
  belady_->decide_next(ev, wb);
  for (const auto& e : ev) {
    Cand& cd = cands_[e.uid];
    if (e.op == 1) {
      const bool dirty = std::any_of(wb.begin(), wb.end(), [&](const auto& w) { return w.second == e.uid; });
      evict(cd, dirty, copy);
    } else {
      load(cd, copy);
    }
    log.push_back(e);
  }
  for (int64_t u : task_uids(t)) {
    NP_REQUIRE(cands_[u].w32 != nullptr, NASPIPE_EINTERNAL, "candidate %lld not resident at its task", (long long)u);
    CU(cudaStreamWaitEvent(comp, cands_[u].ready, 0));
  }
}

void CandidateStore::enable_bsp(DevArena* arena) {
  NP_REQUIRE(!managed(), NASPIPE_EINVAL, "BSP needs every candidate resident");
  CU(cudaSetDevice(dev_));
  for (auto& cd : cands_) {
    if (cd.j < 0) continue;
    cd.acc = arena->alloc<float>(cd.n32);
    CU(cudaMemcpy(cd.acc, cd.w32, cd.n32 * 4, cudaMemcpyDeviceToDevice));
    fam_->bind_update(cd.j, cd.c, cd.acc);
  }
  bsp_ = true;
}

void CandidateStore::bsp_flush(cudaStream_t s) {
  for (auto& cd : cands_) {
    if (!cd.dirty) continue;
    CU(cudaMemcpyAsync(cd.w32, cd.acc, cd.n32 * 4, cudaMemcpyDeviceToDevice, s));
    fam_->refresh_shadow(cd.j, cd.c, s);
    cd.dirty = false;
  }
}

void CandidateStore::after_task(const Task& t, cudaStream_t comp) {
  if (bsp_ && t.kind == 1)
    for (int64_t u : task_uids(t)) cands_[u].dirty = true;
  if (!managed()) return;
  for (int64_t u : task_uids(t)) CU(cudaEventRecord(cands_[u].last_use, comp));
}

void CandidateStore::sync() {
  if (evict_) CU(cudaStreamSynchronize(evict_));
  if (wb_) CU(cudaStreamSynchronize(wb_));
  if (shadow_) CU(cudaStreamSynchronize(shadow_));
}

void CandidateStore::get(int b, int c, float* dst) {
  Cand& cd = cands_[uid_of(b, c)];
  CU(cudaSetDevice(dev_));
  if (cd.w32) CU(cudaMemcpy(dst, cd.w32, cd.n32 * 4, cudaMemcpyDeviceToHost));
  else std::memcpy(dst, cd.stash, cd.n32 * 4);
}

void CandidateStore::set(int b, int c, const float* src, cudaStream_t s) {
  Cand& cd = cands_[uid_of(b, c)];
  CU(cudaSetDevice(dev_));
  if (cd.stash) std::memcpy(cd.stash, src, cd.n32 * 4);
  if (cd.acc) CU(cudaMemcpy(cd.acc, src, cd.n32 * 4, cudaMemcpyHostToDevice));
  if (cd.w32) {
    CU(cudaMemcpy(cd.w32, src, cd.n32 * 4, cudaMemcpyHostToDevice));
    fam_->refresh_shadow(cd.j, cd.c, s);
    CU(cudaStreamSynchronize(s));
  }
}

}  // namespace naspipe
