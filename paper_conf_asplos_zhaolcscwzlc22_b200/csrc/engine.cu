// Stage executor (see engine.h).  The host walks the CSP plan in tick order and enqueues
// every task on its stage's compute stream; cross-stage dependencies are CUDA events
// (single process) or NCCL send/recv on dedicated per-direction channels (multi-process),
// so execution follows the plan exactly while the devices run asynchronously.
#include <dlfcn.h>
#include <nccl.h>

#include <unistd.h>

#include <algorithm>
#include <cstring>

#include "engine.h"

#include <chrono>
#include <set>
#include <thread>
#include "launch.h"
#include "mirror.h"

namespace naspipe {

#define CU(call)                                                                                 \
  do {                                                                                           \
    cudaError_t e_ = (call);                                                                     \
    NP_REQUIRE(e_ == cudaSuccess, NASPIPE_ECUDA, "%s: %s", #call, cudaGetErrorString(e_));       \
  } while (0)

// ------------------------------------------------------------------------------ NCCL (dlopen)
namespace {
struct NcclApi {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi& nccl() {
  static NcclApi api;
  static bool tried = false;
  if (!tried) {
    tried = true;
    const char* env = getenv("NASPIPE_NCCL_LIB");
    const char* names[] = {env ? env : "libnccl.so.2", "libnccl.so.2", "libnccl.so"};
    for (const char* n : names) {
      api.h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
      if (api.h) break;
    }
    if (api.h) {
      api.GetUniqueId = (decltype(api.GetUniqueId))dlsym(api.h, "ncclGetUniqueId");
      api.CommInitRank = (decltype(api.CommInitRank))dlsym(api.h, "ncclCommInitRank");
      api.CommDestroy = (decltype(api.CommDestroy))dlsym(api.h, "ncclCommDestroy");
      api.Send = (decltype(api.Send))dlsym(api.h, "ncclSend");
      api.Recv = (decltype(api.Recv))dlsym(api.h, "ncclRecv");
      api.GroupStart = (decltype(api.GroupStart))dlsym(api.h, "ncclGroupStart");
      api.GroupEnd = (decltype(api.GroupEnd))dlsym(api.h, "ncclGroupEnd");
      api.GetErrorString = (decltype(api.GetErrorString))dlsym(api.h, "ncclGetErrorString");
    }
  }
  NP_REQUIRE(api.h && api.Send && api.Recv && api.CommInitRank, NASPIPE_ENCCL, "libnccl.so.2 not loadable");
  return api;
}
#define NC(call)                                                                                     \
  do {                                                                                               \
    ncclResult_t r_ = (call);                                                                        \
    NP_REQUIRE(r_ == ncclSuccess, NASPIPE_ENCCL, "%s: %s", #call, nccl().GetErrorString(r_));        \
  } while (0)
}  // namespace

int nccl_unique_id(void* out) {
  ncclUniqueId id;
  NC(nccl().GetUniqueId(&id));
  std::memcpy(out, &id, sizeof id);
  return 0;
}

// Per-rank NCCL channels: activation K-1 -> K (recv) and K -> K+1 (send); gradient K+1 -> K
// (recv) and K -> K-1 (send).  Each channel is a 2-rank communicator (sender = rank 0) used
// on its own stream, so the two directions never serialise behind each other.
struct Transport {
  ncclComm_t act_in = nullptr, act_out = nullptr, grad_in = nullptr, grad_out = nullptr;
  cudaStream_t s_act_in, s_act_out, s_grad_in, s_grad_out;
  std::vector<cudaEvent_t> ev_act_rx, ev_grad_rx, ev_act_tx, ev_grad_tx;  // per slot
  ~Transport() {
    for (ncclComm_t c : {act_in, act_out, grad_in, grad_out})
      if (c) nccl().CommDestroy(c);
  }
};

// ------------------------------------------------------------------------------ construction
// Slots: every in-flight subnet lies in [wm0, wm0 + W) under CSP / INORDER / ASP (reading A7);
// under BSP the planner releases a whole bulk regardless of W (the bulk opens after the
// previous one finished on stage 0, i.e. everywhere), so in-flight ids lie in one bulk and the
// ring needs max(W, G) slots — with W slots, F(y + W) would overwrite y's stash before B(y).
static int slot_count(const Spec& s, int D) {
  return s.raw.sync_policy == NASPIPE_SYNC_BSP ? std::max(s.window(D), s.bulk(D)) : s.window(D);
}

Engine::Engine(const Spec& spec, int D) : spec_(spec), D_(D), W_(slot_count(spec, D)), planner_(spec_, D) {
  NP_REQUIRE(spec_.raw.sync_policy != NASPIPE_SYNC_BSP || spec_.raw.hbm_weight_budget_bytes == 0, NASPIPE_EINVAL,
             "BSP runs with every candidate resident (hbm_weight_budget_bytes = 0)");
  version_.assign((size_t)spec_.m() * spec_.n(), 0);
  timer_.on = (spec_.raw.flags & NASPIPE_FLAG_TIMING) != 0;
  if (spec_.raw.hbm_weight_budget_bytes > 0) suppress_pdl();  // context switching: no PDL (launch.h)
}

void Engine::suppress_pdl() {
  if (suppress_pdl_) return;
  pdl_suppressors().fetch_add(1);
  suppress_pdl_ = true;
}

std::unique_ptr<Engine> Engine::create_local(const Spec& spec, int D) {
  spec.validate_stages(D);
  int ndev = 0, cur = 0;
  CU(cudaGetDeviceCount(&ndev));
  NP_REQUIRE(ndev >= 1, NASPIPE_ECUDA, "no CUDA device");
  CU(cudaGetDevice(&cur));
  const bool mirror = (spec.raw.flags & NASPIPE_FLAG_MIRROR) != 0;
  NP_REQUIRE(!mirror || (spec.raw.sync_policy == NASPIPE_SYNC_CSP && spec.raw.bwd_policy == 0 &&
                         spec.raw.hbm_weight_budget_bytes == 0 && !(spec.raw.flags & NASPIPE_FLAG_RECOMPUTE)),
             NASPIPE_EINVAL, "layer mirroring: CSP, strict backward-first, all candidates resident, no recompute");
  const bool timed = (spec.raw.flags & NASPIPE_FLAG_TIMED) != 0;
  NP_REQUIRE(!timed || (spec.raw.sync_policy == NASPIPE_SYNC_CSP && spec.raw.bwd_policy == 0 &&
                        spec.raw.hbm_weight_budget_bytes == 0 && !mirror),
             NASPIPE_EINVAL, "timing-driven execution: CSP, strict backward-first, all candidates resident, no mirroring");
  std::unique_ptr<Engine> e(new Engine(spec, D));
  e->mirror_ = mirror;
  e->timed_ = timed;
  e->st_.resize(D);
  e->stage_sizes();
  for (int K = 0; K < D; ++K) e->setup_stage(K, (cur + K) % ndev, true);
  e->link_local_buffers();
  if (mirror) {
    const size_t nc = (size_t)spec.m() * spec.n();
    e->mwriter_.assign(nc, -1);
    e->ev_push_.resize(nc);
    for (auto& ev : e->ev_push_) CU(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    e->push_.resize(D);
    e->ev_wrote_.resize(D);
    for (int K = 0; K < D; ++K) {
      CU(cudaSetDevice(e->st_[K].dev));
      CU(cudaStreamCreateWithFlags(&e->push_[K], cudaStreamNonBlocking));
      CU(cudaEventCreateWithFlags(&e->ev_wrote_[K], cudaEventDisableTiming));
    }
  }
  if (timed) {
    e->ev_run_.resize(D);
    for (int K = 0; K < D; ++K) {
      CU(cudaSetDevice(e->st_[K].dev));
      CU(cudaEventCreateWithFlags(&e->ev_run_[K], cudaEventDisableTiming));
    }
  }
  CU(cudaSetDevice(cur));
  return e;
}

std::unique_ptr<Engine> Engine::create_rank(const Spec& spec, int D, int rank, int device, const void* ids) {
  spec.validate_stages(D);
  NP_REQUIRE(rank >= 0 && rank < D, NASPIPE_EINVAL, "stage_rank %d not in [0,%d)", rank, D);
  NP_REQUIRE(D == 1 || ids != nullptr, NASPIPE_EINVAL, "nccl_ids NULL");
  std::unique_ptr<Engine> e(new Engine(spec, D));
  e->rank_ = rank;
  // Multi-process: the compute stream waits on transport streams (NCCL) between kernels;
  // that cross-stream pattern deadlocked with PDL under context switching (launch.h), so
  // rank engines launch without PDL until a reproduction clears it.
  if (D > 1) e->suppress_pdl();
  e->st_.resize(D);
  e->stage_sizes();
  for (int K = 0; K < D; ++K) {
    e->st_[K].K = K;
    e->st_[K].dev = device;
  }
  e->setup_stage(rank, device, true);
  e->link_local_buffers();
  if (D > 1) {
    auto tx = std::make_unique<Transport>();
    CU(cudaSetDevice(device));
    for (cudaStream_t* s : {&tx->s_act_in, &tx->s_act_out, &tx->s_grad_in, &tx->s_grad_out})
      CU(cudaStreamCreateWithFlags(s, cudaStreamNonBlocking));
    for (auto* v : {&tx->ev_act_rx, &tx->ev_grad_rx, &tx->ev_act_tx, &tx->ev_grad_tx}) {
      v->resize(e->W_);
      for (auto& ev : *v) CU(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    }
    const ncclUniqueId* id = static_cast<const ncclUniqueId*>(ids);
    // channel k uses ids[2k] (activation k -> k+1, sender rank 0) and ids[2k+1]
    // (gradient k+1 -> k, sender rank 0).  Initialise channel rank-1 then channel rank: a
    // chain that cannot deadlock.
    if (rank > 0) {
      NC(nccl().GroupStart());
      NC(nccl().CommInitRank(&tx->act_in, 2, id[2 * (rank - 1)], 1));
      NC(nccl().CommInitRank(&tx->grad_out, 2, id[2 * (rank - 1) + 1], 0));
      NC(nccl().GroupEnd());
    }
    if (rank < D - 1) {
      NC(nccl().GroupStart());
      NC(nccl().CommInitRank(&tx->act_out, 2, id[2 * rank], 0));
      NC(nccl().CommInitRank(&tx->grad_in, 2, id[2 * rank + 1], 1));
      NC(nccl().GroupEnd());
    }
    e->tx_ = std::move(tx);
  }
  return e;
}

// ------------------------------------------------------------------------------ peer transport
std::unique_ptr<Engine> Engine::create_rank_peer(const Spec& spec, int D, int rank, int device) {
  spec.validate_stages(D);
  NP_REQUIRE(rank >= 0 && rank < D, NASPIPE_EINVAL, "stage_rank %d not in [0,%d)", rank, D);
  std::unique_ptr<Engine> e(new Engine(spec, D));
  e->rank_ = rank;
  // the compute stream waits on stream memory operations between kernels: no PDL across
  // them (a programmatic launch must never overtake a wait on a peer's flag)
  if (D > 1) e->suppress_pdl();
  e->peer_ = std::make_unique<PeerLink>();
  e->peer_->dev = device;
  e->st_.resize(D);
  e->stage_sizes();
  for (int K = 0; K < D; ++K) {
    e->st_[K].K = K;
    e->st_[K].dev = device;
  }
  e->setup_stage(rank, device, true);
  StageRt& st = e->st_[rank];
  PeerLink& pl = *e->peer_;
  const int W = e->W_;
  CU(cudaSetDevice(device));
  // receive rings and the flag page: plain cudaMalloc allocations (IPC-exportable)
  if (rank > 0) {
    CU(cudaMalloc(&pl.in_ring, (size_t)W * st.in_bytes));
    for (int s = 0; s < W; ++s) st.in[s] = static_cast<uint8_t*>(pl.in_ring) + (size_t)s * st.in_bytes;
  }
  if (rank < D - 1) {
    CU(cudaMalloc(&pl.gout_ring, (size_t)W * st.out_gbytes));
    for (int s = 0; s < W; ++s) st.gout[s] = static_cast<uint8_t*>(pl.gout_ring) + (size_t)s * st.out_gbytes;
  }
  CU(cudaMalloc(reinterpret_cast<void**>(&pl.flags), 2 * (size_t)W * sizeof(uint32_t)));
  CU(cudaMemset(pl.flags, 0, 2 * (size_t)W * sizeof(uint32_t)));
  CU(cudaDeviceSynchronize());
  return e;
}

void Engine::peer_export(void* dst, size_t cap, size_t* n) {
  NP_REQUIRE(peer_, NASPIPE_EINVAL, "not a peer-transport engine (naspipe_create_rank_peer)");
  NP_REQUIRE(n, NASPIPE_EINVAL, "n NULL");
  *n = sizeof(PeerBlob);
  if (!dst) return;
  NP_REQUIRE(cap >= sizeof(PeerBlob), NASPIPE_EINVAL, "blob capacity %zu < %zu", cap, sizeof(PeerBlob));
  PeerBlob b;
  std::memset(&b, 0, sizeof b);
  b.magic = PEER_BLOB_MAGIC;
  b.version = PEER_BLOB_VERSION;
  b.rank = rank_;
  b.device = peer_->dev;
  b.D = D_;
  b.W = W_;
  b.pid = (int32_t)getpid();
  const StageRt& st = st_[rank_];
  CU(cudaSetDevice(peer_->dev));
  if (peer_->in_ring) {
    b.in_slot_bytes = st.in_bytes;
    CU(cudaIpcGetMemHandle(&b.in_ring, peer_->in_ring));
  }
  if (peer_->gout_ring) {
    b.gout_slot_bytes = st.out_gbytes;
    CU(cudaIpcGetMemHandle(&b.gout_ring, peer_->gout_ring));
  }
  CU(cudaIpcGetMemHandle(&b.flags, peer_->flags));
  std::memcpy(dst, &b, sizeof b);
}

void Engine::peer_connect(const void* prev, size_t prev_n, const void* next, size_t next_n) {
  NP_REQUIRE(peer_, NASPIPE_EINVAL, "not a peer-transport engine (naspipe_create_rank_peer)");
  NP_REQUIRE(!peer_->connected, NASPIPE_ESTATE, "peer transport already connected");
  NP_REQUIRE((rank_ > 0) == (prev != nullptr) && (rank_ < D_ - 1) == (next != nullptr), NASPIPE_EINVAL,
             "rank %d of %d needs %s", rank_, D_,
             rank_ == 0 ? "no prev blob" : rank_ == D_ - 1 ? "no next blob" : "both neighbour blobs");
  PeerLink& pl = *peer_;
  StageRt& st = st_[rank_];
  CU(cudaSetDevice(pl.dev));
  auto open = [&](const cudaIpcMemHandle_t& h) {
    void* p = nullptr;
    CU(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
    pl.opened.push_back(p);
    return p;
  };
  auto check = [&](const void* blob, size_t n, int want_rank) {
    NP_REQUIRE(n >= sizeof(PeerBlob), NASPIPE_EINVAL, "peer blob of %zu bytes", n);
    PeerBlob b;
    std::memcpy(&b, blob, sizeof b);
    NP_REQUIRE(b.magic == PEER_BLOB_MAGIC && b.version == PEER_BLOB_VERSION, NASPIPE_EINVAL, "not a peer blob");
    NP_REQUIRE(b.rank == want_rank && b.D == D_ && b.W == W_, NASPIPE_EINVAL,
               "peer blob of rank %d (D %d, W %d), expected rank %d (D %d, W %d)", b.rank, b.D, b.W, want_rank, D_,
               W_);
    return b;
  };
  if (rank_ < D_ - 1) {
    const PeerBlob b = check(next, next_n, rank_ + 1);
    NP_REQUIRE(b.in_slot_bytes == st.out_bytes, NASPIPE_EINVAL, "activation slot %llu bytes, stage output %zu",
               (unsigned long long)b.in_slot_bytes, st.out_bytes);
    pl.next_in = open(b.in_ring);
    pl.next_flags = static_cast<uint32_t*>(open(b.flags));
    for (int s = 0; s < W_; ++s) st.out[s] = static_cast<uint8_t*>(pl.next_in) + (size_t)s * st.out_bytes;
  }
  if (rank_ > 0) {
    const PeerBlob b = check(prev, prev_n, rank_ - 1);
    NP_REQUIRE(b.gout_slot_bytes == st.in_gbytes, NASPIPE_EINVAL, "gradient slot %llu bytes, stage input grad %zu",
               (unsigned long long)b.gout_slot_bytes, st.in_gbytes);
    pl.prev_gout = open(b.gout_ring);
    pl.prev_flags = static_cast<uint32_t*>(open(b.flags));
    for (int s = 0; s < W_; ++s) st.gin[s] = static_cast<uint8_t*>(pl.prev_gout) + (size_t)s * st.in_gbytes;
  }
  pl.connected = true;
}

// Boundary tensor sizes of every stage (also of the non-local ones: a rank posts receives
// sized by its neighbours' outputs).
void Engine::stage_sizes() {
  if (spec_.raw.flags & NASPIPE_FLAG_MIRROR) {  // a stage boundary may fall at any block boundary
    size_t a = 0, g = 0;
    for (int b = 1; b < spec_.m(); ++b) {
      a = std::max(a, spec_.act_bytes(b));
      g = std::max(g, spec_.grad_bytes(b));
    }
    for (int K = 0; K < D_; ++K) {
      st_[K].in_bytes = K == 0 ? spec_.input_bytes() : a;
      st_[K].out_bytes = K == D_ - 1 ? spec_.act_bytes(spec_.m()) : a;
      st_[K].in_gbytes = K == 0 ? spec_.grad_bytes(0) : g;
      st_[K].out_gbytes = K == D_ - 1 ? spec_.grad_bytes(spec_.m()) : g;
    }
    return;
  }
  for (int K = 0; K < D_; ++K) {
    const auto& bl = planner_.blocks_of(K);
    st_[K].in_bytes = K == 0 ? spec_.input_bytes() : spec_.act_bytes(bl.front());
    st_[K].out_bytes = spec_.act_bytes(bl.back() + 1);
    st_[K].in_gbytes = spec_.grad_bytes(bl.front());
    st_[K].out_gbytes = spec_.grad_bytes(bl.back() + 1);
  }
}

void Engine::setup_stage(int K, int dev, bool local) {
  StageRt& st = st_[K];
  st.K = K;
  st.dev = dev;
  st.local = local;
  CU(cudaSetDevice(dev));
  CU(create_stream(&st.comp, true));
  CU(cudaStreamCreateWithFlags(&st.copy, cudaStreamNonBlocking));
  st.arena = std::make_unique<DevArena>(dev);
  std::vector<int> blocks = planner_.blocks_of(K);
  if (spec_.raw.flags & NASPIPE_FLAG_MIRROR) {  // a mirror copy of every block's candidates
    blocks.resize(spec_.m());
    for (int b = 0; b < spec_.m(); ++b) blocks[b] = b;
  }
  st.fam = make_family(spec_, blocks, W_, *st.arena, st.comp);
  st.fam->timer = &timer_;
  st.store = std::make_unique<CandidateStore>(spec_, planner_, K, dev, st.fam.get(), st.arena.get(),
                                              spec_.raw.hbm_weight_budget_bytes, blocks);
  if (spec_.raw.sync_policy == NASPIPE_SYNC_BSP) st.store->enable_bsp(st.arena.get());
  st.in.assign(W_, nullptr);
  st.gout.assign(W_, nullptr);
  st.out.resize(W_);
  st.gin.assign(W_, nullptr);
  const bool peer = peer_ != nullptr;  // peer transport: out / gin live in the neighbours' rings
  for (int s = 0; s < W_; ++s) {
    if (!peer || K == D_ - 1) st.out[s] = st.arena->alloc<uint8_t>(st.out_bytes);
    if (K > 0 && !peer) st.gin[s] = st.arena->alloc<uint8_t>(st.in_gbytes);
    if (K == 0) st.in[s] = st.arena->alloc<uint8_t>(st.in_bytes);
    if (K == D_ - 1) st.gout[s] = st.arena->alloc<uint8_t>(st.out_gbytes);
  }
  if (K == D_ - 1) {
    st.target.resize(W_);
    for (auto& p : st.target) p = st.arena->alloc<uint8_t>(spec_.target_bytes());
    st.loss = st.arena->alloc<float>(loss_cap_);
    CU(cudaMemsetAsync(st.loss, 0, loss_cap_ * sizeof(float), st.comp));
  }
  for (auto* v : {&st.ev_f, &st.ev_b, &st.ev_in, &st.ev_tgt}) {
    v->resize(W_);
    for (auto& ev : *v) CU(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  }
  CU(cudaStreamSynchronize(st.comp));
}

// Same-device neighbours share boundary buffers (zero copy); otherwise each side owns a
// receive buffer filled by a peer copy (single process) or NCCL (multi-process).
void Engine::link_local_buffers() {
  for (int K = 0; K < D_; ++K) {
    StageRt& st = st_[K];
    if (!st.local) continue;
    CU(cudaSetDevice(st.dev));
    for (int s = 0; s < W_; ++s) {
      if (K > 0) {
        const StageRt& p = st_[K - 1];
        st.in[s] = (p.local && p.dev == st.dev) ? p.out[s] : st.arena->alloc<uint8_t>(st.in_bytes);
      }
      if (K < D_ - 1) {
        const StageRt& q = st_[K + 1];
        st.gout[s] = (q.local && q.dev == st.dev) ? q.gin[s] : st.arena->alloc<uint8_t>(st.out_gbytes);
      }
    }
  }
}

Engine::~Engine() {
  shutdown();
  if (suppress_pdl_) pdl_suppressors().fetch_sub(1);
}

void Engine::shutdown() {
  for (auto& st : st_) {
    if (!st.local || !st.comp) continue;
    cudaSetDevice(st.dev);
    cudaStreamSynchronize(st.comp);
    cudaStreamSynchronize(st.copy);
  }
  if (tx_) {
    for (cudaStream_t s : {tx_->s_act_in, tx_->s_act_out, tx_->s_grad_in, tx_->s_grad_out}) cudaStreamSynchronize(s);
  }
  tx_.reset();
  peer_.reset();
  for (cudaStream_t s : push_) cudaStreamSynchronize(s);
  for (cudaStream_t s : push_) cudaStreamDestroy(s);
  for (cudaEvent_t ev : ev_push_) cudaEventDestroy(ev);
  for (cudaEvent_t ev : ev_wrote_) cudaEventDestroy(ev);
  push_.clear();
  ev_push_.clear();
  ev_wrote_.clear();
  for (auto& st : st_) {
    if (!st.local || !st.comp) continue;
    cudaSetDevice(st.dev);
    st.store.reset();
    st.fam.reset();
    st.arena.reset();
    for (auto* v : {&st.ev_f, &st.ev_b, &st.ev_in, &st.ev_tgt})
      for (auto ev : *v) cudaEventDestroy(ev);
    cudaStreamDestroy(st.comp);
    cudaStreamDestroy(st.copy);
    st.comp = st.copy = nullptr;
  }
}

void Engine::check_sticky() const {
  if (sticky_code_) throw Error(sticky_code_, "sticky error: " + sticky_msg_);
}
void Engine::set_sticky(int code, const std::string& msg) {
  if (!sticky_code_) {
    sticky_code_ = code;
    sticky_msg_ = msg;
  }
}

void Engine::cuda_check(const char* what) {
  cudaError_t e = cudaGetLastError();
  NP_REQUIRE(e == cudaSuccess, NASPIPE_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

// ------------------------------------------------------------------------------ submit / issue
int64_t Engine::submit(const int32_t* choice, const naspipe_batch* batch) {
  NP_REQUIRE(choice && batch, NASPIPE_EINVAL, "choice/batch NULL");
  NP_REQUIRE(!peer_ || peer_->connected || D_ == 1, NASPIPE_ESTATE, "peer transport not connected (naspipe_peer_connect)");
  NP_REQUIRE(batch->where >= NASPIPE_BATCH_HOST && batch->where <= NASPIPE_BATCH_SYNTHETIC, NASPIPE_EINVAL,
             "batch.where %d", batch->where);
  NP_REQUIRE(batch->where == NASPIPE_BATCH_SYNTHETIC || (batch->input && batch->target), NASPIPE_EINVAL,
             "batch input/target NULL");
  NP_REQUIRE(planner_.n_subnets() < loss_cap_, NASPIPE_EINVAL, "more than %lld subnets", (long long)loss_cap_);
  for (int b = 0; b < spec_.m(); ++b)
    NP_REQUIRE(choice[b] >= 0 && choice[b] < spec_.n(), NASPIPE_EINVAL, "choice[%d]=%d outside [0,%d)", b,
               choice[b], spec_.n());
  if (drained_) {
    if (!mirror_ && !timed_) planner_.reopen();  // those two schedule at drain, not through the plan
    drained_ = false;
  }
  const int64_t y = planner_.add_subnet(choice);
  batches_.push_back({*batch});
  if (mirror_ || timed_) return y;  // scheduled and issued at drain (drain_mirrored / drain_timed)
  planner_.advance();
  feed_stores();
  issue_planned();
  return y;
}

void Engine::drain() {
  if (!drained_ && mirror_) drain_mirrored();
  if (!drained_ && timed_) drain_timed();
  if (!drained_ && !mirror_ && !timed_) {
    planner_.finalize();
    planner_.advance();
    NP_REQUIRE(planner_.done(), NASPIPE_EINTERNAL, "planner did not finish");
    feed_stores();
    for (auto& st : st_)
      if (st.local) st.store->set_final();
    issue_planned();
    NP_REQUIRE(issued_ == planner_.tasks().size(), NASPIPE_EINTERNAL, "tasks left unissued at drain");
  }
  for (auto& st : st_) {
    if (!st.local) continue;
    CU(cudaSetDevice(st.dev));
    if (spec_.raw.sync_policy == NASPIPE_SYNC_BSP) st.store->bsp_flush(st.comp);  // the last bulk's flush
    CU(cudaStreamSynchronize(st.copy));
    CU(cudaStreamSynchronize(st.comp));
    st.store->sync();
    st.fam->check_after_drain();
  }
  if (tx_)
    for (cudaStream_t s : {tx_->s_act_in, tx_->s_act_out, tx_->s_grad_in, tx_->s_grad_out})
      CU(cudaStreamSynchronize(s));
  for (cudaStream_t s : push_) CU(cudaStreamSynchronize(s));
  cuda_check("drain");
  timer_.collect();
  drained_ = true;
}

// Append newly planned stage tasks to the local stages' candidate stores (residency plan).
void Engine::feed_stores() {
  for (auto& st : st_) {
    if (!st.local) continue;
    const auto& idx = planner_.stage_tasks()[st.K];
    for (; st.pushed < idx.size(); ++st.pushed) st.store->push_task(planner_.tasks()[idx[st.pushed]]);
  }
}

// Issue planned tasks in tick order; a local stage whose next residency decision needs more
// of the plan (reading A26's horizon) holds the issue point until more subnets arrive.
void Engine::issue_planned() {
  const auto& tasks = planner_.tasks();
  while (issued_ < tasks.size()) {
    const Task& t = tasks[issued_];
    if (st_[t.K].local && !st_[t.K].store->ready()) break;
    issue(tasks[issued_++]);
  }
}

// ------------------------------------------------------------------------------ layer mirroring
// Plan the undrained subnets [mbase_, N) with per-subnet balanced partitions (mirror.cpp,
// reading A31; mirror latency = link_latency) and issue the plan in its decision order.
void Engine::drain_mirrored() {
  const int64_t N = planner_.n_subnets(), n = N - mbase_, m = spec_.m();
  std::vector<int32_t> ch((size_t)n * m);
  for (int64_t y = 0; y < n; ++y)
    for (int b = 0; b < m; ++b) ch[y * m + b] = planner_.choice(mbase_ + y, b);
  const MirrorPlan P = plan_mirrored(spec_, D_, ch.data(), n, spec_.raw.link_latency);
  msob_.resize((size_t)N * m);
  std::copy(P.sob.begin(), P.sob.end(), msob_.begin() + mbase_ * m);
  for (Task t : P.trace) {
    t.y += mbase_;
    t.t += mticks_;
    issue_mirrored(t);
  }
  mticks_ += P.makespan;
  mbase_ = N;
  issued_ = 0;
}

void Engine::issue_mirrored(const Task& t) {
  const int slot = (int)(t.y % W_);
  const int m = spec_.m();
  StageRt& st = st_[t.K];
  int lo = m, hi = 0;
  for (int b = 0; b < m; ++b)
    if (msob_[t.y * m + b] == t.K) lo = std::min(lo, b), hi = std::max(hi, b + 1);
  NP_REQUIRE(lo < hi, NASPIPE_EINTERNAL, "subnet %lld has no block on stage %d", (long long)t.y, t.K);
  CU(cudaSetDevice(st.dev));
  for (int b = lo; b < hi; ++b) {
    const size_t key = (size_t)b * spec_.n() + planner_.choice(t.y, b);
    if (spec_.raw.flags & NASPIPE_FLAG_VERSION_CHECK) {
      NP_REQUIRE(version_[key] == planner_.version(t.y, b), NASPIPE_EINTERNAL,
                 "version check: subnet %lld stage %d block %d sees version %lld, expected %lld", (long long)t.y,
                 t.K, b, (long long)version_[key], (long long)planner_.version(t.y, b));
      ++version_checks_;
    }
    if (t.kind == 1) version_[key] += 1;
    // the READ (forward) / READ + WRITE (backward) of a candidate last written on another
    // stage waits for the push of that WRITE into this stage's mirror copy
    if (mwriter_[key] >= 0 && mwriter_[key] != t.K) CU(cudaStreamWaitEvent(st.comp, ev_push_[key], 0));
  }
  if (spec_.raw.flags & NASPIPE_FLAG_TRACE) trace_.push_back(t);
  st.fam->set_range(lo, hi);
  if (t.kind == 0) issue_forward(st, t.y, slot);
  else issue_backward(st, t.y, slot);
  ++issued_;
  if (t.kind != 1) return;
  // push the WRITE (fp32 master + bf16 shadow) of every candidate of this task to the other
  // stages' mirror copies, on this stage's push stream once the backward is done
  CU(cudaEventRecord(ev_wrote_[t.K], st.comp));
  CU(cudaStreamWaitEvent(push_[t.K], ev_wrote_[t.K], 0));
  for (int b = lo; b < hi; ++b) {
    const int c = planner_.choice(t.y, b);
    const size_t key = (size_t)b * spec_.n() + c;
    CandidateStore& src = *st.store;
    for (int K2 = 0; K2 < D_; ++K2) {
      if (K2 == t.K) continue;
      CandidateStore& dst = *st_[K2].store;
      CU(cudaMemcpyPeerAsync(dst.dev_master(b, c), st_[K2].dev, src.dev_master(b, c), st.dev, src.n32(b, c) * 4,
                             push_[t.K]));
      if (src.n16(b, c))
        CU(cudaMemcpyPeerAsync(dst.dev_shadow(b, c), st_[K2].dev, src.dev_shadow(b, c), st.dev, src.n16(b, c) * 2,
                               push_[t.K]));
      p2p_bytes_ += 4.0 * src.n32(b, c) + 2.0 * src.n16(b, c);
    }
    CU(cudaEventRecord(ev_push_[key], push_[t.K]));
    mwriter_[key] = t.K;
  }
}

// ------------------------------------------------------------------------------ timing-driven execution
// Alg.1 + Alg.2 on observed completions (NASPIPE_FLAG_TIMED, reading A39): the
// host keeps, per stage, the forward queue (input arrived), the backward queue (output
// gradient arrived) and the finished set, learns of completions by polling each stage's
// running task, and gives a free stage its next task at once: the lowest-id queued backward,
// else the lowest-id queued forward admissible under Def.2 (every block's previous user
// dep[y][b] has finished its backward, i.e. its WRITE, on this stage).  Stage 0 admits y <
// (lowest id unfinished on stage 0) + W (reading A7).  Alg.3 (its backward
// branch, reading A10): when B(x, K) starts, Alg.2 over K's queue with x counted finished
// predicts the forward K runs next (the context to prefetch); it is scored against what K
// actually runs next.  Every realised order is a CSP schedule, so the numerics are those of
// the planned executor, bitwise.
void Engine::drain_timed() {
  const int64_t N = planner_.n_subnets(), base = tbase_;
  if (N == base) return;
  const auto t0 = std::chrono::steady_clock::now();
  auto us_now = [&] {
    return (int64_t)std::chrono::duration_cast<std::chrono::microseconds>(std::chrono::steady_clock::now() - t0).count();
  };
  std::vector<std::set<int64_t>> fq(D_), bq(D_);
  std::vector<std::vector<uint8_t>> fin(D_, std::vector<uint8_t>((size_t)(N - base), 0));
  std::vector<int64_t> wm(D_, base);  // lowest id not finished on stage K
  struct Run {
    bool on = false;
    int kind = 0;
    int64_t y = 0;
  };
  std::vector<Run> run(D_);
  std::vector<int64_t> pred(D_, -1);     // pending Alg.3 prediction per stage (-1: none)
  std::vector<uint8_t> pending(D_, 0);   // a backward started and K has not run its next task yet
  auto finished = [&](int K, int64_t x, int64_t extra) { return x < base || x == extra || fin[K][x - base]; };
  auto admissible = [&](int K, int64_t y, int64_t extra) {
    for (int b : planner_.blocks_of(K))
      if (!finished(K, planner_.dep(y, b), extra)) return false;
    return true;
  };
  int64_t next_src = base, done = 0;
  const int64_t total = 2 * (N - base) * D_;
  while (done < total) {
    bool progress = false;
    for (int K = 0; K < D_; ++K) {  // completions
      if (!run[K].on) continue;
      const cudaError_t q = cudaEventQuery(ev_run_[K]);
      if (q == cudaErrorNotReady) continue;
      CU(q);
      const int64_t y = run[K].y;
      if (run[K].kind == 0) {
        if (K < D_ - 1) fq[K + 1].insert(y);
        else bq[K].insert(y);  // the loss ran inside F(y, D-1)
      } else {
        fin[K][y - base] = 1;
        while (wm[K] < N && fin[K][wm[K] - base]) ++wm[K];
        if (K > 0) bq[K - 1].insert(y);
      }
      run[K].on = false;
      ++done;
      progress = true;
    }
    while (next_src < N && next_src < wm[0] + W_) fq[0].insert(next_src++);  // stage-0 window
    for (int K = 0; K < D_; ++K) {  // decisions of the free stages
      if (run[K].on) continue;
      Task t{0, K, -1, 0};
      if (!bq[K].empty()) {
        t.kind = 1;
        t.y = *bq[K].begin();
        bq[K].erase(bq[K].begin());
      } else {
        for (int64_t y : fq[K])
          if (admissible(K, y, -1)) {
            t.kind = 0;
            t.y = y;
            break;
          }
        if (t.kind == 0) fq[K].erase(t.y);
      }
      if (t.kind < 0) continue;
      if (pending[K]) {  // score the prediction made at the previous backward's start
        if (pred[K] >= 0 && t.kind == 0 && t.y == pred[K]) tstat_[3] += 1;
        pending[K] = 0;
      }
      if (t.kind == 1) {  // Alg.3: predict K's next forward with t.y counted finished
        tstat_[1] += 1;
        pred[K] = -1;
        for (int64_t y : fq[K])
          if (admissible(K, y, t.y)) {
            pred[K] = y;
            break;
          }
        if (pred[K] >= 0) tstat_[2] += 1;
        pending[K] = 1;
      }
      t.t = us_now();
      issue(t);
      ++issued_;
      CU(cudaSetDevice(st_[K].dev));
      CU(cudaEventRecord(ev_run_[K], st_[K].comp));
      run[K] = {true, t.kind, t.y};
      tstat_[0] += 1;
      progress = true;
    }
    if (!progress) std::this_thread::yield();
  }
  tstat_[4] += (double)us_now() / 1e3;
  tbase_ = N;
  issued_ = 0;
}

void Engine::get_timed_stats(double* o) {
  NP_REQUIRE(o, NASPIPE_EINVAL, "dst NULL");
  std::copy(tstat_, tstat_ + 6, o);
}

void Engine::version_check(const Task& t) {
  // Expected version of candidate (b, c_y[b]) at any task of y = #{x < y : c_x[b] == c_y[b]}
  // (SURVEY §8c "version invariant"); the backward's update makes it v + 1.
  for (int b : planner_.blocks_of(t.K)) {
    const size_t key = (size_t)b * spec_.n() + planner_.choice(t.y, b);
    NP_REQUIRE(version_[key] == planner_.version(t.y, b), NASPIPE_EINTERNAL,
               "version check: subnet %lld stage %d block %d sees version %lld, expected %lld", (long long)t.y, t.K,
               b, (long long)version_[key], (long long)planner_.version(t.y, b));
    ++version_checks_;
    if (t.kind == 1) version_[key] += 1;
  }
}

void Engine::issue(const Task& t) {
  const int slot = (int)(t.y % W_);
  StageRt& st = st_[t.K];
  if (rank_ >= 0 && tx_) {
    // multi-process: post receives for the neighbours' tasks in their plan order (the sends
    // follow the same rules inside issue_forward / issue_backward; see comm_ops)
    StageRt& me = st_[rank_];
    CommStep ops[2];
    const int nops = comm_ops(t, rank_, D_, ops);
    for (int k = 0; k < nops; ++k) {
      if (ops[k].op == RECV_ACT) {
        CU(cudaSetDevice(me.dev));
        CU(cudaStreamWaitEvent(tx_->s_act_in, me.ev_b[slot], 0));  // slot free (B(y-W) done)
        NC(nccl().Recv(me.in[slot], me.in_bytes, ncclUint8, 0, tx_->act_in, tx_->s_act_in));
        CU(cudaEventRecord(tx_->ev_act_rx[slot], tx_->s_act_in));
        p2p_bytes_ += (double)me.in_bytes;
      } else if (ops[k].op == RECV_GRAD) {
        CU(cudaSetDevice(me.dev));
        CU(cudaStreamWaitEvent(tx_->s_grad_in, me.ev_b[slot], 0));
        NC(nccl().Recv(me.gout[slot], me.out_gbytes, ncclUint8, 0, tx_->grad_in, tx_->s_grad_in));
        CU(cudaEventRecord(tx_->ev_grad_rx[slot], tx_->s_grad_in));
        p2p_bytes_ += (double)me.out_gbytes;
      }
    }
  }
  if (!st.local) return;
  // the version invariant is CSP's (and INORDER's); ASP reads whatever version is current
  if ((spec_.raw.flags & NASPIPE_FLAG_VERSION_CHECK) && spec_.raw.sync_policy != NASPIPE_SYNC_ASP &&
      spec_.raw.sync_policy != NASPIPE_SYNC_BSP)
    version_check(t);
  if (spec_.raw.flags & NASPIPE_FLAG_TRACE) trace_.push_back(t);
  CU(cudaSetDevice(st.dev));
  if (spec_.raw.sync_policy == NASPIPE_SYNC_BSP) {
    // BSP flush (reading A30): the first task of a new bulk on this stage runs after every
    // task of the previous bulk (the plan's flush; same stream), so the accumulated WRITEs
    // become the masters the new bulk reads
    const int64_t bulk = t.y / spec_.bulk(D_);
    if (bulk != st.bulk) st.store->bsp_flush(st.comp);
    st.bulk = bulk;
  }
  st.store->before_task(t, st.comp, st.copy);  // context switch: LOAD/EVICT, wait for this task's candidates
  if (t.kind == 0) issue_forward(st, t.y, slot);
  else issue_backward(st, t.y, slot);
  st.store->after_task(t, st.comp);
}

void Engine::issue_forward(StageRt& st, int64_t y, int slot) {
  const int K = st.K;
  const naspipe_batch& bt = batches_[y].b;
  const bool null_k = (spec_.raw.flags & NASPIPE_FLAG_NULL_KERNELS) != 0;
  const void* xin = nullptr;
  if (K == 0) {
    const size_t nb = spec_.input_bytes();
    if (bt.where == NASPIPE_BATCH_HOST) {
      CU(cudaStreamWaitEvent(st.copy, st.ev_b[slot], 0));
      CU(cudaMemcpyAsync(st.in[slot], bt.input, nb, cudaMemcpyHostToDevice, st.copy));
      CU(cudaEventRecord(st.ev_in[slot], st.copy));
      CU(cudaStreamWaitEvent(st.comp, st.ev_in[slot], 0));
      h2d_bytes_ += (double)nb;
      xin = st.in[slot];
    } else if (bt.where == NASPIPE_BATCH_DEVICE) {
      xin = bt.input;
    } else {
      if (!null_k) { synth_fill(st.comp, static_cast<float*>(st.in[slot]), nb / 4, bt.synth_seed * 2 + 0); ++engine_launches_; }
      xin = st.in[slot];
    }
  } else if (rank_ < 0) {
    StageRt& p = st_[K - 1];
    CU(cudaStreamWaitEvent(st.comp, p.ev_f[slot], 0));
    if (p.dev != st.dev) {
      CU(cudaMemcpyPeerAsync(st.in[slot], st.dev, p.out[slot], p.dev, st.in_bytes, st.comp));
      p2p_bytes_ += (double)st.in_bytes;
    }
    xin = st.in[slot];
  } else if (peer_) {
    stream_wait_geq(st.comp, peer_->flags + slot, (uint32_t)(y + 1));  // F(y, K-1) wrote in[slot]
    xin = st.in[slot];
  } else {
    CU(cudaStreamWaitEvent(st.comp, tx_->ev_act_rx[slot], 0));
    xin = st.in[slot];
  }
  const void* tgt = nullptr;
  if (K == D_ - 1) {
    const size_t tb = spec_.target_bytes();
    if (bt.where == NASPIPE_BATCH_HOST) {
      CU(cudaStreamWaitEvent(st.copy, st.ev_f[slot], 0));  // previous user's loss done
      CU(cudaMemcpyAsync(st.target[slot], bt.target, tb, cudaMemcpyHostToDevice, st.copy));
      CU(cudaEventRecord(st.ev_tgt[slot], st.copy));
      h2d_bytes_ += (double)tb;
      tgt = st.target[slot];
    } else if (bt.where == NASPIPE_BATCH_DEVICE) {
      tgt = bt.target;
    } else {
      if (!null_k) { st.fam->synth_target(st.target[slot], bt.synth_seed * 2 + 1, st.comp); ++engine_launches_; }
      tgt = st.target[slot];
    }
  }
  if (rank_ >= 0 && tx_ && K < D_ - 1)  // out[slot] free once the previous send left
    CU(cudaStreamWaitEvent(st.comp, tx_->ev_act_tx[slot], 0));
  // stage forward: the candidates chosen by y in this stage's blocks
  if (!null_k) st.fam->forward(slot, planner_.choice_row(y), xin, st.out[slot], st.comp);
  if (K == D_ - 1) {
    if (bt.where == NASPIPE_BATCH_HOST) CU(cudaStreamWaitEvent(st.comp, st.ev_tgt[slot], 0));
    if (!null_k) st.fam->loss(slot, st.out[slot], tgt, st.gout[slot], st.loss + y, st.comp);
  }
  CU(cudaEventRecord(st.ev_f[slot], st.comp));
  if (peer_ && K < D_ - 1) {  // the forward wrote rank K+1's in[slot]: publish it
    stream_write(st.comp, peer_->next_flags + slot, (uint32_t)(y + 1));
    p2p_bytes_ += (double)st.out_bytes;
  }
  if (rank_ >= 0 && tx_ && K < D_ - 1) {
    CU(cudaStreamWaitEvent(tx_->s_act_out, st.ev_f[slot], 0));
    NC(nccl().Send(st.out[slot], st.out_bytes, ncclUint8, 1, tx_->act_out, tx_->s_act_out));
    CU(cudaEventRecord(tx_->ev_act_tx[slot], tx_->s_act_out));
  }
  cuda_check("forward");
}

void Engine::issue_backward(StageRt& st, int64_t y, int slot) {
  const int K = st.K;
  const bool null_k = (spec_.raw.flags & NASPIPE_FLAG_NULL_KERNELS) != 0;
  if (K < D_ - 1) {
    if (rank_ < 0) {
      StageRt& q = st_[K + 1];
      CU(cudaStreamWaitEvent(st.comp, q.ev_b[slot], 0));
      if (q.dev != st.dev) {
        CU(cudaMemcpyPeerAsync(st.gout[slot], st.dev, q.gin[slot], q.dev, st.out_gbytes, st.comp));
        p2p_bytes_ += (double)st.out_gbytes;
      }
    } else if (peer_) {
      stream_wait_geq(st.comp, peer_->flags + W_ + slot, (uint32_t)(y + 1));  // B(y, K+1) wrote gout[slot]
    } else {
      CU(cudaStreamWaitEvent(st.comp, tx_->ev_grad_rx[slot], 0));
    }
  }
  if (rank_ >= 0 && tx_ && K > 0) CU(cudaStreamWaitEvent(st.comp, tx_->ev_grad_tx[slot], 0));
  void* dx = K > 0 ? st.gin[slot] : nullptr;
  if (!null_k) st.fam->backward(slot, planner_.choice_row(y), st.gout[slot], dx, st.comp);
  CU(cudaEventRecord(st.ev_b[slot], st.comp));
  if (peer_ && K > 0) {  // the backward wrote rank K-1's gout[slot]: publish it
    stream_write(st.comp, peer_->prev_flags + W_ + slot, (uint32_t)(y + 1));
    p2p_bytes_ += (double)st.in_gbytes;
  }
  if (rank_ >= 0 && tx_ && K > 0) {
    CU(cudaStreamWaitEvent(tx_->s_grad_out, st.ev_b[slot], 0));
    NC(nccl().Send(st.gin[slot], st.in_gbytes, ncclUint8, 0, tx_->grad_out, tx_->s_grad_out));
    CU(cudaEventRecord(tx_->ev_grad_tx[slot], tx_->s_grad_out));
  }
  cuda_check("backward");
}

// ------------------------------------------------------------------------------ read-out
void Engine::get_params(int block, int choice, float* dst, size_t n) {
  NP_REQUIRE(block >= 0 && block < spec_.m() && choice >= 0 && choice < spec_.n(), NASPIPE_EINVAL,
             "candidate (%d,%d) out of range", block, choice);
  NP_REQUIRE(dst && n == spec_.param_count(block, choice), NASPIPE_EINVAL, "n_floats %zu != %zu", n,
             spec_.param_count(block, choice));
  NP_REQUIRE(drained_ || planner_.n_subnets() == 0, NASPIPE_ESTATE, "get_params before naspipe_drain");
  // (mirroring: after a drain every mirror copy holds the last WRITE; read stage 0's)
  const int K = mirror_ ? 0 : planner_.stage_of_block()[block];
  StageRt& st = st_[K];
  NP_REQUIRE(st.local, NASPIPE_EINVAL, "block %d lives on stage %d, not on this rank", block, K);
  st.store->get(block, choice, dst);
  d2h_bytes_ += 4.0 * n;
}

void Engine::set_params(int block, int choice, const float* src, size_t n) {
  NP_REQUIRE(block >= 0 && block < spec_.m() && choice >= 0 && choice < spec_.n(), NASPIPE_EINVAL,
             "candidate (%d,%d) out of range", block, choice);
  NP_REQUIRE(src && n == spec_.param_count(block, choice), NASPIPE_EINVAL, "n_floats %zu != %zu", n,
             spec_.param_count(block, choice));
  NP_REQUIRE(drained_ || planner_.n_subnets() == 0, NASPIPE_ESTATE, "set_params with work in flight");
  if (mirror_) {  // every stage's mirror copy
    for (auto& s2 : st_) s2.store->set(block, choice, src, s2.comp);
    return;
  }
  const int K = planner_.stage_of_block()[block];
  StageRt& st = st_[K];
  NP_REQUIRE(st.local, NASPIPE_EINVAL, "block %d lives on stage %d, not on this rank", block, K);
  st.store->set(block, choice, src, st.comp);
}

void Engine::get_losses(float* dst, int64_t n) {
  NP_REQUIRE(dst && n >= 0 && n <= planner_.n_subnets(), NASPIPE_EINVAL, "bad loss count %lld", (long long)n);
  NP_REQUIRE(drained_, NASPIPE_ESTATE, "get_losses before naspipe_drain");
  StageRt& st = st_[D_ - 1];
  NP_REQUIRE(st.local, NASPIPE_EINVAL, "losses live on the last stage's rank");
  CU(cudaSetDevice(st.dev));
  if (n) CU(cudaMemcpy(dst, st.loss, n * 4, cudaMemcpyDeviceToHost));
}

void Engine::get_trace(int64_t* dst, size_t cap, size_t* n) {
  NP_REQUIRE(n, NASPIPE_EINVAL, "n NULL");
  *n = trace_.size();
  for (size_t i = 0; i < trace_.size() && i < cap && dst; ++i) {
    dst[4 * i] = trace_[i].t;
    dst[4 * i + 1] = trace_[i].K;
    dst[4 * i + 2] = trace_[i].kind;
    dst[4 * i + 3] = trace_[i].y;
  }
}

void Engine::set_timing(bool on) {
  NP_REQUIRE(drained_ || planner_.n_subnets() == 0, NASPIPE_ESTATE, "set_timing with work in flight");
  timer_.on = on;
}

void Engine::get_stats(double* o) {
  NP_REQUIRE(o, NASPIPE_EINVAL, "dst NULL");
  std::fill(o, o + 16, 0.0);
  double launches = 0;
  for (auto& st : st_)
    if (st.local && st.fam) launches += (double)st.fam->counters.launches;
  double loads = 0, evicts = 0, wbs = 0, rh2d = 0, rd2h = 0;
  for (auto& st : st_)
    if (st.local && st.store) {
      loads += (double)st.store->loads;
      evicts += (double)st.store->evicts;
      wbs += (double)st.store->writebacks;
      rh2d += st.store->h2d_bytes;
      rd2h += st.store->d2h_bytes;
    }
  o[0] = (double)issued_;
  o[1] = launches + (double)engine_launches_;
  o[2] = h2d_bytes_ + rh2d;
  o[3] = d2h_bytes_ + rd2h;
  o[9] = loads;
  o[10] = evicts;
  o[11] = wbs;
  o[4] = p2p_bytes_;
  o[5] = mirror_ ? (double)mticks_ : (double)planner_.makespan();
  o[6] = timer_.launches;
  o[7] = timer_.flops;
  o[8] = timer_.ms;
  o[12] = (double)version_checks_;
  double fbytes = 0;
  for (auto& st : st_)
    if (st.local && st.fam) fbytes += st.fam->counters.bytes;
  o[15] = fbytes;
  o[13] = (double)gemm_flop_count();
  o[14] = (double)gemm_launch_count();
}

void Engine::get_residency_trace(int64_t* dst, size_t cap, size_t* n) {
  NP_REQUIRE(n, NASPIPE_EINVAL, "n NULL");
  size_t k = 0;
  for (auto& st : st_) {
    if (!st.local || !st.store) continue;
    for (const auto& e : st.store->log) {
      if (dst && k < cap) {
        dst[4 * k] = e.K;
        dst[4 * k + 1] = e.i;
        dst[4 * k + 2] = e.op;
        dst[4 * k + 3] = e.uid;
      }
      ++k;
    }
  }
  *n = k;
}

}  // namespace naspipe
