// Peer-memory stage-boundary transport (one process per GPU).
//
// The paper moves activations and gradients between pipeline stages with
// torch.distributed send/recv.  Here every rank exports its RECEIVE rings (stage
// input activations, W slots; gradients w.r.t. its output, W slots) and a flag page over CUDA
// IPC; its neighbours map them and their kernels write the boundary tensors straight into the
// neighbour's ring (the producing kernel's stores go over NVLink / NVSwitch, or stay in HBM
// when two ranks share a GPU): no staging copy, no send/recv pair.  A stream memory
// operation then publishes "slot s holds subnet y" (flag = y + 1) on the receiver's flag
// page; the receiver's compute stream waits for it with a front-end wait (no SM spins).
//
// Slot reuse needs no credits: the plan orders every overwrite after the previous
// occupant's consumer on the device (engine.h, DESIGN.md §5 "Transport").
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <vector>

namespace naspipe {

constexpr uint32_t PEER_BLOB_MAGIC = 0x4E505052;  // "NPPR"
constexpr uint32_t PEER_BLOB_VERSION = 1;

// What a rank exports (naspipe_peer_export); plain bytes, identical layout on every rank.
struct PeerBlob {
  uint32_t magic, version;
  int32_t rank, device, D, W, pid, pad;
  uint64_t in_slot_bytes, gout_slot_bytes;  // per-slot bytes of the exported rings (0: none)
  cudaIpcMemHandle_t in_ring, gout_ring, flags;
};

struct PeerLink {
  // local, exported: input-activation ring (rank > 0), output-gradient ring (rank < D-1),
  // flags [0, W) = activation slot ready, [W, 2W) = gradient slot ready (value = y + 1)
  void* in_ring = nullptr;
  void* gout_ring = nullptr;
  uint32_t* flags = nullptr;
  // mapped from the neighbours
  void* next_in = nullptr;         // rank + 1's input ring: this rank's stage outputs
  uint32_t* next_flags = nullptr;  // rank + 1's flag page
  void* prev_gout = nullptr;       // rank - 1's gradient ring: this rank's input gradients
  uint32_t* prev_flags = nullptr;  // rank - 1's flag page
  std::vector<void*> opened;
  bool connected = false;
  int dev = 0;
  ~PeerLink();
};

// Stream memory operations (driver API through cudaGetDriverEntryPoint): wait until
// *addr >= v (front-end wait, no SM), and write *addr = v after all prior work of the
// stream with a memory barrier (prior stores, local or peer, are visible first).
void stream_wait_geq(cudaStream_t s, const uint32_t* addr, uint32_t v);
void stream_write(cudaStream_t s, uint32_t* addr, uint32_t v);

}  // namespace naspipe
