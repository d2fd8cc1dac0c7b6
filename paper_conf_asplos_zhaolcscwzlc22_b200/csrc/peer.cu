// Peer-memory transport helpers (see peer.h).
#include <cuda.h>

#include "common.h"
#include "peer.h"

namespace naspipe {

namespace {
using WaitFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
using WriteFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

template <class F>
F entry(const char* name) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
    p = nullptr;
  NP_REQUIRE(p != nullptr, NASPIPE_ECUDA, "driver entry point %s unavailable", name);
  return reinterpret_cast<F>(p);
}
}  // namespace

void stream_wait_geq(cudaStream_t s, const uint32_t* addr, uint32_t v) {
  static const WaitFn fn = entry<WaitFn>("cuStreamWaitValue32");
  const CUresult r = fn((CUstream)s, (CUdeviceptr)addr, v, CU_STREAM_WAIT_VALUE_GEQ);
  NP_REQUIRE(r == CUDA_SUCCESS, NASPIPE_ECUDA, "cuStreamWaitValue32 failed (%d)", (int)r);
}

void stream_write(cudaStream_t s, uint32_t* addr, uint32_t v) {
  static const WriteFn fn = entry<WriteFn>("cuStreamWriteValue32");
  const CUresult r = fn((CUstream)s, (CUdeviceptr)addr, v, CU_STREAM_WRITE_VALUE_DEFAULT);
  NP_REQUIRE(r == CUDA_SUCCESS, NASPIPE_ECUDA, "cuStreamWriteValue32 failed (%d)", (int)r);
}

PeerLink::~PeerLink() {
  cudaSetDevice(dev);
  for (void* p : opened) cudaIpcCloseMemHandle(p);
  for (void* p : {in_ring, gout_ring, static_cast<void*>(flags)})
    if (p) cudaFree(p);
}

}  // namespace naspipe
