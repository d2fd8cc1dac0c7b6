// Host-side TMA tensor maps shared by the tcgen05 kernels (gemm.cu builds them).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>

#include <cstdint>

namespace naspipe {
// 2-D bf16 tensor [outer][inner] with row pitch `ld` elements; box = 64 inner x box_outer,
// 128-byte swizzle (the UMMA SW128 K-major / MN-major operand layout)
CUtensorMap tma_map_bf16(const __nv_bfloat16* base, uint64_t inner, uint64_t outer, uint64_t ld, uint32_t box_outer);
}  // namespace naspipe
