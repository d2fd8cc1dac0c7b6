// BatchNorm arithmetic shared by the SPOS kernels (spos.cu) and the GEMM epilogue that fuses
// the BatchNorm-backward sums (gemm.cu, EPI_BNBWD): one definition, so the fused producers
// and the stand-alone kernels take the same decisions (ReLU mask) and round the same way.
#pragma once

namespace naspipe {

// BN output y = g (z - mean) rstd + b (explicit roundings: no contraction choice can differ
// between the forward and the kernels that recompute it for the ReLU mask)
__device__ __forceinline__ float bn_y(float z, float mu, float rs, float g, float b) {
  return __fmaf_rn(g, __fmul_rn(__fsub_rn(z, mu), rs), b);
}

// One element of the BatchNorm backward: d <- dy masked by the forward's ReLU (relu != 0),
// xh = (z - mean) rstd.  s1 += d and s2 += d xh are the reduction's terms.
__device__ __forceinline__ void bn_bwd_elem(float& d, float z, float mu, float rs, float g, float b, int relu,
                                            float& xh) {
  xh = __fmul_rn(__fsub_rn(z, mu), rs);
  if (relu && !(bn_y(z, mu, rs, g, b) > 0.f)) d = 0.f;
}

}  // namespace naspipe
