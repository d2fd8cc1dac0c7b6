"""Run a few GEMM shapes of the C3 block once each (for ncu capture)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from tools.gemm_perf import L
shapes = [("ffn1_f4096", 4096, 4096, 1024, 0, 0, 4), ("dW1_f4096", 4096, 1024, 4096, 1, 1, 6),
          ("da2_f4096", 4096, 1024, 4096, 0, 1, 1), ("qkv", 4096, 3072, 1024, 0, 0, 2)]
for name, M, N, K, amn, bmn, epi in shapes:
    A = torch.randn((K, M) if amn else (M, K), device="cuda", dtype=torch.bfloat16)
    B = torch.randn((K, N) if bmn else (N, K), device="cuda", dtype=torch.bfloat16)
    o32 = torch.empty((M, N), device="cuda"); o16 = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    o16b = torch.empty_like(o16); bias = torch.zeros(N, device="cuda"); w32 = torch.zeros((M, N), device="cuda")
    out = o32 if epi in (1, 3) else o16
    for _ in range(2):
        assert L.naspipe_debug_gemm(M, N, K, A.data_ptr(), amn, A.shape[1], B.data_ptr(), bmn, B.shape[1], epi,
                                    bias.data_ptr(), o32.data_ptr(), o16b.data_ptr(), out.data_ptr(), o16b.data_ptr(),
                                    w32.data_ptr(), o16.data_ptr(), 0.0, None) == 0
    torch.cuda.synchronize()
