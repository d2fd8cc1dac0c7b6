"""Per-shape timing of the tcgen05 GEMM (naspipe_debug_gemm) vs torch.matmul (cuBLAS) on the
transformer block's shapes.  CUDA events, warm-up, median of repeats.  GPU only."""
import ctypes as C
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402

L = npipe.lib
_vp = C.c_void_p
L.naspipe_debug_gemm.argtypes = [C.c_int] * 3 + [_vp, C.c_int, C.c_int, _vp, C.c_int, C.c_int, C.c_int,
                                                 _vp, _vp, _vp, _vp, _vp, _vp, _vp, C.c_float, _vp]


def bench(fn, reps=5, inner=20):
    """Median over `reps` of the mean time of `inner` back-to-back calls (the host enqueues
    ahead of the GPU, as in a training step, so host-side launch cost is not timed)."""
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(2_000_000)  # keep the GPU busy while the host enqueues the calls
        a.record()
        for _ in range(inner):
            fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / inner)
    ts.sort()
    return ts[len(ts) // 2]


def main():
    T, d = 4096, 1024
    shapes = []
    for f in (2048, 4096):
        shapes += [("qkv", T, 3 * d, d, 0, 0, 2), ("oproj", T, d, d, 0, 0, 3), (f"ffn1_f{f}", T, f, d, 0, 0, 4),
                   (f"ffn2_f{f}", T, d, f, 0, 0, 3), (f"dz_f{f}", T, f, d, 0, 1, 5), (f"da2_f{f}", T, d, f, 0, 1, 1),
                   ("do", T, d, d, 0, 1, 0), ("da", T, d, 3 * d, 0, 1, 1), (f"dW2_f{f}", d, f, T, 1, 1, 6),
                   (f"dW1_f{f}", f, d, T, 1, 1, 6), ("dWo", d, d, T, 1, 1, 6), ("dWqkv", 3 * d, d, T, 1, 1, 6)]
    shapes.append(("square8192", 8192, 8192, 8192, 0, 0, 1))
    seen, results = set(), []
    for name, M, N, K, amn, bmn, epi in shapes:
        if name in seen:
            continue
        seen.add(name)
        A = torch.randn((K, M) if amn else (M, K), device="cuda", dtype=torch.bfloat16)
        B = torch.randn((K, N) if bmn else (N, K), device="cuda", dtype=torch.bfloat16)
        o32 = torch.empty((M, N), device="cuda", dtype=torch.float32)
        o16 = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
        o16b = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
        bias = torch.zeros(N, device="cuda")
        w32 = torch.zeros((M, N), device="cuda")
        out = o32 if epi in (1, 3) else o16

        def ours():
            rc = L.naspipe_debug_gemm(M, N, K, A.data_ptr(), amn, A.shape[1], B.data_ptr(), bmn, B.shape[1], epi,
                                      bias.data_ptr(), o32.data_ptr(), o16b.data_ptr(), out.data_ptr(),
                                      o16b.data_ptr(), w32.data_ptr(), o16.data_ptr(), 0.0, None)
            assert rc == 0, L.naspipe_last_error()

        At = A.t() if amn else A
        Bt = B if bmn else B.t()

        def ref():
            torch.matmul(At, Bt, out=o16b)

        t_ours, t_ref = bench(ours), bench(ref)
        fl = 2.0 * M * N * K
        row = dict(name=name, M=M, N=N, K=K, epi=epi, ours_us=1000 * t_ours, cublas_us=1000 * t_ref,
                   ours_tflops=fl / t_ours / 1e9, cublas_tflops=fl / t_ref / 1e9)
        results.append(row)
        print(json.dumps(row))
    return results


if __name__ == "__main__":
    main()
