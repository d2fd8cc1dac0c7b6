"""Timing of the attention kernels (naspipe_debug_attn_fwd/bwd) on the configs[2] shapes
(B=32, S=128, d=1024, h in {8, 16}): mean of 20 back-to-back calls, CUDA events.  GPU only."""
import ctypes as C
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402

L = npipe.lib
_vp = C.c_void_p
L.naspipe_debug_attn_fwd.argtypes = [_vp, _vp, _vp] + [C.c_int] * 4 + [_vp]
L.naspipe_debug_attn_bwd.argtypes = [_vp] * 5 + [C.c_int] * 4 + [_vp]


def timed(fn, inner=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda._sleep(2_000_000)
    a.record()
    for _ in range(inner):
        fn()
    b.record()
    torch.cuda.synchronize()
    return 1000 * a.elapsed_time(b) / inner


def main():
    B, S, d = 32, 128, 1024
    for h in (8, 16):
        qkv = torch.randn(B * S, 3 * d, device="cuda").to(torch.bfloat16)
        o = torch.empty(B * S, d, device="cuda", dtype=torch.bfloat16)
        lse = torch.empty(B * h * S, device="cuda")
        do = torch.randn(B * S, d, device="cuda").to(torch.bfloat16)
        dqkv = torch.empty_like(qkv)
        f = lambda: L.naspipe_debug_attn_fwd(qkv.data_ptr(), o.data_ptr(), lse.data_ptr(), B, S, d, h, None)
        g = lambda: L.naspipe_debug_attn_bwd(qkv.data_ptr(), o.data_ptr(), lse.data_ptr(), do.data_ptr(),
                                             dqkv.data_ptr(), B, S, d, h, None)
        print(json.dumps(dict(h=h, hd=d // h, fwd_us=timed(f), bwd_us=timed(g))))


if __name__ == "__main__":
    main()
