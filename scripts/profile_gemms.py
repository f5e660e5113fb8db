"""The transform / gradient GEMMs of a C5-sized epoch on random data (no graph):
xw0 [M x 128]·[128 x 128], xw1 [M x 128]·[128 x 32], dwt [M x 32]·[32 x 128]ᵀ
with mask, xtg1 [M x 128]ᵀ·[M x 32], xtg0 [M x 128]ᵀ·[M x 128].  Times each
with CUDA events (median of 5) and runs one more pass between
cudaProfilerStart/Stop for ncu."""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_tianmyd20_b200 import _lib as L  # noqa: E402


def main():
    M = int(sys.argv[1]) if len(sys.argv) > 1 else 33_554_432
    H, C = 128, 32
    dev = torch.device("cuda", 0)
    X = torch.randn(M, H, device=dev)
    H1 = torch.randn(M, H, device=dev)
    G1 = torch.randn(M, C, device=dev)
    G0 = torch.randn(M, H, device=dev)
    Y0 = torch.empty(M, H, device=dev)
    Y1 = torch.empty(M, C, device=dev)
    dP = torch.empty(M, H, device=dev)
    W0 = torch.randn(H, H, device=dev) * 0.1
    W1 = torch.randn(H, C, device=dev) * 0.1
    r = torch.rand(M, device=dev)
    rr = ctypes.c_void_p(r.data_ptr())
    mask = torch.randint(-2**31, 2**31 - 1, (M, H // 32), dtype=torch.int32, device=dev)
    gW0 = torch.empty(H, H, device=dev)
    gW1 = torch.empty(H, C, device=dev)
    xw_work = torch.empty(max(L.gemm_xw_work_floats(H, H), L.gemm_dwt_work_floats(H, C)), device=dev)
    xtg_work = torch.empty(max(L.gemm_xtg_work_floats(M, H, H), L.gemm_xtg_work_floats(M, H, C)), device=dev)
    ops = {
        "xw0": lambda: L.gemm_xw(X, W0, rr, Y0, work=xw_work),
        "xw1": lambda: L.gemm_xw(H1, W1, rr, Y1, work=xw_work),
        "dwt": lambda: L.gemm_dwt(G1, W1, mask, rr, dP, M=M, N=C, K=H, work=xw_work),
        "xtg1": lambda: L.gemm_xtg(H1, G1, gW1, xtg_work),
        "xtg0": lambda: L.gemm_xtg(X, G0, gW0, xtg_work),
    }
    res = {}
    for k, f in ops.items():
        ts = []
        for _ in range(6):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            f()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        res[k] = float(np.median(ts[1:]))
    torch.cuda.profiler.start()
    for f in ops.values():
        f()
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(json.dumps({"M": M, "ms": res}))


if __name__ == "__main__":
    main()
