"""H2D upload rate of the host X (pinned, row-major 2 M x 4096 fp32 = 32.8 GB) for the strip-wise
upload in bin_features_host: contiguous copy vs cudaMemcpy2DAsync strips of w columns, and the
whole bin_features_host call.  python tools/h2d_probe.py"""
import json
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_liupw25_b200 as pkg  # noqa: E402
from paper_conf_icpp_liupw25_b200 import booster  # noqa: E402
from gen import gen  # noqa: E402



def _memcpy2d_h2d(dst_ptr, dpitch, src_ptr, spitch, width, height, stream_handle):
    import ctypes as C
    rt = C.CDLL("libcudart.so.12")
    rt.cudaMemcpy2DAsync.argtypes = [C.c_void_p, C.c_size_t, C.c_void_p, C.c_size_t, C.c_size_t, C.c_size_t,
                                     C.c_int, C.c_void_p]
    if rt.cudaMemcpy2DAsync(dst_ptr, dpitch, src_ptr, spitch, width, height, 1, stream_handle) != 0:
        raise RuntimeError("cudaMemcpy2DAsync failed")

def main():
    w = gen.WORKLOADS["C5"]
    n, m = w.n, w.m
    Xh = torch.empty((n, m), dtype=torch.float32, pin_memory=True)
    gen.matrix_host(w.seed, gen.STREAM_X, w.x_kind, 0, n, 0, m, m, out=Xh.numpy())
    dev = torch.device("cuda:0")
    out = {}
    Xd = torch.empty((n, m), dtype=torch.float32, device=dev)
    for _ in range(2):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        Xd.copy_(Xh, non_blocking=True)
        torch.cuda.synchronize(); out["contiguous_GBs"] = Xh.numel() * 4 / (time.perf_counter() - t0) / 1e9
    del Xd
    s = torch.cuda.current_stream()
    for sw in (256, 512, 1024, 2048):
        buf = torch.empty((n, sw), dtype=torch.float32, device=dev)
        torch.cuda.synchronize(); t0 = time.perf_counter()
        for f0 in range(0, m, sw):
            _memcpy2d_h2d(buf.data_ptr(), 4 * sw, Xh.data_ptr() + 4 * f0, 4 * m, 4 * sw, n, s.cuda_stream)
        torch.cuda.synchronize(); out[f"strips{sw}_GBs"] = Xh.numel() * 4 / (time.perf_counter() - t0) / 1e9
        del buf
    ctx = pkg.Context(0)
    for sw in (512, 1024):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        ds = pkg.bin_features_host(ctx, Xh, w.B, dev, strip=sw)
        torch.cuda.synchronize(); out[f"bin_features_host_{sw}_s"] = time.perf_counter() - t0
        del ds
    print(json.dumps(out))


if __name__ == "__main__":
    main()
