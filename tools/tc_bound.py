"""Upper bound of a tensor-core histogram (the north star's "one-hot x gradient contraction,
kept only if it wins at large d"), measured with the library int8 GEMM (cuBLASLt via
torch._int_mm) instead of building the kernel.

One feature's histogram over a chunk of R rows is  OneHot[B x R] @ Qlimbs[R x 4V]  with the
31-bit fixed-point q split into 4 int8 limbs (exact: int32 accumulation of <= 2^24 one-hot
products per limb).  The GEMM alone — before building any one-hot tile — bounds what a
tcgen05 kind::i8 kernel could reach.  Reported as (row, feature) pairs per second, next to the
shared-atomic kernel's measured rate for the same V (bench lines: rows x m per second inside
build_hist).  Usage: python tools/tc_bound.py
"""
import json

import torch


def gemm_rate(B, V, R=65536, reps=20):
    dev = torch.device("cuda:0")
    a = torch.randint(0, 2, (B, R), dtype=torch.int8, device=dev)           # one-hot^T (values 0/1)
    b = torch.randint(-128, 127, (R, 4 * V), dtype=torch.int8, device=dev)  # q limbs
    for _ in range(3):
        torch._int_mm(a, b)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        torch._int_mm(a, b)
    e1.record()
    torch.cuda.synchronize()
    s = e0.elapsed_time(e1) * 1e-3 / reps
    ops = 2.0 * B * R * 4 * V
    return {"B": B, "V": V, "R": R, "ms": s * 1e3, "int8_tops": ops / s / 1e12,
            "row_feature_per_s": R / s}


def main():
    out = {"what": "int8 GEMM OneHot[B x R] @ Qlimbs[R x 4V] (cuBLASLt, torch._int_mm), one feature per GEMM",
           "cases": []}
    for B, V in [(256, 16), (256, 32), (256, 256)]:
        out["cases"].append(gemm_rate(B, V))
    # batched over features: the same Qlimbs for 8 features stacked along M (B x 8 rows of one-hot)
    for B, V in [(256 * 8, 16), (256 * 8, 256)]:
        r = gemm_rate(B, V)
        r["features_per_gemm"] = 8
        r["row_feature_per_s"] *= 8
        out["cases"].append(r)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
