"""Per-layer throughput of the conv micro-op kernels (C ABI `ts_conv2d`: tcgen05
implicit GEMM) vs cuDNN (torch channels_last bf16 conv + convolution_backward) for
the distinct VGG-16 / ResNet-50 conv shapes at a given micro-op sample count.

    python tools/conv_bench.py [--net vgg16|resnet50|both] [--n N] [--out file.json]
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import graphs  # noqa: E402


def timeit(fn, reps=10):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps / 1e3


def conv_shapes(net):
    g = graphs.config_graph(net, batch=1)
    ts = g["tensors"]
    seen, out = set(), []
    for o in g["ops"]:
        if o["kind"] != "conv2d":
            continue
        x, w = ts[o["inputs"][0]], ts[o["inputs"][1]]
        key = (x["shape"][1], x["shape"][2], x["shape"][3], w["shape"][0], w["shape"][1], w["shape"][2],
               o["iattrs"][0], o["iattrs"][1])
        if key not in seen:
            seen.add(key)
            out.append((o["name"], key, x["kind"] != "input"))
    return out


def case(name, n, key, need_dx):
    H, W, C, K, R, S, st, pad = key
    P = (H + 2 * pad - R) // st + 1
    Q = (W + 2 * pad - S) // st + 1
    bf = torch.bfloat16
    x = torch.randn(n, H, W, C, device="cuda", dtype=bf)
    w = (torch.randn(K, R, S, C, device="cuda") / (R * S * C) ** 0.5).to(bf)
    dy = torch.randn(n, P, Q, K, device="cuda", dtype=bf)
    y = torch.empty(n, P, Q, K, device="cuda", dtype=bf)
    dx = torch.empty_like(x)
    dw = torch.empty(K, R, S, C, device="cuda", dtype=torch.float32)
    geom = (n, H, W, C, K, R, S, st, pad)
    fl = 2.0 * n * P * Q * K * R * S * C
    res = {"name": name, "n": n, "H": H, "W": W, "C": C, "K": K, "R": R, "S": S, "stride": st, "gflop": fl / 1e9}
    # cuDNN reference (channels_last views of the NHWC / KRSC buffers)
    xc = x.permute(0, 3, 1, 2)
    wc = w.permute(0, 3, 1, 2)
    dyc = dy.permute(0, 3, 1, 2)
    for mode, tag in ((1, "fprop"), (2, "dgrad"), (3, "wgrad")):
        if mode == 2 and not need_dx:
            continue
        if mode == 1:
            ours = lambda: tsplit.conv2d(1, geom, x, w, None, y)  # noqa: E731
            ref = lambda: torch.nn.functional.conv2d(xc, wc, None, st, pad)  # noqa: E731
        elif mode == 2:
            ours = lambda: tsplit.conv2d(2, geom, None, w, dy, dx)  # noqa: E731
            ref = lambda: torch.ops.aten.convolution_backward(dyc, xc, wc, None, [st, st], [pad, pad], [1, 1],  # noqa: E731
                                                              False, [0, 0], 1, [True, False, False])
        else:
            ours = lambda: tsplit.conv2d(3, geom, x, w, dy, dw)  # noqa: E731
            ref = lambda: torch.ops.aten.convolution_backward(dyc, xc, wc, None, [st, st], [pad, pad], [1, 1],  # noqa: E731
                                                              False, [0, 0], 1, [False, True, False])
        t_o = timeit(ours)
        t_r = timeit(ref)
        res[f"{tag}_ours_tflops"] = fl / t_o / 1e12
        res[f"{tag}_cudnn_tflops"] = fl / t_r / 1e12
        res[f"{tag}_ours_us"] = t_o * 1e6
    print(json.dumps(res), flush=True)
    return res


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--net", default="both")
    ap.add_argument("--n", type=int, default=0, help="samples per micro-op (default: 32 VGG, 64 ResNet)")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    torch.backends.cudnn.benchmark = True
    rows = []
    for net in (["vgg16", "resnet50"] if a.net == "both" else [a.net]):
        n = a.n or (32 if net == "vgg16" else 64)
        for name, key, need_dx in conv_shapes(net):
            rows.append(case(f"{net}:{name}", n, key, need_dx))
    if a.out:
        json.dump(rows, open(a.out, "w"), indent=1)
