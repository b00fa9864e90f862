"""One step of batch-1 VGG-16 (bf16) under Alg. 2's plan at 45 % of its dynamic peak (height
bands, reading D-ATTR) — the workload for an ncu capture of the staging kernels
(band_gather_k / band_scatter_add_k: HBM-bound copies, algorithmic bytes = staged bytes read +
written).  Run under ncu; prints the plan's staging temporaries."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--frac", type=float, default=0.45)
    ap.add_argument("--batch", type=int, default=1)
    a = ap.parse_args()
    g = graphs.config_graph("vgg16", batch=a.batch)
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    P = tsplit.Plan.plan(G, st["static_bytes"] + int(a.frac * (st["peak_extent"] - st["static_bytes"])))
    n = len(g["tensors"])
    temps = [(k, j, b) for _, _, ev, k, j, _, b in P.trace() if ev == "A" and k >= 2 * n]
    print("staging temporaries:", len(temps), "bytes", sum(b for _, _, b in temps))
    S = tsplit.Session(G, P, use_cuda_graph=False)
    S.set_params(gen.init_params(g))
    x = tsplit.inputs_to_device(G, gen.make_inputs(g))
    S.step(x)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
