"""A/B of session-lowering / GEMM settings on one BERT-Large step, interleaved in one
process so clock and thermal drift cancel.  Each variant: env vars set before the session
is built (the lowering reads them then) and a ts_gemm_set_mode value.
    python tools/ab_step.py [budget_frac (0 = all-reside)] [rounds]"""
import json
import os
import subprocess
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402

VARIANTS = {
    "nofusion": ({"TSPLIT_NO_FUSION": "1"}, 0),
    "fusion": ({}, 0),
}


def sm_clock():
    try:
        return float(subprocess.check_output(["nvidia-smi", "--query-gpu=clocks.sm", "--format=csv,noheader,nounits"],
                                             text=True).split()[0])
    except Exception:
        return None


def main():
    frac = float(sys.argv[1]) if len(sys.argv) > 1 else 0.25
    rounds = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    spec = graphs.bert(layers=24, batch=32, fused_attention=True)
    G = tsplit.Graph(spec)
    P = tsplit.Plan.default(G)
    dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
    if frac > 0:
        st = P.stats()
        prof = tsplit.Profile.measure(G, dev, max_p=16)
        P = tsplit.Plan.plan(G, st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"])), prof)
    params = gen.init_params(spec)
    res = {k: [] for k in VARIANTS}
    for r in range(rounds):
        for name, (env, mode) in VARIANTS.items():
            for k in ("TSPLIT_NO_QKV_FUSION", "TSPLIT_NO_FUSION"):
                os.environ.pop(k, None)
            os.environ.update(env)
            tsplit.check(tsplit.lib().ts_gemm_set_mode(mode))
            stream = torch.cuda.Stream()
            S = tsplit.Session(G, P, lr=1e-4, streams=(stream, torch.cuda.Stream(), torch.cuda.Stream()))
            S.set_params(params)
            for _ in range(3):
                S.step(dev)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            n = 10
            for _ in range(n):
                S.step_async(dev)
            time.sleep(0.2)
            clk = sm_clock()
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / n
            res[name].append((ms, clk, S.launches()))
            print(f"round {r} {name:20s} {ms:7.2f} ms/step  sm {clk} MHz  launches {S.launches()}", flush=True)
            del S
            torch.cuda.empty_cache()
    print(json.dumps({k: min(v)[0] for k, v in res.items()}))


if __name__ == "__main__":
    main()
