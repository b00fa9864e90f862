"""Measure a workload's profile on the GPU (ts_profile_measure) and dump it as JSON, so a
plan can be reproduced on the CPU with Profile.from_dict.
    python tools/dump_profile.py [vgg16|resnet50|bert_large] [out.json]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "vgg16"
out = sys.argv[2] if len(sys.argv) > 2 else f"gpurun_out/profile_{wl}.json"
spec = bench.workload_graph(wl)
G = tsplit.Graph(spec)
dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
prof = tsplit.Profile.measure(G, dev, max_p=16)
json.dump(prof.to_dict(), open(out, "w"))
print("wrote", out)
