"""Time one GEMM form repeatedly (for ncu): python tools/gemm_one.py M N K ta tb out beta [batch]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tools.gemm_bench import case  # noqa
M, N, K, ta, tb = map(int, sys.argv[1:6]); out = sys.argv[6]; beta = float(sys.argv[7])
batch = int(sys.argv[8]) if len(sys.argv) > 8 else 1
case("one", M, N, K, ta, tb, out=out, beta=beta, batch=batch)
