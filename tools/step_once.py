"""Run a few bench-config steps through a given libmars.so (dev tool, for ncu
captures of single kernels):  python tools/step_once.py LIB {fp32|bf16} [steps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_lancl21_b200.mars as M  # noqa: E402
from synth import graphs as SG  # noqa: E402

M.LIB_PATH = os.path.abspath(sys.argv[1])
prec = M.MARS_BF16 if sys.argv[2] == "bf16" else M.MARS_FP32
n = int(sys.argv[3]) if len(sys.argv) > 3 else 1
g = M.graph_load([SG.cached("gnmt", i) for i in range(16)])
m = M.dgi_create(in_dim=64, hidden_dim=256, seed=0, precision=prec)
m.set_graph_capture(False)
for k in range(n):
    m.step(g, k, 0)
print("ok")
