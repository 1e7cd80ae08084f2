"""Run each dense-transform kernel once on bench-sized operands (for ncu)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_icpp_lancl21_b200 as mars
rng = np.random.default_rng(0)
R = 419232
A = rng.standard_normal((R, 256)).astype(np.float32)
W = rng.standard_normal((256, 256)).astype(np.float32)
D = rng.standard_normal((R, 256)).astype(np.float32)
which = sys.argv[1] if len(sys.argv) > 1 else "both"
if which in ("rows", "both"):
    print("rows", mars.debug_gemm("rows", A, W, "auto", iters=1)[1])
if which in ("dw", "both"):
    print("dw", mars.debug_gemm("dw", A, D, "auto", iters=1)[1])
