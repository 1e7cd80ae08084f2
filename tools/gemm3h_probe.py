"""Dev tool: time the row GEMMs ('auto' = 3xFP16, '3xtf32') at the bench shape
through mars_debug_gemm (weight split included), for ncu captures."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import paper_conf_icpp_lancl21_b200 as mars  # noqa: E402

rng = np.random.default_rng(0)
R = 419232
for K in (256, 64):
    A = rng.standard_normal((R, K)).astype(np.float32)
    W = rng.standard_normal((256, K)).astype(np.float32)
    for impl in sys.argv[1:] or ["auto", "3xtf32"]:
        _, t = mars.debug_gemm("rows", A, W, impl, iters=5)
        print(f"K={K} {impl}: rows {t:.3f} ms", flush=True)
