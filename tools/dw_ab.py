"""Dev tool: time the weight-gradient GEMM (mars_debug_gemm 'dw', which also
runs the two row-scale kernels) at the bench shape for every libmars variant
given on the command line (paths to .so files; default: the in-tree build)."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CODE = r'''
import sys, numpy as np
sys.path.insert(0, %r)
import paper_conf_icpp_lancl21_b200.mars as mm
mm.LIB_PATH = sys.argv[1]
R = 419232
rng = np.random.default_rng(0)
for K in (64, 256):
    A = rng.standard_normal((R, K)).astype(np.float32)
    D = rng.standard_normal((R, 256)).astype(np.float32)
    C, t = mm.debug_gemm("dw", A, D, "auto", iters=20)
    e = np.abs(C - A.astype(np.float64).T @ D).max() / np.abs(A.astype(np.float64).T @ D).max()
    print(f"{sys.argv[1].split('/')[-1]} K={K}: dw {t:.3f} ms/launch (incl. row scales)  err {e:.2e}", flush=True)
''' % ROOT
for lib in sys.argv[1:] or [os.path.join(ROOT, "paper_conf_icpp_lancl21_b200", "libmars.so")]:
    subprocess.call([sys.executable, "-c", CODE, lib])
