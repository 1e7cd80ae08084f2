import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_icpp_lancl21_b200 as mars
np.set_printoptions(linewidth=200)
M, K = 16, 64
A = np.zeros((M, K), np.float32); B = np.zeros((M, 256), np.float32)
# probe 1: single A entry, B row r = index
for r in range(M):
    B[r] = np.arange(256) + 1000 * r
A[3, 5] = 1.0
C, _ = mars.debug_gemm("dw", A, B, "auto")
nz = np.argwhere(C != 0)
print("probe1 expect C[5,n] = 3000+n; nonzeros", len(nz), nz[:8].tolist(), C[nz[:8, 0], nz[:8, 1]].tolist() if len(nz) else None)
# probe 2: B single entry, A row index
A = np.zeros((M, K), np.float32); B = np.zeros((M, 256), np.float32)
for r in range(M):
    A[r] = np.arange(K) + 100 * r
B[3, 7] = 1.0
C, _ = mars.debug_gemm("dw", A, B, "auto")
nz = np.argwhere(C != 0)
print("probe2 expect C[c,7] = 300+c; nonzeros", len(nz), nz[:8].tolist(), C[nz[:8, 0], nz[:8, 1]].tolist() if len(nz) else None)
# probe 3: rows variant with K-major (sanity)
A = np.random.default_rng(0).standard_normal((M, K)).astype(np.float32)
B = np.random.default_rng(1).standard_normal((M, 256)).astype(np.float32)
C, _ = mars.debug_gemm("dw", A, B, "auto")
ref = A.T.astype(np.float64) @ B
print("probe3 err", np.abs(C - ref).max(), "C[:2,:6]", C[:2, :6], "ref", ref[:2, :6])
