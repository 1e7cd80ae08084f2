"""Dev tool: where the e2e loop's time goes on the bench set (16 GNMT graphs,
fp32): per-step wall time of the double-buffered loop with / without the
per-step reload and the per-step loss read."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_icpp_lancl21_b200 as mars  # noqa: E402
import paper_conf_icpp_lancl21_b200.mars as _mm  # noqa: E402
if os.environ.get("MARS_LIB"):                     # A/B: another libmars build
    _mm.LIB_PATH = os.environ["MARS_LIB"]
from synth import graphs as SG  # noqa: E402


class P:
    pass


WL = os.environ.get("MARS_AB_WORKLOAD", "gnmt")
NG = 8 if WL == "bert" else 16
gs = []
for i in range(NG):
    g = SG.cached(WL, i)
    p = P()
    p.num_nodes = g.num_nodes
    p.indptr = torch.from_numpy(np.ascontiguousarray(g.indptr)).pin_memory().numpy()
    p.indices = torch.from_numpy(np.ascontiguousarray(g.indices)).pin_memory().numpy()
    p.features = torch.from_numpy(np.ascontiguousarray(g.features)).pin_memory().numpy()
    gs.append(p)
stream = torch.cuda.Stream()
m = mars.dgi_create(in_dim=64, hidden_dim=128 if WL == "inception" else 256, seed=0)
m.set_stream(stream.cuda_stream)
ga = mars.graph_load(gs)
gb = mars.graph_load(gs)
for k in range(4):
    m.step(ga if k % 2 == 0 else gb, 100 + k, 0, NG)
torch.cuda.synchronize()
n = 40


def run(reload, read):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    cur, nxt = ga, gb
    if reload:
        cur.reload(gs)
    for k in range(n):
        m.step(cur, 1 + k, 0, NG)
        if reload and k + 1 < n:
            nxt.reload(gs)
        if read:
            m.read_step(want_grads=False)
        cur, nxt = nxt, cur
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / n * 1e3


for rep in range(2):
    for reload in (True, False):
        for read in (True,):
            print(f"reload={reload:d} read={read:d}: {run(reload, read):.3f} ms/step", flush=True)
# the reload alone (H2D + CSR build on the loader stream), serialised
torch.cuda.synchronize()
t0 = time.perf_counter()
for k in range(10):
    ga.reload(gs)
    torch.cuda.synchronize()
print(f"reload alone: {(time.perf_counter() - t0) / 10 * 1e3:.3f} ms", flush=True)
# the CSR build alone: the reload's device work on the loader stream, timed
# with events around a reload of an already-resident batch is not separable
# from the H2D, so report the e2e loop above and this wall time only
