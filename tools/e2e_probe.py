"""Dev tool: per-iteration wall times of the pipelined e2e loop (load / step /
read / free) on the bench set, to locate stalls."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_icpp_lancl21_b200 as mars  # noqa: E402
from synth import graphs as SG  # noqa: E402


class P:
    pass


gs = []
for i in range(16):
    g = SG.cached("gnmt", i)
    p = P()
    p.num_nodes = g.num_nodes
    p.indptr = torch.from_numpy(np.ascontiguousarray(g.indptr)).pin_memory().numpy()
    p.indices = torch.from_numpy(np.ascontiguousarray(g.indices)).pin_memory().numpy()
    p.features = torch.from_numpy(np.ascontiguousarray(g.features)).pin_memory().numpy()
    gs.append(p)
m = mars.dgi_create(in_dim=64, hidden_dim=256, seed=0)
gg = mars.graph_load(gs)
m.step(gg, 0, 0, 16, want_loss=True)
gg.free()
gg = mars.graph_load(gs)
for k in range(40):
    t0 = time.perf_counter()
    m.step(gg, 1 + k, 0, 16)
    t1 = time.perf_counter()
    nxt = mars.graph_load(gs)
    t2 = time.perf_counter()
    m.read_step(want_grads=False)
    t3 = time.perf_counter()
    gg.free()
    t4 = time.perf_counter()
    gg = nxt
    print(f"{k:2d} step {1e3*(t1-t0):6.2f} load {1e3*(t2-t1):6.2f} read {1e3*(t3-t2):6.2f} "
          f"free {1e3*(t4-t3):6.2f} total {1e3*(t4-t0):6.2f} ms", flush=True)
