"""Timings of the NEXT rows on one GPU (wall clock around synchronous ABI calls,
after a warm-up): placer forward (S = 10 draws, paper sizes), the PPO loss
gradient of one minibatch (5 placements), one PPO iteration (P:L237 schedule)
and one joint iteration, on the Inception-V3 and GNMT op graphs.  Prints one
JSON line per case."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import paper_conf_icpp_lancl21_b200 as mars  # noqa: E402
from synth import graphs as SG  # noqa: E402


def timed(fn, reps=1):
    fn()
    t0 = time.perf_counter()
    for _ in range(reps):
        out = fn()
    return (time.perf_counter() - t0) / reps, out


for name in sys.argv[1:] or ["inception", "gnmt"]:
    g0 = SG.cached(name, 0)
    N = g0.num_nodes
    g = mars.graph_load([g0])
    enc = mars.dgi_create(in_dim=64, hidden_dim=256, seed=1)
    E = enc.encode(g)
    p = mars.placer_create(seed=1)
    t_fwd, (pl, lp, _) = timed(lambda: p.sample(E, 10, 7))
    adv = np.linspace(-1, 1, 5).astype(np.float32)
    t_grad, _ = timed(lambda: p.ppo_grad(E, pl[:5], lp[:5], adv))
    o = mars.ppo_create(p, seed=2, capacity_bytes=4e9)
    t_it, _ = timed(lambda: o.iteration(E, g0))
    oj = mars.ppo_create(p, enc, seed=3, capacity_bytes=4e9)
    t_j, _ = timed(lambda: oj.iteration_joint(g, g0))
    print(json.dumps({"graph": name, "ops": N, "placer_forward_10_samples_s": t_fwd,
                      "us_per_op_forward": 1e6 * t_fwd / N,
                      "ppo_grad_5_samples_s": t_grad, "us_per_op_grad": 1e6 * t_grad / N,
                      "ppo_iteration_s": t_it, "ppo_iteration_joint_s": t_j}), flush=True)
    for h in (oj, o, p, enc, g):
        h.free()
