import sys, numpy as np
import os; sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG
from tests.util import scaled_err
from tests.test_gpu_shard import _sharded, _step_all
import oracle
graph = SG.cached("inception", 1)
F, H, seed, P, n = 64, 128, 8, 3, 5
for impl in ("auto", "3xtf32"):
    g1 = mars.graph_load([graph])
    m1 = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed); m1.set_gemm_impl(impl)
    ref = [m1.step(g1, t, 0, global_batch=1, want_loss=True, want_grads=True) for t in range(n)]
    gs, ms = _sharded(graph, P, F, H, seed)
    for m in ms: m.set_gemm_impl(impl)
    outs = [_step_all(gs, ms, t)[0] for t in range(n)]
    print(impl, "params", scaled_err(ms[0].get_state()[0], m1.get_state()[0]),
          "grads step0", scaled_err(outs[0][1], ref[0]["grads"]), "loss", scaled_err([o[0] for o in outs], [r["loss"] for r in ref]))
    # grads vs oracle at step 0
