"""Device time per step of the NEXT-4 contrastive variants on the bench workload
(GNMT x16 per GPU, F = 64, H = 256, fp32): the default DGI step, K = 4
corruption samples with ONE positive branch (c34) against the same K samples
run as K copies of every graph (c20, the positive branch recomputed K times),
feature masking, the mean readout, SAGE-GCN aggregation and the SAGE-mean
encoder (c38).  CUDA events on the
library's stream around `steps` captured steps after a warm-up; inputs larger
than L2.  Prints one JSON line per case."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_icpp_lancl21_b200 as mars  # noqa: E402
from synth import graphs as SG  # noqa: E402

B, F, H, steps, warm = 16, 64, 256, 30, 5
base = [SG.cached("gnmt", i) for i in range(B)]
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)


def run(name, graphs, variant, batch, encoder="gcn"):
    g = mars.graph_load(graphs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=1, encoder=encoder)
    m.set_stream(stream.cuda_stream)
    m.set_contrastive(**variant)
    for s in range(warm):
        m.step(g, s, 0, batch)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for s in range(steps):
        m.step(g, warm + s, 0, batch)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    loss = m.step(g, warm + steps, 0, batch, want_loss=True)["loss"]
    print(json.dumps({"case": name, "variant": variant, "graphs": len(graphs), "ms_per_step": ms,
                      "graph_steps_per_s": B / ms * 1e3, "launches": m.last_launches(),
                      "loss": loss}), flush=True)
    m.free(); g.free()
    return ms


run("default", base, {}, B)
shared = run("K=4 shared positive", base, dict(num_neg=4), B)
copies = run("K=4 as copies", mars.corruption_samples(base, 4), {}, 4 * B)
print(json.dumps({"shared_over_copies_speedup": copies / shared}), flush=True)
run("K=2 shared positive", base, dict(num_neg=2), B)
run("mask 0.2", base, dict(corruption="mask", mask_rate=0.2), B)
run("readout mean", base, dict(readout="mean"), B)
run("InfoNCE", base, dict(loss="infonce"), B)
run("InfoNCE, K=4", base, dict(num_neg=4, loss="infonce"), B)
run("SAGE-GCN", base, dict(aggregator="sage_gcn"), B)
run("SAGE-mean encoder", base, {}, B, encoder="sage")
run("SAGE-mean encoder, K=3", base, dict(num_neg=3), B, encoder="sage")
run("SAGE-pool encoder", base, {}, B, encoder="sage_pool")
