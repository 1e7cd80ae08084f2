"""compute-sanitizer workload (tools/sanitize.sh): one eager step per case on
small sets -- tiny (SIMT GEMMs), Inception x2 at H = 128 and one Inception
graph at H = 256 (tcgen05 row / dW kernels, incl. the CTA-pair dW), two GNMT
graphs (R > 2 x 128 x #SM rows: the CTA-pair row GEMMs, both instantiations), both
precisions, plus an encode and the featuriser; then the NEXT-4 variants
(MARS_SAN_ONLY=default | variants selects one group).  Small so the
instrumented run finishes in minutes."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import paper_conf_icpp_lancl21_b200 as mars  # noqa: E402
from synth import graphs as SG  # noqa: E402

cases = [([SG.tiny(0), SG.tiny(1)], 16, 32, mars.MARS_FP32),
         ([SG.cached("inception", i) for i in range(2)], 64, 128, mars.MARS_FP32),
         ([SG.cached("inception", 0)], 64, 256, mars.MARS_FP32),
         ([SG.cached("inception", 0)], 64, 256, mars.MARS_BF16),
         ([SG.cached("bert", 0)], 64, 256, mars.MARS_FP32),          # long rows
         ([SG.cached("gnmt", i) for i in range(2)], 64, 256, mars.MARS_FP32)]   # pair row GEMMs
# NEXT-4 variants (c34-c38): shared positive with padding, masking, mean
# readout, SAGE-GCN values, and the SAGE-mean encoder's redirected CSR
variants = [([SG.tiny(0), SG.tiny(1)], 16, 32, mars.MARS_FP32, "gcn",
             dict(num_neg=2, corruption="mask", mask_rate=0.3, readout="mean")),
            ([SG.cached("inception", 0)], 64, 256, mars.MARS_FP32, "gcn",
             dict(num_neg=3, aggregator="sage_gcn")),
            ([SG.cached("inception", 0)], 64, 256, mars.MARS_BF16, "gcn", dict(num_neg=2)),
            ([SG.tiny(0), SG.tiny(1)], 16, 32, mars.MARS_FP32, "sage", dict(num_neg=2)),
            ([SG.cached("inception", 0)], 64, 256, mars.MARS_FP32, "sage",
             dict(num_neg=4, corruption="mask", mask_rate=0.2)),
            ([SG.tiny(0), SG.tiny(1)], 16, 32, mars.MARS_FP32, "sage_pool", dict(num_neg=2)),
            ([SG.cached("inception", 0)], 64, 128, mars.MARS_FP32, "sage_pool",
             dict(num_neg=3, loss="infonce"))]
only = os.environ.get("MARS_SAN_ONLY", "")
runs = ([] if only == "variants" else [(gs, F, H, p, "gcn", {}) for gs, F, H, p in cases]) + \
    ([] if only == "default" else variants)
for gs, F, H, prec, enc, var in runs:
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=1, precision=prec, encoder=enc)
    m.set_graph_capture(False)
    if os.environ.get("MARS_SAN_GEMM") and prec == mars.MARS_FP32:
        m.set_gemm_impl(os.environ["MARS_SAN_GEMM"])    # simt: no TMA-stored GEMM outputs
    m.set_contrastive(**var)
    out = m.step(g, 0, 0, want_loss=True)
    emb = m.encode(g)
    print(f"N={sum(x.num_nodes for x in gs)} F={F} H={H} prec={prec} enc={enc} {var} "
          f"loss={out['loss']:.6f} emb finite={bool(np.isfinite(emb).all())}", flush=True)
    m.free(); g.free()
g0 = SG.cached("tiny", 0)
X = mars.featurize(g0.types, g0.dims, 16)
print("featurize ok", X.shape, flush=True)
