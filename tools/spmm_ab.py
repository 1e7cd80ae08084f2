"""A/B timing of libmars variants (dev tool): for each given libmars.so, in a
fresh process, profile the bench step (16 GNMT graphs, F=64, H=256) in fp32
and bf16 and print the median device time of every SpMM / head phase entry.

  python tools/spmm_ab.py build/variants/*.so
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(path):
    sys.path.insert(0, ROOT)
    os.environ["MARS_BINDING_LENIENT"] = "1"
    import numpy as np
    import paper_conf_icpp_lancl21_b200.mars as M
    M.LIB_PATH = path
    from synth import graphs as SG
    wl = os.environ.get("MARS_AB_WORKLOAD", "gnmt")          # gnmt | inception | bert
    gs = [SG.cached(wl, i) for i in range({"gnmt": 16, "inception": 16, "bert": 8}[wl])]
    H = 128 if wl == "inception" else 256
    g = M.graph_load(gs)
    out = {}
    for prec in (M.MARS_FP32, M.MARS_BF16):
        m = M.dgi_create(in_dim=64, hidden_dim=H, seed=0, precision=prec)
        if os.environ.get("MARS_AB_GEMM"):
            m.set_gemm_impl(os.environ["MARS_AB_GEMM"])
        for k in range(3):
            m.step(g, k, 0)
        runs = [m.profile_step(g, 10 + k, 0) for k in range(7)]
        names = [n for n, _ in runs[0]]
        tab = np.array([[t for _, t in r] for r in runs])
        med = np.median(tab, axis=0)
        agg = {}
        for n, t in zip(names, med):
            agg[n] = agg.get(n, 0.0) + float(t)
        out["bf16" if prec == M.MARS_BF16 else "fp32"] = {k: round(v, 4) for k, v in agg.items()}
        m.free()
    print(json.dumps(out))


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "--child":
        child(sys.argv[2])
        sys.exit(0)
    for p in sys.argv[1:]:
        r = subprocess.run([sys.executable, __file__, "--child", os.path.abspath(p)],
                           capture_output=True, text=True, timeout=600)
        if r.returncode:
            print(os.path.basename(p), "FAILED", r.stderr[-400:])
            continue
        d = json.loads(r.stdout.strip().splitlines()[-1])
        for prec in ("fp32", "bf16"):
            ph = d[prec]
            print(f"{os.path.basename(p):28s} {prec}  spmm_fwd {ph.get('spmm_fwd', 0):.4f}  "
                  f"spmm_bwd {ph.get('spmm_bwd', 0):.4f}  head {ph.get('head', 0):.4f}  "
                  f"gemm_fwd {ph.get('gemm_fwd', 0):.4f}  gemm_dy {ph.get('gemm_dy', 0):.4f}  "
                  f"gemm_dw {ph.get('gemm_dw', 0):.4f}  total {sum(ph.values()):.4f}", flush=True)
