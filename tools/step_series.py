"""Dev tool: per-step device times of the captured bench step (16 GNMT
graphs, fp32) for each libmars given, each in a fresh process: mean, p10 /
p50 / p90 and the first steps, to compare graph-replay timing across builds."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CODE = r'''
import sys, numpy as np, torch
sys.path.insert(0, %r)
import paper_conf_icpp_lancl21_b200.mars as M
M.LIB_PATH = sys.argv[1]
from synth import graphs as SG
import os
wl = os.environ.get("MARS_AB_WORKLOAD", "gnmt")
gs = [SG.cached(wl, i) for i in range(16 if wl != "bert" else 8)]
g = M.graph_load(gs)
m = M.dgi_create(in_dim=64, hidden_dim=128 if wl == "inception" else 256, seed=0)
st = torch.cuda.Stream(); torch.cuda.set_stream(st); m.set_stream(st.cuda_stream)
for w in range(10): m.step(g, w, 0, len(gs))
torch.cuda.synchronize()
n = 100
ev = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
ev[0].record(st)
for k in range(n):
    m.step(g, 10 + k, 0, len(gs)); ev[k + 1].record(st)
ev[-1].synchronize()
t = np.array([ev[k].elapsed_time(ev[k + 1]) for k in range(n)])
print(f"{sys.argv[1].split('/')[-1]:22s} mean {t.mean():.3f}  p10 {np.percentile(t,10):.3f} p50 {np.median(t):.3f} p90 {np.percentile(t,90):.3f}  first: " + " ".join(f"{x:.2f}" for x in t[:16]), flush=True)
''' % ROOT
for lib in sys.argv[1:]:
    subprocess.call([sys.executable, "-c", CODE, lib])
