"""Dev tool: one bench-config step (16 GNMT graphs, F = 64, H = 256, fp32)
through each given libmars.so in a fresh process; prints the loss and the
scaled max difference of the gradients against the first library's."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(path, out):
    sys.path.insert(0, ROOT)
    import numpy as np
    import paper_conf_icpp_lancl21_b200.mars as M
    M.LIB_PATH = path
    from synth import graphs as SG
    g = M.graph_load([SG.cached("gnmt", i) for i in range(16)])
    m = M.dgi_create(in_dim=64, hidden_dim=256, seed=0)
    r = m.step(g, 0, 0, want_loss=True, want_grads=True)
    np.save(out, r["grads"])
    print(json.dumps({"loss": r["loss"]}))


if __name__ == "__main__":
    if sys.argv[1] == "--child":
        child(sys.argv[2], sys.argv[3])
        sys.exit(0)
    import numpy as np
    ref = None
    for i, p in enumerate(sys.argv[1:]):
        out = f"/tmp/lib_compare_{i}.npy"
        r = subprocess.run([sys.executable, __file__, "--child", os.path.abspath(p), out],
                           capture_output=True, text=True, timeout=300)
        if r.returncode:
            print(os.path.basename(p), "FAILED", r.stderr[-300:])
            continue
        loss = json.loads(r.stdout.strip().splitlines()[-1])["loss"]
        gr = np.load(out).astype(np.float64)
        if ref is None:
            ref = gr
        err = np.abs(gr - ref).max() / np.abs(ref).max()
        print(f"{os.path.basename(p):24s} loss {loss:.8f}  grads vs first {err:.2e}", flush=True)
