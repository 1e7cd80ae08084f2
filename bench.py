#!/usr/bin/env python
"""bench.py -- DGI contrastive pre-training throughput on GNMT-shaped op graphs.

Metric (BASELINE.json): "DGI contrastive steps/s on GNMT-shaped op graph; SpMM
GB/s vs HBM peak".  One bench step = one full pass of the hot path (corruption,
3 GCN layers on both branches, readout / discriminator / BCE, full backward,
NCCL gradient allreduce when N > 1, Adam) over a batch of 16 GNMT-shaped op
graphs per GPU (one (graph, sample) pair each, weak scaling).  `value` counts
per-graph DGI steps per second over the whole job (N x 16 x K / time).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
  torchrun --nproc-per-node N bench.py --gpus N ...   (one rank per GPU)

`--gpus N` without a torchrun environment re-launches itself under
`python -m torch.distributed.run --nproc-per-node N` (fails loudly if fewer
than N GPUs are visible).  Graphs are assigned to ranks by deterministic LPT
on their size (dp.lpt_assign), each keeping its global pair index; the
gradient exchange is libmars's peer-memory kernel (`--dp peer`, default) or
an NCCL allreduce (`--dp nccl`).

Device time: CUDA events on the stream the library launches on (torch's
current stream, handed to libmars), barrier + synchronize on both sides, max
over ranks.  The per-step working set (~2.8 GB of activations) exceeds the
126 MB L2, so no explicit flush is needed between steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "DGI contrastive steps/s on GNMT-shaped op graph; SpMM GB/s vs HBM peak"
UNIT = "graph-steps/s"
F, H = 64, 256
# BASELINE.json configs as bench workloads: generator, default graphs per GPU, F, H.
# "gnmt" is the metric's workload (the default line); the others are the
# configs[] rows measured the same way.  "1m" is ONE graph of ~1.1M ops: one
# GPU unsharded, or row-sharded over the ranks under torchrun.
WORKLOADS = {
    "gnmt": ("gnmt", 16, 64, 256, "GNMT-4 shaped training op graphs, T~U[20,50]"),
    "inception": ("inception", 16, 64, 128, "Inception-V3 shaped training op graphs"),
    "bert": ("bert", 8, 64, 256, "BERT-large shaped training op graphs"),
    "1m": ("1m", 1, 64, 256, "1.1M-op GNMT stress graph (T=3000)"),
}
FFMA_TFLOPS_NOTE = "148 SM x 128 FP32 lanes x 2 flop x 1.965 GHz (B200_PROFILING.md counts)"


def peaks():
    p = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "source": "fallback (B200_PROFILING.md)"}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            m = json.load(f)
        p.update(hbm_gbs=float(m["hbm_gbs"]), bf16_tflops=float(m["bf16_tflops"]),
                 bf16_tflops_sustained=float(m.get("bf16_tflops_sustained", m["bf16_tflops"])),
                 sm_max_mhz=float(m.get("sm_max_mhz", 1965.0)), source="measured")
    except Exception:
        pass
    p["ffma_tflops"] = 148 * 128 * 2 * p.get("sm_max_mhz", 1965.0) * 1e6 / 1e12
    return p


# ------------------------------------------------------------------ clocks sampler
class Clocks:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        with open(self.f.name) as fh:
            for ln in fh:
                parts = [x.strip() for x in ln.split(",")]
                if len(parts) < 9 or not parts[0].isdigit() or int(parts[0]) != self.idx:
                    continue
                rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        reasons = set()
        for r in rows:
            for name, col in (("hw_slowdown", 5), ("hw_thermal_slowdown", 6),
                              ("sw_thermal_slowdown", 7), ("sw_power_cap", 8)):
                if r[col].lower().startswith("active"):
                    reasons.add(name)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": float(rows[0][2]) if rows[0][2].replace(".", "").isdigit() else None,
                "reasons": sorted(reasons), "samples": len(rows)}


def ncu_traffic(prec: str, group: str):
    """DRAM bytes per step of a kernel group from the committed one-step
    `ncu --set full` capture (profiles/<tag>_traffic.json, written by
    tools/traffic_from_ncu.py); None when absent."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "*_traffic.json")))
    if not files:
        return None
    try:
        with open(files[-1]) as f:
            g = json.load(f)[prec][group]
        return float(g["dram_bytes_per_step"]), os.path.relpath(files[-1], ROOT)
    except Exception:
        return None


# ------------------------------------------------------------------ algorithmic bytes / flops
def spmm_bytes(N, Z, C, layer1=False, bwd=False, s=4, s_in=None):
    """Per SpMM launch over the stacked [pos; neg] rows:
    rowptr + (colind, val) + input rows + output rows (+ perm for layer 1,
    + Z read for the backward epilogue).  s = storage bytes per element,
    s_in = input element bytes when it differs (layer 1 reads fp32 X)."""
    s_in = s if s_in is None else s_in
    b = 4 * (N + 1) + 8 * Z + 2 * N * C * s_in + 2 * N * C * s
    if layer1:
        b += 4 * N
    if bwd:
        b += 2 * N * C * s
    return b


def step_accounting(N, Z, s=4):
    """Per-step launches of each phase with algorithmic bytes / flops."""
    R = 2 * N
    sp = [("spmm_fwd", spmm_bytes(N, Z, F, layer1=True, s=s, s_in=4)),
          ("spmm_fwd", spmm_bytes(N, Z, H, s=s)), ("spmm_fwd", spmm_bytes(N, Z, H, s=s)),
          ("spmm_bwd", spmm_bytes(N, Z, H, bwd=True, s=s)),
          ("spmm_bwd", spmm_bytes(N, Z, H, bwd=True, s=s))]
    gemm = {"gemm_fwd": 2 * R * H * (F + H + H), "gemm_dw": 2 * R * H * (F + H + H),
            "gemm_dy": 2 * R * H * (H + H)}
    gemm_bytes = {"gemm_fwd": s * R * ((F + H) + (H + H) + (H + H)),
                  "gemm_dw": s * R * ((F + H) + (H + H) + (H + H)),
                  "gemm_dy": s * R * ((H + H) + (H + H))}
    return sp, gemm, gemm_bytes


# ------------------------------------------------------------------ arms
def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def host_info():
    """os.cpu_count() and the CPU model (lscpu), for the CPU-baseline lines."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name:"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return {"cpu_count": os.cpu_count(), "model": model}


def oracle_step_seconds(oracle, graphs, H, seed=0):
    """Wall seconds of one full fp64 oracle DGI step + Adam on `graphs`."""
    b = oracle.Batch(graphs)
    p = oracle.xavier(seed, b.F, H).astype(np.float64)
    t0 = time.perf_counter()
    loss, grads, _, _ = oracle.step_grads(b, H, p, b.perms(seed, 0, 0))
    oracle.adam(p, np.zeros_like(p), np.zeros_like(p), grads, 1)
    return time.perf_counter() - t0


def run_reference(args):
    """The oracle (fp64; its OpenMP build on every host core) as it stands."""
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    import oracle
    oracle.set_variant("omp")
    from synth import graphs as SG
    gen = WORKLOADS[args.workload][0]
    if args.workload == "1m":      # one GNMT graph stands in: a 1.1M-op fp64 step takes ~10 min
        gen = "gnmt"
    graphs = [SG.cached(gen, i) for i in range(args.graphs_per_gpu)]
    small = min(graphs, key=lambda g: g.num_nodes)
    tiny = SG.tiny(0)
    for w in range(args.warmup):                      # untimed (CPU has nothing to warm up)
        b = oracle.Batch([tiny])
        oracle.step_grads(b, 32, oracle.xavier(0, 16, 32).astype(np.float64), b.perms(0, w, 0))
    b = oracle.Batch([small])
    p = oracle.xavier(0, F, H).astype(np.float64)
    m = np.zeros_like(p); v = np.zeros_like(p)
    t0 = time.perf_counter()
    for k in range(args.steps):
        loss, grads, _, _ = oracle.step_grads(b, H, p, b.perms(0, k, 0))
        p, m, v = oracle.adam(p, m, v, grads, k + 1)
    dt = time.perf_counter() - t0
    val = args.steps / dt
    sample = (f"1 {gen}-shaped graph per step (the smallest of the workload's "
              f"{args.graphs_per_gpu}, N={small.num_nodes}), full DGI step + Adam in fp64, "
              f"OpenMP build on {os.cpu_count()} host threads")
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * dt / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"{args.workload} x{args.graphs_per_gpu} per GPU "
                                   f"(sampled: 1 graph/step)", "F": F, "H": H},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": os.cpu_count(), "kind": "oracle",
                             "sample": sample, "host": host_info()},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_mine(args):
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_lancl21_b200 as mars
    from paper_conf_icpp_lancl21_b200 import dp
    from synth import graphs as SG

    rank, world, local = dp.env()
    if world > 1:                     # NCCL communicator lines (incl. nranks) in the log
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    b = args.graphs_per_gpu
    gen, _, _, _, desc = WORKLOADS[args.workload]
    sharded = args.workload == "1m" and world > 1
    mine = [0]
    if args.workload == "1m":
        graphs = [SG.make("1m", 0)]           # ~7 s to generate; one graph for the whole job
    else:
        # LPT on graph size over the job's world*b graphs; graph i keeps pair index i
        costs = [dp.graph_cost(SG.cached(gen, i)) for i in range(world * b)]
        mine = dp.lpt_assign(costs, world, b)[rank]
        graphs = [SG.cached(gen, i) for i in mine]
    if sharded:
        # rank r owns row block r of the one graph; the peers'
        # activation buffers are opened over CUDA IPC (NVLink peer memory)
        g = mars.graph_load_shard(graphs[0], world, rank, device=local)
        m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=args.seed, device=local)
        mars.shard_attach(m, g)
        blobs = [None] * world
        dist.all_gather_object(blobs, mars.shard_export(m))
        mars.shard_connect(m, blobs)
        shard_info = mars.graph_shard_info(g)
        uid = None
    else:
        uid = dp.broadcast_unique_id(mars.nccl_get_unique_id) if args.dp == "nccl" else None
        g = mars.graph_load(graphs, device=local)
        g.set_pair_offsets(mine)
        m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=args.seed, device=local, world_size=world,
                            rank=rank, nccl_unique_id=uid)
        if world > 1 and args.dp == "peer":
            dp.connect_peers(m)
        shard_info = None
    info = g.info()
    if not sharded:
        m.set_gemm_impl(args.gemm)
    # a dedicated (non-legacy) stream: libmars launches and captures on it and
    # torch's CUDA events are recorded on it
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    m.set_stream(stream.cuda_stream)
    base, B = (0, 1) if sharded else (0, world * b)
    for w in range(args.warmup):
        m.step(g, w, base, B)
    torch.cuda.synchronize()
    phys = local
    cvd = os.environ.get("CUDA_VISIBLE_DEVICES")
    if cvd:
        try:
            phys = int(cvd.split(",")[local])
        except Exception:
            pass
    clk = Clocks(phys)
    time.sleep(0.3)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    # one event between consecutive steps: the whole region for the value, the
    # per-step spread for the p10 / p50 / p90 report
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    evs[0].record(stream)
    for k in range(args.steps):
        m.step(g, args.warmup + k, base, B)
        evs[k + 1].record(stream)
    evs[-1].synchronize()
    ms = evs[0].elapsed_time(evs[-1])
    step_ms = np.array([evs[k].elapsed_time(evs[k + 1]) for k in range(args.steps)])
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks = clk.stop()
    launches = m.last_launches() * args.steps
    if world > 1:
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    # graph-steps per second of the whole job (the sharded 1m job is ONE graph)
    value = (1 if sharded else world * b) * args.steps / (ms / 1000.0)

    # per-phase device time, CUDA events on the launching stream (same kernels, eager)
    nprof = max(1, min(args.steps, args.profile_steps))
    acc = {}
    prof_total = 0.0
    for k in range(nprof):
        ph = m.profile_step(g, args.warmup + args.steps + k, base, B)
        for name, t in ph:
            acc.setdefault(name, []).append(t)
        prof_total += sum(t for _, t in ph)
    per_step = {k: sum(v) / nprof for k, v in acc.items()}
    N, Z = info["total_nodes"], info["nnz"]
    if sharded:                       # per-rank accounting: the owned rows and their nnz
        N = shard_info["row_end"] - shard_info["row_begin"]
        Z = shard_info["local_nnz"]
    sp, gflops, gbytes = step_accounting(N, Z)
    pk = peaks()
    spmm_ms = per_step.get("spmm_fwd", 0) + per_step.get("spmm_bwd", 0)
    spmm_algo = sum(bb for _, bb in sp)
    spmm_gbs = spmm_algo / (spmm_ms / 1e3) / 1e9 if spmm_ms else None
    shares = {k: v / sum(per_step.values()) for k, v in per_step.items()}
    step_total = sum(per_step.values())
    rows_ms = per_step.get("gemm_fwd", 0) + per_step.get("gemm_dy", 0)
    dw_ms = per_step.get("gemm_dw", 0)
    head_ms = per_step.get("head", 0)
    auto = args.gemm == "auto"
    # Row GEMMs (Z = Y·W, dY = dZ·Wᵀ): 3xFP16 on kind::f16 -- fp32-equivalent
    # tensor peak bf16 / 3 = ~540 TF/s, ridge ~83 flop/B above their 64 flop/B
    # (fp32 operands), so HBM bounds them: algorithmic bytes R·(K+N)·4 per GEMM.
    rows_bytes = gbytes["gemm_fwd"] + gbytes["gemm_dy"]
    rows_flops = gflops["gemm_fwd"] + gflops["gemm_dy"]
    rows_gbs = rows_bytes / (rows_ms / 1e3) / 1e9 if rows_ms else None
    # Weight gradient (dW = Yᵀ·dZ): 3xFP16 as well, same intensity (<= 64 flop/B
    # against the ~83 flop/B ridge), so also HBM-bound: R·(Cin+H)·4 per GEMM.
    dw_bytes = gbytes["gemm_dw"]
    dw_gbs = dw_bytes / (dw_ms / 1e3) / 1e9 if dw_ms else None
    dw_ach = gflops["gemm_dw"] / (dw_ms / 1e3) / 1e12 if dw_ms else None
    head_bytes = 16 * N * H                     # Z3 in, dZ3 out (stacked pos/neg)
    head_gbs = head_bytes / (head_ms / 1e3) / 1e9 if head_ms else None
    if auto:
        gemm_rows = {"kernel": "row GEMMs Z = Y·W, dY = dZ·Wᵀ (tcgen05 3xFP16, k_tc3h_rows)",
                     "bound": "hbm", "achieved": rows_gbs, "peak": pk["hbm_gbs"], "unit": "GB/s",
                     "frac": rows_gbs / pk["hbm_gbs"] if rows_gbs else None, "traffic": None,
                     "peak_source": pk["source"], "algorithmic_bytes_per_step": rows_bytes,
                     "achieved_tflops_fp32_equiv": rows_flops / (rows_ms / 1e3) / 1e12 if rows_ms else None,
                     "share_of_step": rows_ms / step_total}
    else:
        ach = rows_flops / (rows_ms / 1e3) / 1e12 if rows_ms else None
        gemm_rows = {"kernel": "row GEMMs (FFMA)", "bound": "alu", "achieved": ach,
                     "peak": pk["ffma_tflops"], "unit": "TFLOP/s",
                     "frac": ach / pk["ffma_tflops"] if ach else None, "traffic": None,
                     "peak_source": FFMA_TFLOPS_NOTE, "share_of_step": rows_ms / step_total}
    rooflines = {
        "gemm_rows": gemm_rows,
        "gemm_dw": ({"kernel": "weight gradient dW = Yᵀ·dZ (tcgen05 3xFP16, k_tc3h_dw)",
                     "bound": "hbm", "achieved": dw_gbs, "peak": pk["hbm_gbs"], "unit": "GB/s",
                     "frac": dw_gbs / pk["hbm_gbs"] if dw_gbs else None, "traffic": None,
                     "peak_source": pk["source"], "algorithmic_bytes_per_step": dw_bytes,
                     "achieved_tflops_fp32_equiv": dw_ach, "share_of_step": dw_ms / step_total}
                    if auto else
                    {"kernel": "weight gradient dW = Yᵀ·dZ (FFMA)", "bound": "alu",
                     "achieved": dw_ach, "peak": pk["ffma_tflops"], "unit": "TFLOP/s",
                     "frac": dw_ach / pk["ffma_tflops"] if dw_ach else None, "traffic": None,
                     "peak_source": FFMA_TFLOPS_NOTE, "share_of_step": dw_ms / step_total}),
        "spmm": {"kernel": "spmm (fwd x3 + bwd x2)", "bound": "hbm", "achieved": spmm_gbs,
                 "peak": pk["hbm_gbs"], "unit": "GB/s",
                 "frac": spmm_gbs / pk["hbm_gbs"] if spmm_gbs else None, "traffic": None,
                 "peak_source": pk["source"], "share_of_step": spmm_ms / step_total},
        "head": {"kernel": "head (readout, scores, BCE, head backward, dZ3)", "bound": "hbm",
                 "achieved": head_gbs, "peak": pk["hbm_gbs"], "unit": "GB/s",
                 "frac": head_gbs / pk["hbm_gbs"] if head_gbs else None, "traffic": None,
                 "peak_source": pk["source"], "share_of_step": head_ms / step_total},
    }
    algo_bytes = {"gemm_rows": rows_bytes, "gemm_dw": gbytes["gemm_dw"], "spmm": spmm_algo,
                  "head": head_bytes}
    for grp, r in rooflines.items():
        t = ncu_traffic("fp32", grp)
        if t is not None:
            r["traffic"] = t[0]
            r["traffic_note"] = (f"DRAM read+write bytes per step of the group, ncu --set full ({t[1]}); "
                                 f"algorithmic bytes per step {algo_bytes[grp]:.4g}")
    roof = max(rooflines.values(), key=lambda r: r["share_of_step"])
    spmm_obj = {"achieved_gbs": spmm_gbs, "peak_gbs": pk["hbm_gbs"],
                "frac": (spmm_gbs / pk["hbm_gbs"]) if spmm_gbs else None,
                "algorithmic_bytes_per_step": spmm_algo, "ms_per_step": spmm_ms,
                "peak_source": pk["source"]}

    # e2e through the public API: H2D of the step's graph batch from host memory,
    # CSR build, the step, D2H of the loss -- every step
    e2e = None
    if not args.no_e2e and not sharded:
        # the step's inputs live in page-locked host memory (a data loader's
        # pinned batch); libmars copies them straight to the device
        class _Pinned:
            pass
        pinned = []
        for gr in graphs:
            pg = _Pinned()
            pg.num_nodes = gr.num_nodes
            pg.indptr = torch.from_numpy(np.ascontiguousarray(gr.indptr)).pin_memory().numpy()
            pg.indices = torch.from_numpy(np.ascontiguousarray(gr.indices)).pin_memory().numpy()
            pg.features = torch.from_numpy(np.ascontiguousarray(gr.features)).pin_memory().numpy()
            pinned.append(pg)
        offs = np.ascontiguousarray(mine, np.int64)
        h2d = sum(gr.indptr.nbytes + gr.indices.nbytes + gr.features.nbytes for gr in pinned)
        ke = max(1, min(args.steps, args.e2e_steps))
        m2 = mars.dgi_create(in_dim=F, hidden_dim=H, seed=args.seed, device=local,
                             world_size=1, rank=0)
        m2.set_gemm_impl(args.gemm)
        m2.set_stream(stream.cuda_stream)
        gg = mars.graph_load(pinned, device=local)          # warm allocator pool
        gg.set_pair_offsets(offs)
        m2.step(gg, 0, base, B, want_loss=True)
        gg.free()
        torch.cuda.synchronize()
        # A data loader's double buffer: two graph-set handles; while step k runs
        # on one, the next batch is reloaded into the other (mars_graph_reload:
        # H2D of the pinned batch + CSR build on libmars's loader stream, after
        # the device-side wait for the step that last read that handle), then
        # step k's loss is read back (D2H).  Every step's inputs are copied and
        # rebuilt inside the timed region; the steps replay each handle's
        # captured CUDA Graph.
        ga = mars.graph_load(pinned, device=local)
        ga.set_pair_offsets(offs)
        gb = mars.graph_load(pinned, device=local)
        gb.set_pair_offsets(offs)
        for k in range(4):                                   # capture both handles
            m2.step(ga if k % 2 == 0 else gb, 100 + k, base, B)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        cur, nxt = ga, gb
        cur.reload(pinned)
        losses, prev = [], None
        for k in range(ke):
            m2.step(cur, 1 + k, base, B)
            tk = m2.enqueue_loss()                   # D2H of step k's loss, asynchronous
            if k + 1 < ke:
                nxt.reload(pinned)
            if prev is not None:                     # the host reads step k-1's loss while
                losses.append(m2.wait_loss(prev))    # step k runs (one-step logging lag)
            prev = tk
            cur, nxt = nxt, cur
        losses.append(m2.wait_loss(prev))
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        if len(losses) != ke or not all(np.isfinite(losses)):
            raise RuntimeError("e2e: a step's loss was not read back or is not finite")
        m2.free()
        ga.free()
        gb.free()
        e2e = {"value": b * ke / dt, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": 4, "steps": ke,
               "note": "per step: mars_graph_reload of a double-buffered graph handle (H2D from "
                       "pinned host memory + CSR build on libmars's loader stream, overlapping "
                       "the previous step's compute) + mars_dgi_step (captured graph replay) + "
                       "loss D2H (mars_dgi_enqueue_loss after the step; the host reads it with "
                       "mars_dgi_wait_loss while the next step runs, every step's loss checked "
                       "finite); wall clock, rank-local (no allreduce)"}

    # the bf16 path (MARS_BF16, 2e-2 parity bar) on the same workload, same timing
    b16 = None
    if not args.no_bf16 and not sharded:
        m16 = mars.dgi_create(in_dim=F, hidden_dim=H, seed=args.seed, device=local,
                              world_size=world, rank=rank, nccl_unique_id=uid,
                              precision=mars.MARS_BF16) if world == 1 else None
        if m16 is not None:
            m16.set_stream(stream.cuda_stream)
            for w in range(args.warmup):
                m16.step(g, w, base, B)
            torch.cuda.synchronize()
            ev0, ev1 = evs[0], evs[-1]
            ev0.record(stream)
            for k in range(args.steps):
                m16.step(g, args.warmup + k, base, B)
            ev1.record(stream)
            ev1.synchronize()
            ms16 = ev0.elapsed_time(ev1)
            acc16 = {}
            for k in range(nprof):
                for name, t in m16.profile_step(g, 10**6 + k, base, B):
                    acc16.setdefault(name, []).append(t)
            ps16 = {k: sum(v) / nprof for k, v in acc16.items()}
            sp16 = ps16.get("spmm_fwd", 0) + ps16.get("spmm_bwd", 0)
            sp16_bytes = sum(bb for _, bb in step_accounting(N, Z, s=2)[0])
            b16 = {"value": world * b * args.steps / (ms16 / 1000.0), "unit": UNIT,
                   "ms_per_step": ms16 / args.steps, "dtype": "bf16",
                   "phases_ms_per_step": ps16,
                   "spmm_gbs": sp16_bytes / (sp16 / 1e3) / 1e9 if sp16 else None,
                   "spmm_frac": (sp16_bytes / (sp16 / 1e3) / 1e9 / pk["hbm_gbs"]) if sp16 else None,
                   "spmm_traffic": (ncu_traffic("bf16", "spmm") or (None,))[0],
                   "spmm_algorithmic_bytes_per_step": sp16_bytes,
                   "note": "bf16 activations + bf16 tcgen05 MMAs, fp32 accumulation and "
                           "master params; parity bar 2e-2 (tests/test_gpu_bf16.py)"}
            m16.free()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and args.workload != "1m":
        import oracle
        # a bounded sample of the workload: whole graphs of the step, one at a
        # time, with the oracle's OpenMP build on every host core, until ~10 s
        old = oracle.set_variant("omp")
        p0 = oracle.xavier(args.seed, F, H).astype(np.float64)
        t0 = time.perf_counter()
        done = 0
        for gr0 in graphs[:4]:
            bo = oracle.Batch([gr0])
            loss, grads, _, _ = oracle.step_grads(bo, H, p0, bo.perms(args.seed, 0, done))
            oracle.adam(p0, np.zeros_like(p0), np.zeros_like(p0), grads, 1)
            done += 1
            if time.perf_counter() - t0 > 10.0:
                break
        dt = time.perf_counter() - t0
        # SURVEY §8(d)'s oracle table: seconds per step of one graph of each
        # config, OpenMP (all cores) and serial, beside the GPU's per-graph time
        table = {}
        for name, Fc, Hc in (("tiny", 16, 32), ("inception", 64, 128), ("gnmt", 64, 256),
                             ("bert", 64, 256)):
            g1 = [SG.tiny(0)] if name == "tiny" else [SG.cached(name, 0)]
            row = {"N": g1[0].num_nodes, "F": Fc, "H": Hc,
                   "omp_s": oracle_step_seconds(oracle, g1, Hc)}
            oracle.set_variant("serial")
            row["serial_s"] = oracle_step_seconds(oracle, g1, Hc)
            oracle.set_variant("omp")
            table[name] = row
        oracle.set_variant(old)
        cpu = {"value": done / dt, "unit": UNIT, "cores": os.cpu_count(), "kind": "oracle",
               "sample": f"{done} of the {b} {gen}-shaped graphs of a step (graphs 0..{done - 1}, "
                         f"N={sum(x.num_nodes for x in graphs[:done])}), full fp64 DGI step + Adam, "
                         f"OpenMP build of the oracle on {os.cpu_count()} threads, {dt:.1f} s",
               "host": host_info(), "oracle_s_per_step": table,
               "gpu_s_per_graph_step": (ms / args.steps / 1000.0) / b}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
                "higher_is_better": True, "scaling": "strong" if sharded else "weak",
                "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": (f"{args.workload}: one graph, row-sharded over {world} GPUs "
                                        f"({desc})" if sharded else
                                        f"{args.workload} x{b} per GPU ({desc})"),
                           "graphs_per_gpu": b, "F": F, "H": H,
                           "nodes_per_gpu": N, "nnz_per_gpu": Z, "global_batch": B,
                           "parallelism": f"rowshard{world}" if sharded else f"dp{world}",
                           "dp_exchange": None if sharded or world == 1 else
                           ("libmars peer-memory kernel (rank-ordered fp64 sum over NVLink, "
                            "2 device barriers)" if args.dp == "peer" else "NCCL allreduce"),
                           "graph_assignment": None if sharded else "LPT on N+2E, global pair ids",
                           "shard": shard_info,
                           "l2": (("inputs larger than L2 (activations ~%.2f GB/step)"
                                   if 2 * N * 4 * (F + 7 * H) > 126e6 else
                                   "working set ~%.2f GB fits the 126 MB L2: a latency-bound "
                                   "small-config number, no flush")
                                  % (2 * N * 4 * (F + 7 * H) / 1e9))},
                "roofline": roof, "rooflines": rooflines, "spmm": spmm_obj,
                "phases_ms_per_step": per_step, "phase_share": shares,
                "profiled_step_ms": prof_total / nprof,
                "step_ms_percentiles": {"p10": float(np.percentile(step_ms, 10)),
                                        "p50": float(np.percentile(step_ms, 50)),
                                        "p90": float(np.percentile(step_ms, 90)),
                                        "of": "rank 0's timed steps (events between steps)"},
                "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks, "gpu_launches": launches,
                "bf16": b16}
        print(json.dumps(line), flush=True)
    m.free()
    g.free()
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="mine", choices=["mine", "reference"])
    ap.add_argument("--workload", default="gnmt", choices=sorted(WORKLOADS),
                    help="gnmt (the metric's workload, default), inception, bert, or 1m "
                         "(one 1.1M-op graph; row-sharded under torchrun)")
    ap.add_argument("--graphs-per-gpu", type=int, default=None)
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--gemm", default="auto", choices=["auto", "simt"],
                    help="dense-transform kernels: tcgen05 3xFP16 with power-of-two scaling (auto) or FFMA (simt)")
    ap.add_argument("--profile-steps", type=int, default=5)
    ap.add_argument("--e2e-steps", type=int, default=40)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-bf16", action="store_true", help="skip the bf16-path measurement")
    ap.add_argument("--dp", default="peer", choices=["peer", "nccl"],
                    help="gradient exchange for N > 1: libmars peer-memory kernel or NCCL allreduce")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    global F, H
    _, bdef, F, H, _ = WORKLOADS[args.workload]
    if args.graphs_per_gpu is None:
        args.graphs_per_gpu = bdef
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch(args)
    if args.impl == "reference":
        return run_reference(args)
    return run_mine(args)


def relaunch(args):
    """`--gpus N` outside torchrun: one rank per GPU under torch.distributed.run."""
    import socket
    try:
        import torch
        ngpu = torch.cuda.device_count()
    except Exception:
        ngpu = 0
    if ngpu < args.gpus:
        print(f"bench.py: --gpus {args.gpus} needs {args.gpus} visible GPUs, found {ngpu}",
              file=sys.stderr, flush=True)
        return 2
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")            # communicator lines (nranks) in the log
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr=127.0.0.1", f"--master-port={port}",
           os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd, env=env)


if __name__ == "__main__":
    sys.exit(main())
