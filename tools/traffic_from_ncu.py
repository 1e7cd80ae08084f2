"""Per-step DRAM traffic of each kernel group from one-step `ncu --set full`
captures (tools/profile_round.sh): writes profiles/<tag>_traffic.json, which
bench.py reads to fill roofline.traffic.
  python tools/traffic_from_ncu.py TAG REP_FP32 REP_BF16"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_table import rows  # noqa: E402

GROUPS = {"gemm_rows": ("k_tc3h_rows", "k_tc_rows", "k_tc16_rows"),
          "gemm_dw": ("k_tc3h_dw", "k_tc_dw2", "k_tc16_dw"),
          "spmm": ("k_spmm_fwd", "k_spmm_bwd"),
          "head": ("k_colsum", "k_score", "k_dz3")}


def summarise(rep):
    out = {}
    for e in rows(rep):
        grp = next((g for g, ks in GROUPS.items() if e["kernel"].startswith(ks)), None)
        if grp is None:
            continue
        o = out.setdefault(grp, {"dram_bytes_per_step": 0.0, "ncu_us_per_step": 0.0,
                                 "launches": 0, "kernels": []})
        b = (e.get("dram__bytes_read.sum", 0) + e.get("dram__bytes_write.sum", 0)) * 1e6
        o["dram_bytes_per_step"] += b
        o["ncu_us_per_step"] += e.get("gpu__time_duration.sum", 0)
        o["launches"] += 1
        o["kernels"].append({"kernel": e["kernel"], "dram_bytes": b,
                             "us": e.get("gpu__time_duration.sum")})
    return out


if __name__ == "__main__":
    tag, fp32, bf16 = sys.argv[1:4]
    res = {"source": f"ncu --set full --clock-control none, one step of the bench config "
                     f"(tools/profile_round.sh {tag}); cold-cache serialised replays",
           "fp32": summarise(fp32), "bf16": summarise(bf16)}
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                        "profiles", f"{tag}_traffic.json")
    json.dump(res, open(path, "w"), indent=1)
    for p in ("fp32", "bf16"):
        for g, o in res[p].items():
            print(p, g, f"{o['dram_bytes_per_step']/1e9:.3f} GB/step", f"{o['ncu_us_per_step']:.0f} us",
                  o["launches"])
