"""One line per kernel launch of an `ncu --set full` report: duration, DRAM
bytes, L2 / L1 hit rates, achieved occupancy, tensor-pipe utilisation.
  python tools/ncu_table.py REP [--json OUT]"""
import csv
import io
import json
import re
import subprocess
import sys

COLS = [
    ("gpu__time_duration.sum", "us"),
    ("dram__bytes_read.sum", "MB"),
    ("dram__bytes_write.sum", "MB"),
    ("lts__t_sector_hit_rate.pct", "%"),
    ("l1tex__t_sector_hit_rate.pct", "%"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "%"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "%"),
    ("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "%"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "%"),
    ("launch__registers_per_thread", ""),
]
SCALE = {("byte", "MB"): 1e-6, ("Kbyte", "MB"): 1e-3, ("Mbyte", "MB"): 1.0, ("Gbyte", "MB"): 1e3,
         ("nsecond", "us"): 1e-3, ("usecond", "us"): 1.0, ("msecond", "us"): 1e3}


def short(name):
    m = re.search(r"(k_\w+)(<[^(]*>)?", name)
    return (m.group(1) + (m.group(2) or "")) if m else name[:40]


def rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    h, units = r[0], r[1]
    res = []
    for row in r[2:]:
        d = dict(zip(h, row))
        e = {"kernel": short(d.get("Kernel Name", ""))}
        for k, want in COLS:
            if k not in d or d[k] in ("", "n/a"):
                continue
            v = float(d[k].replace(",", ""))
            u = units[h.index(k)]
            v *= SCALE.get((u, want), 1.0)
            e[k] = v
        res.append(e)
    return res


if __name__ == "__main__":
    res = rows(sys.argv[1])
    hdr = ["time_us", "dram_rd_MB", "dram_wr_MB", "L2hit%", "L1hit%", "warps%", "tensor%", "dram%"]
    print(f"{'kernel':44s} " + " ".join(f"{x:>10s}" for x in hdr))
    for e in res:
        t = e.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
                  e.get("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", float("nan")))
        vals = [e.get("gpu__time_duration.sum"), e.get("dram__bytes_read.sum"),
                e.get("dram__bytes_write.sum"), e.get("lts__t_sector_hit_rate.pct"),
                e.get("l1tex__t_sector_hit_rate.pct"),
                e.get("sm__warps_active.avg.pct_of_peak_sustained_active"), t,
                e.get("dram__throughput.avg.pct_of_peak_sustained_elapsed")]
        print(f"{e['kernel'][:44]:44s} " + " ".join(
            f"{v:10.1f}" if isinstance(v, float) else f"{'-':>10s}" for v in vals))
    if len(sys.argv) > 3 and sys.argv[2] == "--json":
        json.dump(res, open(sys.argv[3], "w"), indent=1)
