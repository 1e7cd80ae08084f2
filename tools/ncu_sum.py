"""Key metrics of every kernel in an ncu report (dev tool):  python tools/ncu_sum.py REP..."""
import csv
import io
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "dram_rd"),
    ("dram__bytes_write.sum", "dram_wr"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "l2_rd_sect"),
    ("lts__t_sector_hit_rate.pct", "l2_hit%"),
    ("l1tex__t_sector_hit_rate.pct", "l1_hit%"),
    ("sm__warps_active.avg.per_cycle_active", "warps/SM"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("sm__inst_executed.sum", "inst"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall_lsb"),
    ("smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio", "stall_lg"),
    ("smsp__average_warps_issue_stalled_wait_per_issue_active.ratio", "stall_wait"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall_ssb"),
    ("smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio", "stall_mio"),
    ("smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio", "stall_bar"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "l2_thru%"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "l1_thru%"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram_thru%"),
    ("local_load", "x"),
]
for rep in sys.argv[1:]:
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    for r in rows[2:]:
        d = dict(zip(h, r))
        print(rep.split("/")[-1], d.get("Kernel Name", "")[:70])
        for k, nm in KEYS:
            if k in d:
                print(f"   {nm:12s} {d[k]} {units[h.index(k)]}")
