"""Key metrics of an `ncu --page raw --csv` export (one launch), gzip or plain."""
import csv
import gzip
import json
import sys

p = sys.argv[1]
f = gzip.open(p, "rt") if p.endswith(".gz") else open(p)
r = list(csv.reader(f))
h, units, v = r[0], r[1], r[2]
want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "lts__t_requests_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
        "lts__t_sectors_srcunit_tex_op_red.sum", "lts__t_sectors_srcunit_tex_op_atom.sum",
        "launch__registers_per_thread", "launch__grid_size", "launch__occupancy_limit_registers",
        "smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct",
        "smsp__warp_issue_stalled_lg_throttle_per_warp_active.pct"]
out = {}
for w in want:
    if w in h:
        i = h.index(w)
        out[w] = v[i] + (f" {units[i]}" if units[i] else "")
print(json.dumps(out, indent=1))
