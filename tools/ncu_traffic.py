"""Write profiles/<kernel>_traffic_<cfg>_<dtype>.json from one `ncu --set full` capture:
DRAM bytes per launch and the headline counters bench.py's roofline quotes.

usage: python tools/ncu_traffic.py REPORT.ncu-rep KERNEL_TAG CFG DTYPE "source text"
"""
import csv
import json
import os
import subprocess
import sys

KEYS = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum", "smsp__inst_executed.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_sector_hit_rate.pct",
        "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_branch_resolving_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ms": 1, "us": 1e-3, "ns": 1e-6}


def main():
    rep, tag, cfg, dtype, source = sys.argv[1:6]
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    hdr, units, vals = rows[0], rows[1], rows[2]
    kernel = vals[hdr.index("Kernel Name")]
    got = {}
    for k in KEYS:
        if k in hdr:
            i = hdr.index(k)
            v = float(vals[i].replace(",", ""))
            got[k] = v * SCALE.get(units[i], 1)
    out = {"kernel": kernel, "workload": cfg, "dtype": dtype, "source": source,
           "dram_bytes_read": got.get("dram__bytes_read.sum"), "dram_bytes_write": got.get("dram__bytes_write.sum"),
           "dram_bytes_per_launch": got.get("dram__bytes_read.sum", 0) + got.get("dram__bytes_write.sum", 0),
           "duration_ms": got.get("gpu__time_duration.sum"), "metrics": got}
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                        f"{tag}_traffic_{cfg}_{dtype}.json")
    json.dump(out, open(path, "w"), indent=1)
    print(path, out["dram_bytes_per_launch"], out["duration_ms"])


if __name__ == "__main__":
    main()
