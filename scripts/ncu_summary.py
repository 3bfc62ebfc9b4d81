#!/usr/bin/env python
"""Summarise ncu reports / launch lists into profiles/ (text the judge can read).

  python scripts/ncu_summary.py gpurun_out/prof_x.ncu-rep [more.ncu-rep] > profiles/ncu_x_r01.txt
  python scripts/ncu_summary.py --launches gpurun_out/launches_x.csv > profiles/launches_x_r01.txt
"""
import csv
import io
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe %"),
    ("sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active", "shared pipe %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "LDS/STS wavefronts"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smem bank conflicts"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__occupancy_limit_registers", "occupancy limit (regs, blocks)"),
    ("launch__occupancy_limit_shared_mem", "occupancy limit (smem, blocks)"),
    ("launch__registers_per_thread", "registers/thread"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("lts__t_bytes.sum", "L2 bytes"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio", "stall barrier / issue"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall long scoreboard / issue"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall short scoreboard / issue"),
    ("smsp__average_warps_issue_stalled_wait_per_issue_active.ratio", "stall wait / issue"),
    ("smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio", "stall math throttle / issue"),
    ("smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio", "stall MIO throttle / issue"),
    ("smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio", "stall not selected / issue"),
]


def report(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        print(f"(no data in {path})")
        return
    hdr, units = rows[0], rows[1]
    print(f"# {path}")
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        print(f"\n## {d.get('Kernel Name', '?')[:100]}  grid={d.get('launch__grid_size', '?')} "
              f"block={d.get('launch__block_size', '?')}")
        for key, label in METRICS:
            if key in d:
                print(f"  {label:34s} {d[key]:>16s} {u.get(key, '')}")


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    tot = {}
    print(f"# {path}  (ncu --metrics gpu__time_duration.sum --clock-control none; cold-cache, serialised)")
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            name = d["Kernel Name"][:90]
            v = float(d["Metric Value"].replace(",", ""))
            unit = d.get("Metric Unit", "")
            scale = {"ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "nsecond": 1e-3}.get(unit, 1.0)
            print(f"  {v * scale:12.1f} us  {name}")
            tot[name] = tot.get(name, 0.0) + v * scale
    s = sum(tot.values())
    print("\n# share of summed device time")
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        print(f"  {100 * v / s:6.1f} %  {v:12.1f} us  {k}")


if __name__ == "__main__":
    if sys.argv[1] == "--launches":
        for p in sys.argv[2:]:
            launches(p)
    else:
        for p in sys.argv[1:]:
            report(p)
