#!/usr/bin/env python
"""DRAM traffic per launch of each dominant kernel (dram__bytes_read.sum + dram__bytes_write.sum from
one `ncu --set full` capture per config) -> profiles/traffic_<round>.json, read by bench.py for the
`roofline.traffic` field.

  python scripts/ncu_traffic.py OUT.json KERNEL=path.ncu-rep[:scale][:note] ...

scale: launches of the capture that make one bench launch (e.g. a 50k-problem capture of config 5
scaled to the 1M batch: 20); the JSON stores bytes per bench launch."""
import csv
import io
import json
import subprocess
import sys


def dram(path, name):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    for r in rows[2:]:
        d, u = dict(zip(hdr, r)), dict(zip(hdr, units))
        if name not in d.get("Kernel Name", ""):
            continue
        rd = float(d["dram__bytes_read.sum"].replace(",", "")) * mult.get(u["dram__bytes_read.sum"], 1)
        wr = float(d["dram__bytes_write.sum"].replace(",", "")) * mult.get(u["dram__bytes_write.sum"], 1)
        dur = d.get("gpu__time_duration.sum", "")
        return rd, wr, dur, u.get("gpu__time_duration.sum", "")
    raise SystemExit(f"{name} not in {path}")


def main():
    out = sys.argv[1]
    table = {}
    for arg in sys.argv[2:]:
        kern, rest = arg.split("=", 1)
        parts = rest.split(":")
        path = parts[0]
        scale = float(parts[1]) if len(parts) > 1 and parts[1] else 1.0
        note = parts[2] if len(parts) > 2 else ""
        rd, wr, dur, unit = dram(path, kern)
        table[kern] = {"bytes_per_launch": (rd + wr) * scale, "dram_read": rd * scale, "dram_write": wr * scale,
                       "capture": path.split("/")[-1], "capture_duration": f"{dur} {unit}",
                       "note": note or "ncu --set full --clock-control none, one launch"}
    with open(out, "w") as f:
        json.dump(table, f, indent=1)
    print(json.dumps(table, indent=1))


if __name__ == "__main__":
    main()
