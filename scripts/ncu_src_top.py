#!/usr/bin/env python
"""Top SASS lines by warp-stall samples from an `ncu --page source --csv --print-source sass` dump."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ia, isrc, ismp, iex = hdr.index("Address"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
data = [(int(r[ismp] or 0), int(r[iex] or 0), r[ia], r[isrc].strip()) for r in rows[2:] if len(r) > ismp]
tot = sum(d[0] for d in data)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
print("total samples", tot)
base = int(data[0][2], 16)
# windows of 32 instructions
win = {}
for s, e, a, src in data:
    k = (int(a, 16) - base) // 0x200
    win[k] = win.get(k, 0) + s
for k in sorted(win, key=lambda k: -win[k])[:12]:
    print(f"window +0x{k*0x200:05x}: {100*win[k]/tot:5.1f}%")
for s, e, a, src in sorted(data, key=lambda d: -d[0])[:n]:
    print(f"{100*s/tot:5.1f}% {e:>10} +0x{int(a,16)-base:05x} {src}")
