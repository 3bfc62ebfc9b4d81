#!/usr/bin/env python
"""Instruction mix (+ stall samples) per opcode from an `ncu --page source --csv --print-source sass` dump.
   python scripts/ncu_mix.py dump.csv [kernel-substring]"""
import csv, sys
from collections import Counter
rows = list(csv.reader(open(sys.argv[1])))
kern = []; cur = None
for r in rows:
    if r and r[0] == "Kernel Name": cur = [r[1], None, []]; kern.append(cur); continue
    if r and r[0] == "Address": cur[1] = r; continue
    if cur and cur[1] and len(r) > 5: cur[2].append(r)
for name, hdr, data in kern:
    if len(sys.argv) > 2 and sys.argv[2] not in name: continue
    isrc, iex, ismp = hdr.index("Source"), hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
    tot = sum(int(r[iex] or 0) for r in data); stot = sum(int(r[ismp] or 0) for r in data)
    c = Counter(); cs = Counter()
    for r in data:
        s = r[isrc].strip()
        if not s: continue
        op = s.split()[1] if s.startswith('@') else s.split()[0]
        c[op] += int(r[iex] or 0); cs[op] += int(r[ismp] or 0)
    print(name[:80], "instructions", tot, "stall samples", stot)
    for k, v in c.most_common(40):
        print(f"  {k:28s} {100*v/tot:5.1f}%  stalls {100*cs[k]/max(stot,1):5.1f}%")
