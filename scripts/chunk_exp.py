import os, sys, time, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import dpgen, paper_conf_pldi_carteylm12_b200 as dp
dev = torch.device("cuda:0")
n = 100_000
a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(n)
cu = lambda x: torch.from_numpy(np.ascontiguousarray(x)).to(dev)
A, AO, B, BO = cu(a_cat), cu(a_off), cu(b_cat), cu(b_off)
sig = dpgen.blosum62()
plans = [dp.Plan(dp.SW_LINEAR, 256, 256, sigma=sig, gap=dpgen.SW_GAP, want_traceback=True) for _ in range(2)]
streams = [torch.cuda.Stream(), torch.cuda.Stream()]
scores = torch.empty(n, dtype=torch.int32, device=dev)
out = torch.empty((n, 513), dtype=torch.uint8, device=dev)
ln = torch.empty(n, dtype=torch.int32, device=dev)
co = torch.empty((n, 4), dtype=torch.int32, device=dev)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
def step(nch):
    per = (n + nch - 1) // nch
    ev0 = torch.cuda.Event(); ev0.record()
    for c in range(nch):
        k0, k1 = c * per, min(n, (c + 1) * per)
        s = streams[c & 1]; p = plans[c & 1]
        s.wait_event(ev0)
        with torch.cuda.stream(s):
            p.solve_batch(A, AO[k0:k1 + 1], B, BO[k0:k1 + 1], max_len_a=256, max_len_b=256, out=scores[k0:k1], stream=s)
            p.traceback_into(0, k1 - k0, out[k0:k1], 513, ln[k0:k1], co[k0:k1], stream=s)
    for s in streams: torch.cuda.current_stream().wait_stream(s)
for nch in [1, 2, 4, 8, 16]:
    for _ in range(3): step(nch)
    torch.cuda.synchronize()
    ts = []
    for _ in range(10):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); step(nch); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    print(nch, round(sum(ts) / len(ts), 4), flush=True)
