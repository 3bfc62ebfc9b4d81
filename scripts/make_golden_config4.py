#!/usr/bin/env python
"""Writes tests/golden/config4.json: the oracle's verdict on BASELINE config 4
(one 8192-nt RNA, Nussinov, h = 3, WC + GU, "run the oracle
once off-GPU for parity").

Calls only oracle/ (the memoised C recursion, oracle.c: orc_nussinov_traceback)
and dpgen/ (the seeded input). Nothing here comes from the CUDA path. Takes
~30-60 min single-threaded and ~300 MB (n x n int32 memo).

  python scripts/make_golden_config4.py [--n 8192]
"""
import argparse
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import dpgen  # noqa: E402
import oracle  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=8192)
    ap.add_argument("--out", default=os.path.join(ROOT, "tests", "golden", "config4.json"))
    args = ap.parse_args()
    x = dpgen.config4_rna8192(args.n)
    t = time.time()
    score, db = oracle.nussinov_traceback(x, dpgen.rna_pair_mask(), dpgen.NUSS_HAIRPIN)
    dt = time.time() - t
    rec = {
        "what": "BASELINE config 4: oracle score and canonical dot-bracket (DESIGN.md R-NUSS, R-TB-NUSS)",
        "generator": "dpgen.config4_rna8192(n) (seed 20120611+5), pairs AU/UA/GC/CG/GU/UG, h = 3",
        "written_by": "scripts/make_golden_config4.py (oracle/ only)",
        "n": args.n,
        "input_sha256": hashlib.sha256(x.tobytes()).hexdigest(),
        "score": int(score),
        "dotbracket_sha256": hashlib.sha256(db.encode()).hexdigest(),
        "dotbracket": db,
        "oracle_seconds": round(dt, 1),
    }
    with open(args.out, "w") as f:
        json.dump(rec, f, indent=1)
        f.write("\n")
    print(json.dumps({k: v for k, v in rec.items() if k != "dotbracket"}))


if __name__ == "__main__":
    main()
