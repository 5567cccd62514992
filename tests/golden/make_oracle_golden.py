"""Write tests/golden/oracle_ep.json: whole-run oracle results for the large NPB
classes, so that GPU parity tests at full size (B, C, D) do not have to rerun a
multi-minute CPU oracle on the GPU box.

Calls ONLY oracle/ (never the CUDA path).  Usage:
    python tests/golden/make_oracle_golden.py B C D [--threads N]
Existing entries for other classes are kept.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from ep_workloads import CLASSES, NPB_A, NPB_SEED  # noqa: E402

OUT = os.path.join(os.path.dirname(os.path.abspath(__file__)), "oracle_ep.json")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("classes", nargs="+")
    ap.add_argument("--threads", type=int, default=os.cpu_count())
    args = ap.parse_args()
    data = json.load(open(OUT)) if os.path.exists(OUT) else {}
    for c in args.classes:
        M = CLASSES[c]
        t0 = time.time()
        r = oracle.run(M, NPB_SEED, NPB_A, threads=args.threads, margin=True)
        dt = time.time() - t0
        data[c] = {
            "M": M, "seed": NPB_SEED, "a": NPB_A,
            "sx": r.sx.hex(), "sy": r.sy.hex(), "sx_dec": repr(r.sx), "sy_dec": repr(r.sy),
            "q": r.q, "gc": r.gc, "qbig": r.qbig, "npairs": r.npairs,
            "min_margin_ulp": r.min_margin_ulp,
            "oracle_seconds": round(dt, 2), "oracle_threads": args.threads,
            "writer": "tests/golden/make_oracle_golden.py (oracle/ only)",
        }
        print(c, json.dumps(data[c]), flush=True)
        with open(OUT, "w") as f:
            json.dump(data, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
