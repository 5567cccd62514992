"""Per-opcode stall attribution from an ncu source-page CSV (dev aid).

ncu -i rep --page source --csv --print-source sass > x.csv; python tools/ncu_stalls.py x.csv [top]
"""
import csv, sys, collections, re
rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
ix = {h: i for i, h in enumerate(hdr)}
cols = ["stall_math", "stall_dispatch", "stall_wait", "stall_not_selected", "stall_selected", "stall_short_sb", "stall_mio", "stall_branch_resolving"]
agg = collections.defaultdict(lambda: collections.Counter())
tot = collections.Counter()
hot = []
for r in data:
    src = r[1].strip()
    op = re.sub(r"^@!?U?P\w+\s+", "", src).split(" ")[0]
    n = int(r[ix["Instructions Executed"]] or 0)
    for c in cols:
        v = int(r[ix[c]] or 0)
        agg[op][c] += v
        tot[c] += v
    agg[op]["n"] += n
    hot.append((int(r[ix["# Samples"]] or 0), src, {c: int(r[ix[c]] or 0) for c in cols}))
T = sum(tot.values())
print("total samples", T, {c: round(tot[c] / T, 3) for c in cols})
print("%-22s %12s " % ("opcode", "executed") + " ".join("%9s" % c.replace("stall_", "")[:9] for c in cols))
for op, c in sorted(agg.items(), key=lambda kv: -sum(kv[1][x] for x in cols))[:25]:
    print("%-22s %12d " % (op[:22], c["n"]) + " ".join("%9.3f" % (c[x] / T) for x in cols))
if len(sys.argv) > 2:
    for s, src, d in sorted(hot, key=lambda t: -t[0])[:int(sys.argv[2])]:
        print(s, src, {k.replace("stall_", ""): v for k, v in d.items() if v})
