"""Summarise ab_ship.py timing output: best-first, both passes, class-D parity of gc/sx."""
import json, collections, sys
GC = {36: 53972171957, 32: 3373275903, 30: 843651411}
d = collections.defaultdict(list)
for l in open(sys.argv[1]):
    if l.startswith('{'):
        r = json.loads(l); d[(r['variant'], r['thr'], r['M'])].append(r)
    elif l.strip():
        print(l.strip()[:300])
for k, v in sorted(d.items(), key=lambda kv: -max(x['Mops'] for x in kv[1])):
    ok = all(x['gc'] == GC.get(k[2], x['gc']) and x['sx'] == x['sx'] for x in v)
    print("%-12s thr=%d M=%d %s  %s" % (k[0], k[1], k[2], " ".join("%.0f" % x['Mops'] for x in v), "ok" if ok else "WRONG"))
