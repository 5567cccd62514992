#!/bin/bash
# Mutation check of the oracle's pins (P10/P11): copy the tracked
# tree to a scratch dir, apply one plausible mistake to oracle/ep_oracle.cpp at a
# time, and run tests/test_oracle.py + the CPU half of tests/test_edge_pairs.py; every mutation must fail at least one pin.
#   bash tools/oracle_mutations.sh [scratch-dir]
set -u
ROOT=$(cd "$(dirname "$0")/.." && pwd); W=${1:-/tmp/oracle_mut}
rm -rf "$W"; mkdir -p "$W"; (cd "$ROOT" && git ls-files | grep -v '^profiles/' | tar cf - -T -) | tar xf - -C "$W"
python - "$W" <<'PY'
import sys
w = sys.argv[1]; src = open(w + "/oracle/ep_oracle.cpp").read()
muts = {
  "csum_plain": ("""    double t = s + v;
    if (std::fabs(s) >= std::fabs(v)) c += (s - t) + v;
    else c += (v - t) + s;
    s = t;""", "    s = s + v;"),
  "margin_never_updated": ("if (d < P->min_margin) P->min_margin = d;", "(void)d;"),
  "acceptance_strict": ("if (!(t1 <= 1.0)) return false;", "if (!(t1 < 1.0)) return false;"),
  "pair_order_swapped": ("gauss_pair(buf[2 * i], buf[2 * i + 1],", "gauss_pair(buf[2 * i + 1], buf[2 * i],"),
  "log_base2": ("std::sqrt(-2.0 * std::log(t1) / t1)", "std::sqrt(-2.0 * std::log2(t1) / t1)"),
  "bin_round_not_trunc": ("*l = (int64_t)std::fmax(std::fabs(*X), std::fabs(*Y));", "*l = (int64_t)std::nearbyint(std::fmax(std::fabs(*X), std::fabs(*Y)));"),
  "dropped_sy_term": ("P->sy.add(t4);", "P->sy.add(t4 * (l != 3));"),
}
for k, (a, b) in muts.items():
    if a not in src:
        print("SKIP", k, "(pattern not found)"); continue
    open(w + "/m_" + k + ".cpp", "w").write(src.replace(a, b, 1))
PY
rc=0
for m in "$W"/m_*.cpp; do
  name=$(basename "$m" .cpp); cp "$m" "$W/oracle/ep_oracle.cpp"; rm -f "$W/oracle/libep_oracle.so"
  out=$(cd "$W" && timeout 900 python -m pytest tests/test_oracle.py tests/test_edge_pairs.py -q -m "not gpu" -p no:cacheprovider 2>&1 | tail -1)
  case "$out" in *failed*) echo "$name: caught ($out)";; *) echo "$name: NOT CAUGHT ($out)"; rc=1;; esac
done
exit $rc
