"""Classify the SASS of the EP kernel's hot loop (development aid).

python tools/sass_loop.py [kernel-substring] — finds the largest backward
branch loop in the kernel and counts instructions per pipe class per pair.
"""
import os, re, subprocess, sys, collections
lib = os.environ.get("HPL_LIB", "paper_conf_ipps_bozkusf12_b200/libhpl.so")
pat = sys.argv[1] if len(sys.argv) > 1 else "ep_kernelILi0ELb1"
unroll = int(sys.argv[2]) if len(sys.argv) > 2 else 4
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
lines, on = [], False
for ln in out.splitlines():
    if "Function :" in ln:
        on = pat in ln
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
    if on and m:
        lines.append((int(m.group(1), 16), m.group(2).strip()))
# smallest backward-branch loop containing >= unroll MUFU.RSQ64H (the hot loop)
best = None
for addr, ins in lines:
    m = re.search(r"BRA (?:!?U?P\d, )?0x([0-9a-f]+)", ins)
    if m:
        tgt = int(m.group(1), 16)
        if tgt < addr:
            n = sum(1 for a, i in lines if tgt <= a <= addr and "RSQ64H" in i)
            if n >= unroll and (best is None or addr - tgt < best[1] - best[0]):
                best = (tgt, addr)
lo, hi = best
# cold regions: bodies of forward conditional branches that contain a CALL (rare path)
cold = []
for a, ins in lines:
    m = re.search(r"^@!?U?P\w+\s+BRA (?:!?U?P\d, )?0x([0-9a-f]+)", ins)
    if m and lo <= a <= hi:
        t = int(m.group(1), 16)
        if t > a and any("CALL" in i for b, i in lines if a < b < t):
            cold.append((a, t))
body = [ins for a, ins in lines if lo <= a <= hi and not any(c0 < a < c1 for c0, c1 in cold)]
def cls(i):
    op = re.sub(r"^@!?U?P\w+\s+", "", i).split()[0]
    base = op.split(".")[0]
    if base in ("DFMA", "DMUL", "DADD", "DSETP", "DMNMX"): return "fp64"
    if base in ("MUFU", "F2I", "I2F", "F2F"): return "xu"
    if base in ("LDS", "STS", "LDL", "STL", "LDG", "STG", "ATOMS", "LDC"): return "mem"
    if base in ("IMAD", "HFMA2", "FFMA"): return "fma"
    if base in ("BRA", "BSSY", "BSYNC", "CALL", "RET", "WARPSYNC", "EXIT"): return "ctrl"
    return "alu/" + base
c = collections.Counter(cls(i) for i in body)
print("loop 0x%x-0x%x: %d instructions (%d per pair at unroll %d)" % (lo, hi, len(body), len(body) // unroll, unroll))
for k, v in sorted(c.items(), key=lambda kv: -kv[1]):
    print("  %-14s %4d  (%.2f / pair)" % (k, v, v / unroll))
if "-v" in sys.argv:
    print("\n".join(body))
