"""Print the hot loop as a string of F (FP64) / i (other) and run statistics."""
import re, subprocess, sys, collections
lib = sys.argv[1]; pat = sys.argv[2] if len(sys.argv) > 2 else "ILi0ELb1ELi384ELi1ELi4E"
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
ins, on = [], False
for ln in out.splitlines():
    if "Function :" in ln:
        on = pat in ln; continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
    if on and m: ins.append((int(m.group(1), 16), m.group(2).strip()))
best = None
for addr, i in ins:
    m = re.search(r"BRA (?:!?U?P\d, )?0x([0-9a-f]+)", i)
    if m and int(m.group(1), 16) < addr:
        lo = int(m.group(1), 16)
        n = sum(1 for a, j in ins if lo <= a <= addr and "RSQ64H" in j)
        if n >= 6 and (best is None or addr - lo > best[1] - best[0]): best = (lo, addr)
lo, hi = best
s = ""
for a, i in ins:
    if lo <= a <= hi:
        op = re.sub(r"^@!?U?P\w+\s+", "", i).split()[0]
        s += "F" if op.split(".")[0] in ("DFMA", "DMUL", "DADD", "DSETP") else ("C" if op.startswith("CALL") else "i")
print(s)
runs = collections.Counter(len(r) for r in re.findall("F+", s))
print("F runs:", sorted(runs.items()))
