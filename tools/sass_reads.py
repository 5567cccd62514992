"""Estimate register-file operand reads per pair in the hot loop (dev aid).

Model: an SMSP delivers ~2 32-bit register operands per lane
per cycle; FP64 sources read a register pair; an operand flagged .reuse on
the previous instruction in the same slot is served from the reuse cache.
"""
import os, re, subprocess, sys
sys.argv += [] 
pat = sys.argv[1]; unroll = int(sys.argv[2])
out = subprocess.run([sys.executable, os.path.join(os.path.dirname(__file__), "sass_loop.py"), pat, str(unroll), "-v"],
                     capture_output=True, text=True).stdout.splitlines()
body = [l for l in out if l and not l.startswith(" ") and not l.startswith("loop")]
FP64 = ("DFMA", "DMUL", "DADD", "DSETP")
tot = 0; prev_reuse = {}
per_op = {}
for ins in body:
    s = re.sub(r"^@!?U?P\w+\s+", "", ins)
    op = s.split()[0]; base = op.split(".")[0]
    args = s[len(op):].strip().rstrip(";").split(",")
    srcs = [a.strip() for a in args[1:]]  # first is destination (mostly)
    if base in ("ISETP", "DSETP", "PLOP3", "FSETP"):
        srcs = [a.strip() for a in args[2:]]
    reads = 0; new_reuse = {}
    for slot, a in enumerate(srcs):
        m = re.match(r"^-?\|?-?(R\d+)(\.reuse)?", a)
        if not m:
            continue
        reg = m.group(1)
        w = 2 if base in FP64 or (base == "F2I" and "F64" in op) or (base == "MUFU" and False) else 1
        if prev_reuse.get(slot) == reg:
            w = 0
        reads += w
        if m.group(2):
            new_reuse[slot] = reg
    prev_reuse = new_reuse
    tot += reads
    per_op[base] = per_op.get(base, 0) + reads
print("instructions %d, register reads %d -> %.1f reads/pair, %.1f cycles/pair at 2 reads/clk"
      % (len(body), tot, tot / unroll, tot / unroll / 2))
for k, v in sorted(per_op.items(), key=lambda kv: -kv[1]):
    print("  %-8s %5.1f reads/pair" % (k, v / unroll))
