"""Per-pair instruction mix and register-read model of the pipelined EP hot loop.

python tools/sass_hot.py [lib] [kernel-substring] [pairs-per-iteration]

Finds the backward branch whose body holds the most MUFU.RSQ64H (the
pipelined group loop), drops the cold rare-path regions (from each
`BRA.DIV` / warp-vote branch to its join), and prints per pair: instruction
counts by opcode and an estimate of 32-bit register-file reads (FP64
sources read a register pair; an operand served by the .reuse cache of the
previous instruction in the same slot is free; uniform registers, constants
and immediates are free).  Development aid for DESIGN.md §5.
"""
import collections
import re
import subprocess
import sys

lib = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_ipps_bozkusf12_b200/libhpl.so"
pat = sys.argv[2] if len(sys.argv) > 2 else "ILi0ELb1ELi384ELi1ELi4E"
ppi = int(sys.argv[3]) if len(sys.argv) > 3 else 16
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
ins, on = [], False
for ln in out.splitlines():
    if "Function :" in ln:
        on = pat in ln
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
    if on and m:
        ins.append((int(m.group(1), 16), m.group(2).strip()))
best = None
for addr, i in ins:
    m = re.search(r"BRA (?:!?U?P\d, )?0x([0-9a-f]+)", i)
    # the loop's back edge is conditional (@P BRA); unconditional backward
    # branches are the rare paths' returns into the loop body
    if m and int(m.group(1), 16) < addr and i.startswith("@"):
        lo = int(m.group(1), 16)
        n = sum(1 for a, j in ins if lo <= a <= addr and "RSQ64H" in j)
        # the pipelined group loop holds exactly one MUFU per pair of an
        # iteration (ppi); among such loops take the smallest
        if n == ppi and (best is None or addr - lo < best[1] - best[0]):
            best = (lo, addr, n)
lo, hi, _ = best
body = [(a, i) for a, i in ins if lo <= a <= hi]
# cold regions: after a BRA.DIV the code up to the target of the next "@!P BRA" that skips
# the rare calls; simplest robust rule: drop every instruction between a VOTE.ANY-guarded
# branch and the farthest forward target of branches in that block containing a CALL.
cold = set()
for k, (a, i) in enumerate(body):
    m = re.search(r"@!?P\d BRA 0x([0-9a-f]+)", i)
    if m and int(m.group(1), 16) > a:
        tgt = int(m.group(1), 16)
        region = [(b, j) for b, j in body if a < b < tgt]
        if any("CALL" in j for b, j in region):
            cold.update(b for b, j in region)
hot = [(a, i) for a, i in body if a not in cold]
FP64 = ("DFMA", "DMUL", "DADD", "DSETP", "DMNMX")
mix = collections.Counter()
reads = collections.Counter()
prev_reuse = {}
bank_cyc = 0.0  # RF-bank issue model: max(distinct even, distinct odd) registers read, >= 1
for a, i in hot:
    s = re.sub(r"^@!?U?P\w+\s+", "", i)
    op = s.split()[0]
    base = op.split(".")[0]
    mix[op] += 1
    args = [x.strip() for x in s[len(op):].split(",")]
    nd = 2 if base in ("ISETP", "DSETP", "FSETP", "PLOP3") else 1
    if base in ("STS", "ST", "STG", "RED", "ATOMS"):
        nd = 0
    srcs = args[nd:]
    new_reuse = {}
    regs = set()
    for slot, x in enumerate(srcs):
        m = re.match(r"^\[?-?\|?-?(R\d+)\|?(\.reuse)?", x)
        if not m or m.group(1) == "RZ":
            continue
        w = 2 if (base in FP64 or (base == "MUFU" and "64" in op)) else 1
        if base == "LDS" or base == "IMAD" and "WIDE" in op and slot == 2:
            w = 1 if base == "LDS" else w
        if prev_reuse.get(slot) == m.group(1):
            w = 0
        reads[base] += w
        if w:
            r0 = int(m.group(1)[1:])
            regs.update(range(r0, r0 + w))
        if m.group(2):
            new_reuse[slot] = m.group(1)
    prev_reuse = new_reuse
    ev = sum(1 for r in regs if r % 2 == 0)
    bank_cyc += max(1, ev, len(regs) - ev)
n = len(hot)
print(f"loop 0x{lo:x}-0x{hi:x}: {n} hot instructions = {n / ppi:.2f}/pair "
      f"({len(cold)} cold dropped); reads {sum(reads.values()) / ppi:.1f}/pair")
fp = sum(v for k, v in mix.items() if k.split(".")[0] in FP64)
print(f"  FP64 {fp / ppi:.2f}/pair, other {(n - fp) / ppi:.2f}/pair")
print(f"  RF-bank issue model: {bank_cyc / ppi:.1f} cycles/warp-pair (FP64 pipe floor {2 * fp / ppi:.1f})")
for k, v in mix.most_common():
    print(f"  {k:24s} {v / ppi:5.2f}")
print("  reads by opcode:")
for k, v in reads.most_common():
    print(f"    {k:10s} {v / ppi:5.2f}")
