"""CPU-side screening of EP kernel variants with the RF-bank issue model.

  python tools/model_grid.py "name=DEF1;DEF2" ...

Compiles csrc/ep_kernel.cu to a cubin per variant (parallel) and prints the
sass_hot.py model (cycles per warp-pair of the hot loop); the
model tracked the measured class-D time within ~2 % over the session-4 A/B.
"""
import os, re, subprocess, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_ipps_bozkusf12_b200", "csrc")
TMP = os.environ.get("MG_TMP", "/tmp/mg")
os.makedirs(TMP, exist_ok=True)


def one(spec):
    name, _, defs = spec.partition("=")
    d = [x for x in defs.split(";") if x]
    cub = os.path.join(TMP, name + ".cubin")
    r = subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17", "-cubin",
                        "-I", os.path.join(ROOT, "include"), *["-D" + x for x in d if not x.startswith("-")],
                        *[x for x in d if x.startswith("-")], "-o", cub, os.path.join(CSRC, "ep_kernel.cu")],
                       capture_output=True, text=True)
    if r.returncode:
        return name, "BUILD FAILED " + r.stderr[-400:]
    pat = os.environ.get("MG_PAT", "ILi0ELb1ELi384ELi1ELi4E")
    ppi = os.environ.get("MG_PPI", "16")
    o = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "sass_hot.py"), cub, pat, ppi],
                       capture_output=True, text=True).stdout.splitlines()
    return name, " | ".join(x.strip() for x in o[:3])


with ThreadPoolExecutor(max_workers=int(os.environ.get("MG_J", "6"))) as ex:
    for name, res in ex.map(one, sys.argv[1:]):
        print("%-14s %s" % (name, res), flush=True)
