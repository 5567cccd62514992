"""Build A/B variants here (CPU) into ab_ship/, time them on the GPU box.

  python tools/ab_ship.py build "name=DEF1;DEF2" ...      (CPU, parallel)
  python tools/ab_ship.py time M threads[,threads] passes [names...]   (GPU)
Each pass times every variant (min of 3 launches); even passes run in reverse
order so drift and thermal state do not favour one end of the list.
"""
import json, os, subprocess, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
OUT = os.path.join(ROOT, "ab_ship")

if sys.argv[1] == "build":
    from paper_conf_ipps_bozkusf12_b200 import build
    os.makedirs(OUT, exist_ok=True)

    def one(spec):
        name, _, defs = spec.partition("=")
        items = [x for x in defs.split(";") if x]
        d = tuple(x for x in items if not x.startswith("-"))
        x = tuple(y for x in items if x.startswith("-") for y in x.split())
        build.build(out=os.path.join(OUT, "libhpl_%s.so" % name), defines=d, extra=x)
        return name, d, x
    with ThreadPoolExecutor(max_workers=int(os.environ.get("AB_J", "4"))) as ex:
        for r in ex.map(one, sys.argv[2:]):
            print("built", *r, flush=True)
else:
    M, threads, passes = sys.argv[2], sys.argv[3], int(sys.argv[4])
    names = sys.argv[5:] or sorted(f[7:-3] for f in os.listdir(OUT) if f.startswith("libhpl_") and f.endswith(".so"))
    for p in range(passes):
        for n in (names if p % 2 == 0 else names[::-1]):
            env = dict(os.environ, HPL_LIB=os.path.join(OUT, "libhpl_%s.so" % n))
            r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "quick_time.py"), *M.split(","),
                                "--threads", threads, "--reps", "3"], env=env, capture_output=True, text=True)
            for line in r.stdout.splitlines():
                d = json.loads(line)
                print(json.dumps({"variant": n, "pass": p, **{k: d[k] for k in ("thr", "M", "s", "Mops", "gc", "sx", "sy") if k in d}}), flush=True)
            if r.returncode:
                print(n, "FAILED", r.stderr[-800:], flush=True)
