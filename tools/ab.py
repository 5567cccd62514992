"""A/B build variants of libhpl.so with -D switches (development aid).

  python tools/ab.py build "name=DEF1;DEF2" name2=...     (CPU: compile into build_ab/)
  python tools/ab.py time M threads [names...]          (GPU: time each variant)
"""
import json, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
OUT = os.path.join(ROOT, "build_ab")

if sys.argv[1] == "build":
    from paper_conf_ipps_bozkusf12_b200 import build
    os.makedirs(OUT, exist_ok=True)
    for spec in sys.argv[2:]:
        name, _, defs = spec.partition("=")
        items = [x for x in defs.split(";") if x]
        d = tuple(x for x in items if not x.startswith("-"))     # -D defines
        x = tuple(y for x in items if x.startswith("-") for y in x.split())  # extra nvcc flags
        build.build(out=os.path.join(OUT, "libhpl_%s.so" % name), defines=d, extra=x)
        print("built", name, d)
else:
    M, threads = sys.argv[2], sys.argv[3]
    names = sys.argv[4:] or sorted(f[7:-3] for f in os.listdir(OUT) if f.startswith("libhpl_"))
    for n in names:
        env = dict(os.environ, HPL_LIB=os.path.join(OUT, "libhpl_%s.so" % n))
        r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "quick_time.py"), *M.split(","),
                            "--threads", threads, "--reps", "3"], env=env, capture_output=True, text=True)
        for line in r.stdout.splitlines():
            d = json.loads(line)
            print(json.dumps({"variant": n, **{k: d[k] for k in ("thr", "M", "s", "Mops", "gc", "sx", "sy") if k in d}}), flush=True)
        if r.returncode:
            print(n, "FAILED", r.stderr[-500:])
