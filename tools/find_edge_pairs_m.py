import math, random
from decimal import Decimal, localcontext
H = 1 << 45
def xs(k): return 2.0 * (k * 2.0**-46) - 1.0
def t_of(k1, k2):
    a, b = xs(k1), xs(k2); return a*a + b*b
rng = random.Random(11)
# (b) t near 2^-16
T16 = 2.0**-16
found = {}
targets = {"t16_below": math.nextafter(T16, 0), "t16_eq": T16, "t16_above": math.nextafter(T16, 1)}
for trial in range(0):
    i = rng.randrange(1, int(H * 2**-8.5)) | 1
    r2 = (T16 * 2.0**90)
    if i * i >= r2: continue
    jj = math.isqrt(int(r2) - i * i)
    for dj in range(-3, 4):
        j = jj + dj
        if j <= 0 or j % 2 == 0: continue
        k1 = H - i; k2 = H + j
        t = t_of(k1, k2)
        for name, tv in targets.items():
            if t == tv and name not in found: found[name] = (k1, k2)
    if len(found) == 3: break
print(found)
# (c) m near integers: exact m from 50-digit decimal
def m_exact(k1, k2):
    a, b = xs(k1), xs(k2); t = a*a + b*b
    with localcontext() as c:
        c.prec = 60
        f = (Decimal(-2) * Decimal(t).ln() / Decimal(t)).sqrt()
        return max(abs(Decimal(a)), abs(Decimal(b))) * f
res = {}
for K in (4,):
    want = {}
    for trial in range(200000):
        # choose |x1| >= |x2| as the max; solve |x1| * t2(t) = K for x2 by bisection on j
        i = rng.randrange(int(H * 0.0005), int(H * 0.018)) | 1
        x1 = i / H
        lo, hi = 0, i
        # m decreasing in t? t2 = sqrt(-2 ln t / t) decreases with t; t increases with j
        def m_of(j): 
            x2 = j / H; t = x1*x1 + x2*x2
            if t >= 1: return 0.0
            return x1 * math.sqrt(-2*math.log(t)/t)
        if m_of(1) < K or m_of(i) > K: continue
        while hi - lo > 1:
            mid = (lo + hi) // 2
            if m_of(mid) >= K: lo = mid
            else: hi = mid
        for j in (lo - 2, lo, lo + 2, lo + 1, hi, hi + 2):
            j |= 1
            k1 = H + i; k2 = H + j
            if t_of(k1, k2) > 1.0: continue
            me = m_exact(k1, k2)
            d = float((me - K) / Decimal(math.ulp(K)))
            for tag, (a, b) in {"m1": (-1.5, -0.0), "p1": (0.0, 1.5), "m12": (-16, -8), "p12": (8, 16)}.items():
                if a <= d <= b and tag not in want: want[tag] = (k1, k2, d)
        if len(want) == 4: break
    res[K] = want
    print(K, want)
