import math, random
M46 = 1 << 46
H = 1 << 45
def xs(k): return 2.0 * (k * 2.0**-46) - 1.0
def t_of(k1, k2):
    a, b = xs(k1), xs(k2); return a*a + b*b
rng = random.Random(7)
targets = {"eq1": 1.0, "below1": math.nextafter(1.0, 0), "above1": math.nextafter(1.0, 2)}
found = {}
for trial in range(200000):
    i = rng.randrange(1, H) | 1       # |x1| = i / 2^45
    jj = math.isqrt((1 << 90) - i * i)
    for dj in range(-3, 4):
        j = jj + dj
        if j <= 0 or j % 2 == 0: continue
        for s1 in (1, -1):
            k1 = H + s1 * i; k2 = H + j
            t = t_of(k1, k2)
            for name, tv in targets.items():
                if t == tv and name not in found:
                    found[name] = (k1, k2)
    if len(found) == 3: break
print(found)
