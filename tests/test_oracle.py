"""Pins for the CPU oracle (oracle/ep_oracle.cpp) — SURVEY.md §8(c) P1-P9.

Everything here checks the oracle against something OTHER than itself:
published NPB values (tests/golden, cited), exact integer arithmetic (Python
big ints), exact/50-digit decimal arithmetic (brute force), closed forms and
invariants.  A dropped term, a wrong sign, swapped pair order, an FMA in t,
a wrong batch seed or a wrong bin truncation each fails at least one test
(DESIGN.md §3 maps mistakes to pins).
"""
import math

import numpy as np
import random
from decimal import Decimal, localcontext

import pytest

from _golden import npb_counts, npb_verify
from ep_workloads import CLASSES, NPB_A, NPB_SEED, ROBUST_SEEDS

MOD46 = 1 << 46


# ---------------------------------------------------------------- P1/P2/P3 LCG
def test_randlc_double_split_equals_integer_lcg(oracle_mod):
    """P1: NPB's double-split randlc == (a*x) mod 2^46 exactly, incl. 46-bit a."""
    rng = random.Random(12345)
    for _ in range(20000):
        x = rng.randrange(MOD46)
        a = rng.randrange(MOD46) if rng.random() < 0.5 else rng.randrange(1 << 31)
        u, xn = oracle_mod.randlc(float(x), float(a))
        want = (a * x) % MOD46
        assert xn == float(want)
        assert u == want * 2.0 ** -46  # uniform of the UPDATED state (R2)


def test_stream_start_closed_form(oracle_mod):
    """P2: x_k = seed * a^k mod 2^46 (closed form, exact ints)."""
    got = oracle_mod.states(NPB_SEED, NPB_A, 0, 64)
    want = [NPB_SEED * pow(NPB_A, k, MOD46) % MOD46 for k in range(1, 65)]
    assert got == want
    assert got[:4] == [32883653486115, 55063727434591, 39106144873291, 46899331031975]


@pytest.mark.parametrize("offset", [0, 1, 2 ** 17 - 1, 2 ** 17, 3 * 2 ** 17 + 5, 2 ** 25,
                                    2 ** 26, 2 ** 29, 2 ** 31, 2 ** 33, 2 ** 37 - 1, 2 ** 37,
                                    2 ** 43 + 12345])
def test_skip_ahead(oracle_mod, offset):
    """P3: the oracle's binary-exponentiation jump lands on seed*a^offset."""
    got = oracle_mod.states(NPB_SEED, NPB_A, offset, 3)
    want = [NPB_SEED * pow(NPB_A, offset + k, MOD46) % MOD46 for k in (1, 2, 3)]
    assert got == want


def test_an_and_period(oracle_mod):
    """P3: AN = a^(2^17) mod 2^46; the stream period for odd seed is 2^44."""
    assert oracle_mod.an(NPB_A, 16) == pow(NPB_A, 2 ** 17, MOD46) == 62362532446209
    assert pow(NPB_A, 2 ** 44, MOD46) == 1
    assert pow(NPB_A, 2 ** 43, MOD46) == 35184372088833 != 1


# ------------------------------------------------------ P5 NPB published sums
@pytest.mark.parametrize("cls", ["S", "W", "A", "B"])
def test_npb_verification_sums(oracle_mod, cls):
    """P5: NPB ep.f verify values (tests/golden/npb_ep_verify.txt), eps = 1e-8.

    The oracle actually agrees to ~1e-12 (NPB summed plainly, we compensate),
    so we also pin 1e-10 to catch any systematic error far below NPB's eps."""
    M, sx_ref, sy_ref = npb_verify()[cls]
    assert M == CLASSES[cls]
    r = oracle_mod.run(M, NPB_SEED, NPB_A, threads=8, margin=False)
    assert abs((r.sx - sx_ref) / sx_ref) <= 1e-10
    assert abs((r.sy - sy_ref) / sy_ref) <= 1e-10
    assert r.npairs == 2 ** M and r.qbig == 0


@pytest.mark.parametrize("cls", ["S", "W", "A"])
def test_npb_reference_counts(oracle_mod, cls):
    """P6: NPB reference-output counts (tests/golden/npb_ep_counts.txt), exact."""
    M, gc, q = npb_counts()[cls]
    r = oracle_mod.run(M, NPB_SEED, NPB_A, threads=8, margin=True)
    assert r.gc == gc and r.q == q
    # R7: every accepted pair is far from a bin boundary (> 8 ulp), so q[] is
    # implementation-independent for any log/sqrt within a few ulp
    assert r.min_margin_ulp > 8


def test_npb_sums_reject_plausible_mistakes(oracle_mod):
    """The class-S pin is sensitive: swapped pair order or a dropped sign move
    sx/sy far outside 1e-8, so P5 really discriminates (sanity of the pin)."""
    _, sx_ref, sy_ref = npb_verify()["S"]
    r = oracle_mod.run(24, NPB_SEED, NPB_A, threads=8, margin=False)
    assert abs((r.sy - sx_ref) / sx_ref) > 1e-3  # swapping (x1, x2) would fail
    assert abs((-r.sx - sx_ref) / sx_ref) > 1e-3


# ------------------------------------------------------------- P8 brute force
def brute_force(M, seed, a, prec=50):
    """Independent EP: exact-integer LCG, IEEE-double acceptance exactly as NPB
    evaluates it (Python floats never fuse), 50-digit decimal transform, exact
    decimal sums, bins from the exact max(|X|,|Y|)."""
    q = [0] * 10
    sx = sy = Decimal(0)
    sabs = Decimal(0)
    x = seed
    with localcontext() as ctx:
        ctx.prec = prec
        for _ in range(1 << M):
            x = a * x % MOD46
            u1 = x
            x = a * x % MOD46
            u2 = x
            x1 = 2.0 * (u1 * 2.0 ** -46) - 1.0
            x2 = 2.0 * (u2 * 2.0 ** -46) - 1.0
            t = x1 * x1 + x2 * x2
            if t <= 1.0:
                T = Decimal(t)
                if t == 1.0:
                    X = Y = Decimal(0)
                else:
                    f = (Decimal(-2) * T.ln() / T).sqrt()
                    X, Y = Decimal(x1) * f, Decimal(x2) * f
                q[int(max(abs(X), abs(Y)))] += 1
                sx += X
                sy += Y
                sabs += abs(X) + abs(Y)
    return q, float(sx), float(sy), float(sabs)


@pytest.mark.parametrize("M", list(range(0, 13)))
def test_brute_force_tiny_M(oracle_mod, M):
    q, sx, sy, sabs = brute_force(M, NPB_SEED, NPB_A)
    r = oracle_mod.run(M, NPB_SEED, NPB_A, threads=1)
    assert r.q == q and r.gc == sum(q)
    tol = 4e-16 * sabs + 1e-300
    assert abs(r.sx - sx) <= tol and abs(r.sy - sy) <= tol


@pytest.mark.parametrize("seed", ROBUST_SEEDS)
def test_brute_force_robust_seeds(oracle_mod, seed):
    q, sx, sy, sabs = brute_force(11, seed, NPB_A)
    r = oracle_mod.run(11, seed, NPB_A, threads=1)
    assert r.q == q
    tol = 4e-16 * sabs + 1e-300
    assert abs(r.sx - sx) <= tol and abs(r.sy - sy) <= tol


def test_seed_zero_rejects_everything(oracle_mod):
    """Degenerate case (R9): seed 0 -> every uniform 0 -> x1 = x2 = -1 -> t = 2."""
    r = oracle_mod.run(10, 0, NPB_A)
    assert r.gc == 0 and r.sx == 0.0 and r.sy == 0.0


# ------------------------------------------------ P8/P9 structure invariants
@pytest.mark.parametrize("mk", [2, 4, 8, 13, 18])
def test_batch_size_independence(oracle_mod, mk):
    """R4: MK only changes summation order, never counts."""
    base = oracle_mod.run(18, NPB_SEED, NPB_A, mk=16, threads=4)
    r = oracle_mod.run(18, NPB_SEED, NPB_A, mk=mk, threads=4)
    assert r.q == base.q
    assert abs(r.sx - base.sx) <= 1e-13 * max(abs(base.sx), 1.0)
    assert abs(r.sy - base.sy) <= 1e-13 * max(abs(base.sy), 1.0)


@pytest.mark.parametrize("G", [2, 4, 8, 3])
def test_shards_add_up(oracle_mod, G):
    """P9: pair-range shards sum to the whole run (counts exact)."""
    M = 20
    full = oracle_mod.run(M, NPB_SEED, NPB_A, threads=4)
    n = 1 << M
    bounds = [n * r // G for r in range(G + 1)]
    q = [0] * 10
    sx = sy = 0.0
    for r in range(G):
        p = oracle_mod.run_pairs(NPB_SEED, NPB_A, bounds[r], bounds[r + 1] - bounds[r])
        q = [u + v for u, v in zip(q, p.q)]
        sx += p.sx
        sy += p.sy
    assert q == full.q
    assert abs(sx - full.sx) <= 1e-12 * max(abs(full.sx), 1.0)
    assert abs(sy - full.sy) <= 1e-12 * max(abs(full.sy), 1.0)


def test_threads_do_not_change_result(oracle_mod):
    a = oracle_mod.run(20, NPB_SEED, NPB_A, mk=12, threads=1)
    b = oracle_mod.run(20, NPB_SEED, NPB_A, mk=12, threads=7)
    assert (a.q, a.sx, a.sy) == (b.q, b.sx, b.sy)  # batch-order combine: bitwise equal


# ------------------------------------------------------------ P7 statistics
def test_statistics_class_S(oracle_mod):
    """P7 (sanity): acceptance pi/4, annulus probabilities of max(|X|,|Y|)."""
    M = 24
    r = oracle_mod.run(M, NPB_SEED, NPB_A, threads=8, margin=False)
    n = 2 ** M
    p = math.pi / 4
    assert abs(r.gc - n * p) < 5 * math.sqrt(n * p * (1 - p))
    probs = [math.erf((l + 1) / math.sqrt(2)) ** 2 - math.erf(l / math.sqrt(2)) ** 2
             for l in range(6)]
    chi2 = sum((r.q[l] - r.gc * probs[l]) ** 2 / (r.gc * probs[l]) for l in range(6))
    assert chi2 < 25  # 5 dof; P(chi2 > 25) ~ 1e-4
    assert abs(r.sx) < 5 * math.sqrt(r.gc) and abs(r.sy) < 5 * math.sqrt(r.gc)


def test_stored_large_class_goldens_match_npb():
    """tests/golden/oracle_ep.json (written by oracle/ only) against NPB's
    published verification sums for B, C, D and the recalled class-B counts."""
    from _golden import oracle_golden
    g = oracle_golden()
    ver = npb_verify()
    for cls in ("B", "C", "D"):
        assert cls in g, cls
        M, sxr, syr = ver[cls]
        assert g[cls]["M"] == M and g[cls]["npairs"] == 2 ** M and g[cls]["qbig"] == 0
        assert abs((g[cls]["sx"] - sxr) / sxr) <= 1e-10 and abs((g[cls]["sy"] - syr) / syr) <= 1e-10
        assert sum(g[cls]["q"]) == g[cls]["gc"]
        assert g[cls]["min_margin_ulp"] > 8
    M, gc, q = npb_counts()["B"]
    assert g["B"]["gc"] == gc and g["B"]["q"] == q


def _rn(dec):
    return float(dec)  # Decimal -> nearest double (correct rounding)


def test_t_is_unfused(oracle_mod):
    """R5 pin: t = RN(RN(x1²) + RN(x2²)), not the fused RN(x1² + RN(x2²)).
    Searches LCG-shaped inputs (x = 2u-1, u = k 2^-46) where the two differ and
    checks the oracle returns the unfused value there (and everywhere)."""
    rng = random.Random(55)
    differ = 0
    with localcontext() as ctx:
        ctx.prec = 60
        for _ in range(20000):
            x1 = 2.0 * (rng.randrange(MOD46) * 2.0 ** -46) - 1.0
            x2 = 2.0 * (rng.randrange(MOD46) * 2.0 ** -46) - 1.0
            unfused = x1 * x1 + x2 * x2                     # Python floats never fuse
            fused = _rn(Decimal(x1) * Decimal(x1) + Decimal(x2 * x2))
            assert oracle_mod.pair_t(x1, x2) == unfused
            differ += fused != unfused
    assert differ > 1000  # the check is discriminating


def test_worked_example_first_pairs():
    """P4: the first six pairs (tests/golden/ep_first_pairs.txt) re-derived from
    exact-integer LCG states and 50-digit decimal arithmetic."""
    import os
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "ep_first_pairs.txt")
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    x = NPB_SEED
    with localcontext() as ctx:
        ctx.prec = 50
        for r in rows:
            x = NPB_A * x % MOD46
            u1 = x
            x = NPB_A * x % MOD46
            u2 = x
            x1 = 2.0 * (u1 * 2.0 ** -46) - 1.0
            x2 = 2.0 * (u2 * 2.0 ** -46) - 1.0
            t = x1 * x1 + x2 * x2
            assert t <= 1.0
            f = (Decimal(-2) * Decimal(t).ln() / Decimal(t)).sqrt()
            X, Y = float(Decimal(x1) * f), float(Decimal(x2) * f)
            assert abs(X - float(r[1])) <= 4 * math.ulp(X) and abs(Y - float(r[2])) <= 4 * math.ulp(Y)
            assert int(max(abs(X), abs(Y))) == int(r[3])


# ------------------------------------ C10 / C7 additions: compensated sums, margin
def test_csum_adversarial_sequences(oracle_mod):
    """Reading R10 (C10): the oracle's Neumaier sum is the exactly rounded sum
    (math.fsum) on cancellation patterns where plain, and Kahan, summation fail."""
    cases = [
        [1e16, 1.0, -1e16],                       # plain: 0
        [1.0, 1e100, 1.0, -1e100],                # Kahan: 0, Neumaier: 2
        [2.0 ** 53, 1.0, 1.0, 1.0, -(2.0 ** 53)],  # plain: 2 (ties to even), exact 3
        [0.1] * 10 + [-1.0],                      # classic 1-ulp residue
    ]
    for seq in cases:
        assert oracle_mod.csum(seq) == math.fsum(seq), seq
    assert oracle_mod.csum([]) == 0.0


def test_csum_long_random_sequence(oracle_mod):
    """2^20 N(0,1)-like terms plus large cancelling pairs: within 1 ulp of
    fsum, while plain sequential summation is off by far more (the pin
    discriminates a `s += v` mutation)."""
    rng = random.Random(2024)
    seq = []
    for i in range(1 << 20):
        seq.append(rng.gauss(0.0, 1.0))
        if i % 4096 == 0:
            big = rng.uniform(1e6, 1e9)
            seq += [big, -big * (1 + 2.0 ** -40)]
    exact = math.fsum(seq)
    plain = 0.0
    for v in seq:
        plain += v
    assert abs(oracle_mod.csum(seq) - exact) <= math.ulp(exact)
    assert abs(plain - exact) > 10 * math.ulp(exact)


def test_oracle_deviates_vs_decimal(oracle_mod):
    """The exported per-pair deviates (the same gauss_pair the runs use) are
    within 2 ulp of 50-digit decimal X, Y and their bins match, pair by pair."""
    M = 11
    X, Y, l = oracle_mod.pairs(NPB_SEED, NPB_A, 0, 1 << M)
    x = NPB_SEED
    with localcontext() as ctx:
        ctx.prec = 50
        for i in range(1 << M):
            x = NPB_A * x % MOD46
            x1 = 2.0 * (x * 2.0 ** -46) - 1.0
            x = NPB_A * x % MOD46
            x2 = 2.0 * (x * 2.0 ** -46) - 1.0
            t = x1 * x1 + x2 * x2
            if t > 1.0:
                assert l[i] == -1
                continue
            f = (Decimal(-2) * Decimal(t).ln() / Decimal(t)).sqrt()
            Xd, Yd = float(Decimal(x1) * f), float(Decimal(x2) * f)
            assert abs(X[i] - Xd) <= 2 * math.ulp(Xd) and abs(Y[i] - Yd) <= 2 * math.ulp(Yd)
            assert l[i] == int(max(abs(X[i]), abs(Y[i])))


@pytest.mark.parametrize("M,mk", [(20, 20), (20, 12)])
def test_run_sums_are_compensated(oracle_mod, M, mk):
    """R10 at run level: the oracle's sx, sy equal the exactly rounded sum of its
    own deviates to <= 2 ulp (one batch, and 256 batches combined in order),
    whereas plain sequential summation of the same deviates is off by > 10 ulp."""
    X, Y, l = oracle_mod.pairs(NPB_SEED, NPB_A, 0, 1 << M)
    r = oracle_mod.run(M, NPB_SEED, NPB_A, mk=mk, threads=4, margin=False)
    assert r.gc == int((l >= 0).sum())
    for got, v in ((r.sx, X), (r.sy, Y)):
        exact = math.fsum(v.tolist())
        assert abs(got - exact) <= 2 * math.ulp(exact), (got, exact)
    plain = 0.0
    for v in X.tolist():
        plain += v
    exact = math.fsum(X.tolist())
    assert abs(plain - exact) > 10 * math.ulp(exact)


def _margin_py(X, Y, l):
    """Reading R7 recomputed here: min over accepted pairs of |m - n| / ulp(m),
    n = nearest integer of m = max(|X|,|Y|), counted when 1 <= n <= 10."""
    best = 1e300
    for xv, yv, lv in zip(X.tolist(), Y.tolist(), l.tolist()):
        if lv < 0:
            continue
        m = max(abs(xv), abs(yv))
        n = round(m)
        if 1 <= n <= 10:
            best = min(best, abs(m - n) / math.ulp(m))
    return best


@pytest.mark.parametrize("seed,begin,n", [(NPB_SEED, 0, 1 << 15), (NPB_SEED, 2 ** 30 + 77, 1 << 15),
                                          (1, 0, 1 << 14), ((1 << 46) - 1, 4321, 1 << 14)])
def test_bin_margin_matches_recomputation(oracle_mod, seed, begin, n):
    """C7: the oracle's min_margin_ulp equals the margin recomputed in Python
    from its deviates (catches a tracker that is never updated or mis-measured)."""
    X, Y, l = oracle_mod.pairs(seed, NPB_A, begin, n)
    r = oracle_mod.run_pairs(seed, NPB_A, begin, n, margin=True)
    assert r.min_margin_ulp == _margin_py(X, Y, l)
    assert r.min_margin_ulp < 1e300


def test_bin_margin_locates_the_closest_pair(oracle_mod):
    """C7 on a constructed small-margin window: find the pair of 2^18 closest to a
    bin boundary, then a 64-pair window around it reports exactly that margin
    and a window without it reports a larger one."""
    n = 1 << 18
    X, Y, l = oracle_mod.pairs(NPB_SEED, NPB_A, 0, n)
    m = np.maximum(np.abs(X), np.abs(Y))
    near = np.rint(m)
    ok = (l >= 0) & (near >= 1) & (near <= 10)
    d = np.where(ok, np.abs(m - near) / np.spacing(m), np.inf)
    i = int(np.argmin(d))
    assert d[i] < 2.0 ** 40   # a genuinely small margin at this size (~2^-12 relative)
    lo = max(0, i - 32)
    w = oracle_mod.run_pairs(NPB_SEED, NPB_A, lo, 64, margin=True)
    assert w.min_margin_ulp == float(d[i])
    far = oracle_mod.run_pairs(NPB_SEED, NPB_A, i + 1, 64, margin=True)
    assert far.min_margin_ulp > float(d[i])
    assert oracle_mod.bin_margin(float(m[i])) == float(d[i])
