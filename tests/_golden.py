"""Readers for tests/golden fixtures (each fixture file states its citation)."""
import json
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _rows(name):
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                yield line.split()


def npb_verify():
    """class -> (M, sx_ref, sy_ref) from NPB ep.f verify."""
    return {r[0]: (int(r[1]), float(r[2]), float(r[3])) for r in _rows("npb_ep_verify.txt")}


def npb_counts():
    """class -> (M, gc, [q0..q9]) from NPB reference outputs."""
    out = {}
    for r in _rows("npb_ep_counts.txt"):
        q = [int(v) for v in r[3:10]] + [0, 0, 0]
        out[r[0]] = (int(r[1]), int(r[2]), q)
    return out


def oracle_golden():
    """class -> dict written by tests/golden/make_oracle_golden.py (oracle/ only)."""
    p = os.path.join(GOLDEN, "oracle_ep.json")
    if not os.path.exists(p):
        return {}
    d = json.load(open(p))
    for v in d.values():
        v["sx"] = float.fromhex(v["sx"])
        v["sy"] = float.fromhex(v["sy"])
    return d


def sums_close(got, want, gc, rel=1e-12):
    """DESIGN.md tolerance T1: |got - want| <= rel * max(|want|, sqrt(gc))."""
    return abs(got - want) <= rel * max(abs(want), gc ** 0.5, 1.0)
