#!/usr/bin/env python
"""Writes tests/golden/kmeans_r18_fma.json: the pin of reading R18 for the
K-means assignment (NEXT-1; Sec. 2.4).

R18: E(i, c) = sum over j = 0..d-1, IN INDEX ORDER, of (x_ij - c_cj)^2 in f32, with
t = x_ij - c_cj rounded to f32 and acc = fma(t, t, acc) (ONE rounding per term);
membership = argmin_c E, the first c on ties (strict <).

This script computes every E from first principles with exact rational arithmetic
(fractions.Fraction) and its own round-to-nearest-even to binary32 -- it imports
neither oracle/ nor the CUDA library.  It keeps only points where R18's decision
DIFFERS from a plausible misreading, so that an oracle (or kernel) that makes that
mistake fails the fixture:

  "mul_add"   acc = fl(acc + fl(t*t))                  (two roundings: no FMA)
  "reversed"  the fma loop over j = d-1 .. 0           (wrong summation order)
  "exact"     the real-number argmin of sum (x - c)^2  (no f32 rounding at all)
  "f64_acc"   t in f32, sum of t*t accumulated in f64  (wrong accumulator width)
  "le_ties"   the LAST minimal centre wins (<= instead of <) -- points whose R18
              distances to two centres are bit-identical

Points lie near the bisector of two centres (x = midpoint + a random vector
orthogonal to c1 - c0, rounded to f32), where the distances agree up to rounding.
Run: python tools/gen_golden_r18.py   (deterministic, seed below; ~1 min)
"""
from __future__ import annotations

import json
import os
from fractions import Fraction

import numpy as np

D = 34          # the kdd_cup width (BASELINE configs[2])
SEED = 18
WANT = {"mul_add": 12, "reversed": 12, "exact": 12, "f64_acc": 12, "le_ties": 8}


def rnd32(q: Fraction) -> Fraction:
    """Round an exact rational to the nearest binary32 value, ties to even (no overflow here)."""
    if q == 0:
        return Fraction(0)
    s = -1 if q < 0 else 1
    a = -q if q < 0 else q
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1
    elif Fraction(2) ** (e + 1) <= a:
        e += 1
    e = max(e, -126)                      # subnormal quantum below 2^-126
    quantum = Fraction(2) ** (e - 23)
    m = a / quantum
    n = m.numerator // m.denominator
    r = m - n
    if r > Fraction(1, 2) or (r == Fraction(1, 2) and n % 2 == 1):
        n += 1
    return s * n * quantum


def dists(x, c):
    """All the readings' distances of one point to one centre (x, c: lists of Fractions of f32s)."""
    t = [rnd32(xj - cj) for xj, cj in zip(x, c)]
    fma = Fraction(0)
    for tj in t:
        fma = rnd32(tj * tj + fma)
    mul_add = Fraction(0)
    for tj in t:
        mul_add = rnd32(mul_add + rnd32(tj * tj))
    rev = Fraction(0)
    for tj in reversed(t):
        rev = rnd32(tj * tj + rev)
    exact = sum(((xj - cj) ** 2 for xj, cj in zip(x, c)), Fraction(0))
    f64 = 0.0
    for tj in t:
        f64 = f64 + float(tj) * float(tj)
    return {"r18": fma, "mul_add": mul_add, "reversed": rev, "exact": exact, "f64_acc": Fraction(f64)}


def argmin(vals, strict=True):
    b = 0
    for i, v in enumerate(vals):
        if (v < vals[b]) if strict else (v <= vals[b]):
            b = i
    return b


def self_check(rng):
    """rnd32 agrees with numpy's IEEE f32 rounding of doubles (incl. subnormals, halfway cases)."""
    vals = np.concatenate([rng.standard_normal(2000) * 10.0 ** rng.integers(-40, 30, 2000),
                           (np.arange(1, 200) + 0.5) * 2.0 ** -149, (2 ** 24 + np.arange(50) + 0.5)])
    for v in vals:
        assert float(rnd32(Fraction(float(v)))) == float(np.float32(v)), v


def main():
    rng = np.random.default_rng(SEED)
    self_check(np.random.default_rng(SEED + 1))
    c0 = rng.random(D).astype(np.float32)
    c1 = (c0 + (rng.random(D) * 0.2 - 0.1)).astype(np.float32)
    far = np.full(D, 7.0, np.float32)           # a third centre nobody picks
    cen = np.stack([c0, c1, far])
    C = [[Fraction(float(v)) for v in row] for row in cen]
    mid = (c0.astype(np.float64) + c1.astype(np.float64)) / 2
    n_ = (c1.astype(np.float64) - c0.astype(np.float64))
    n_ /= np.linalg.norm(n_)
    got = {k: [] for k in WANT}
    tries = 0
    while any(len(got[k]) < WANT[k] for k in WANT):
        tries += 1
        v = rng.standard_normal(D)
        v -= v.dot(n_) * n_
        x = (mid + v * rng.uniform(0.05, 0.6) + n_ * rng.normal(0, 2e-7)).astype(np.float32)
        X = [Fraction(float(a)) for a in x]
        ds = [dists(X, c) for c in C]
        r18 = [d["r18"] for d in ds]
        m = argmin(r18)
        for k in ("mul_add", "reversed", "exact", "f64_acc"):
            if len(got[k]) < WANT[k] and argmin([d[k] for d in ds]) != m:
                got[k].append((x, m, r18))
                break
        else:
            if len(got["le_ties"]) < WANT["le_ties"] and r18[0] == r18[1]:
                got["le_ties"].append((x, m, r18))
    points, member, why, e_hex = [], [], [], []
    for k in WANT:
        for x, m, r18 in got[k]:
            points.append([float(a).hex() for a in x])
            member.append(m)
            why.append(k)
            e_hex.append([float(e).hex() for e in r18])
    out = {
        "cite": "PAPER.md Sec. 2.4 (K-means, L445-531; L1628-1649); reading R18 (DESIGN.md): "
                "E = sum_j (x_j - c_j)^2 in f32, j in index order, t rounded, acc = fma(t, t, acc); "
                "first centre on ties.  Expected membership computed with exact rationals "
                "(fractions.Fraction) by tools/gen_golden_r18.py, not by oracle/ or the kernels.",
        "d": D, "k": 3, "seed": SEED, "tries": tries,
        "centres": [[float(a).hex() for a in row] for row in cen],
        "points": points, "membership": member, "discriminates": why, "E_r18": e_hex,
    }
    path = os.path.join(os.path.dirname(__file__), "..", "tests", "golden", "kmeans_r18_fma.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=0)
    print(f"{len(points)} points after {tries} tries -> {os.path.normpath(path)}")


if __name__ == "__main__":
    main()
