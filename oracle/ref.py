"""Pure-Python twin of the oracle, for tiny brute-force cases -- TEST INFRASTRUCTURE ONLY.

Written independently of oracle_scan.c (no shared code) directly from the definition,
PAPER.md:29 [§1]: element i of the inclusive scan applies the operator to elements 0..i,
element i of the exclusive scan to elements 0..i-1 (empty range -> identity).  Every
element is recomputed from scratch (O(N^2)), which is deliberately the most literal
reading of the definition; use only for N <= a few hundred.
"""
from __future__ import annotations

from fractions import Fraction
from functools import reduce

MASK32 = 0xFFFFFFFF


def _wrap(v: int, dtype: str) -> int:
    v &= MASK32
    if dtype == "i32" and v >= 2 ** 31:
        v -= 2 ** 32
    return v


def identity(op: str, dtype: str):
    if op == "add":
        return Fraction(0) if dtype == "f32" else 0
    return {"i32": -(2 ** 31), "u32": 0, "f32": float("-inf")}[dtype]


def apply(op: str, dtype: str, a, b):
    if op == "add":
        if dtype == "f32":
            return Fraction(a) + Fraction(b)      # exact rational: no rounding at all
        return _wrap(a + b, dtype)
    return b if b > a else a


def scan_literal(xs, op: str, dtype: str, kind: str):
    """out[i] = x_0 (+) ... (+) x_i  (inclusive)  or  x_0 (+) ... (+) x_{i-1}  (exclusive).

    f32 add returns exact Fractions (the real-number prefix of the f32 inputs).
    """
    out = []
    for i in range(len(xs)):
        hi = i + 1 if kind == "inclusive" else i
        out.append(reduce(lambda a, b: apply(op, dtype, a, b), xs[:hi], identity(op, dtype)))
    return out
