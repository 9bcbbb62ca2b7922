"""Seeded random specifications for fuzz parity tests (tiny ranges, every opcode,
zero divisors, negative values, empty ranges, non-contiguous groups).

Pure input generation: draws ranges and random postfix programs; evaluates nothing.
"""
from __future__ import annotations

import random

import numpy as np

from . import (Spec, E, X, C, P, interval, pow2, set_, OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_MOD,
               OP_MIN, OP_MAX, OP_EQ, OP_NE, OP_LT, OP_LE, OP_GT, OP_GE, OP_DIVIDES, OP_MULOF,
               OP_AND, OP_OR, OP_NOT)

_ARITH = [OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_MOD, OP_MIN, OP_MAX]
_REL = [OP_EQ, OP_NE, OP_LT, OP_LE, OP_GT, OP_GE, OP_DIVIDES, OP_MULOF]
_LOGIC = [OP_AND, OP_OR]


def _rand_range(rng: random.Random) -> dict:
    k = rng.random()
    if k < 0.55:
        b = rng.randint(-4, 6)
        e = b + rng.randint(-1 if rng.random() < 0.05 else 0, 12)
        return interval(b, e, rng.choice([1, 1, 1, 2, 3]))
    if k < 0.7:
        b = rng.randint(0, 3)
        return pow2(b, b + rng.randint(0, 4), rng.choice([1, 1, 2]))
    n = rng.randint(1, 6)
    vals = rng.sample(range(-5, 21), n)
    return set_(*vals)


def _rand_expr(rng: random.Random, depth: int, refs, want_x: bool) -> E:
    if depth <= 0 or rng.random() < 0.25:
        c = rng.random()
        if want_x or c < 0.4:
            return X
        if refs and c < 0.8:
            return P(rng.choice(refs))
        return C(rng.randint(-3, 10))
    op = rng.random()
    if op < 0.45:
        a = _rand_expr(rng, depth - 1, refs, want_x)
        b = _rand_expr(rng, depth - 1, refs, False)
        if rng.random() < 0.5:
            a, b = b, a
        return E(a.code + b.code + [rng.choice(_REL)])
    if op < 0.75:
        a = _rand_expr(rng, depth - 1, refs, want_x)
        b = _rand_expr(rng, depth - 1, refs, False)
        if rng.random() < 0.5:
            a, b = b, a
        return E(a.code + b.code + [rng.choice(_ARITH)])
    if op < 0.95:
        a = _rand_expr(rng, depth - 1, refs, want_x)
        b = _rand_expr(rng, depth - 1, refs, False)
        return E(a.code + b.code + [rng.choice(_LOGIC)])
    return E(_rand_expr(rng, depth - 1, refs, want_x).code + [OP_NOT])


def random_spec(seed: int, n_params: int | None = None) -> Spec:
    rng = random.Random(seed)
    n = n_params if n_params is not None else rng.randint(2, 6)
    s = Spec(f"fuzz_{seed}")
    for i in range(n):
        cons = []
        if i > 0 and rng.random() < 0.75:
            refs = rng.sample(range(i), rng.randint(1, min(i, 2)))
            for _ in range(rng.choice([1, 1, 2])):
                cons.append(_rand_expr(rng, rng.randint(1, 3), refs, True))
        elif rng.random() < 0.2:
            cons.append(_rand_expr(rng, 2, [], True))
        s.add(f"p{i}", _rand_range(rng), *cons)
    return s


def _rand_wide_range(rng: random.Random) -> dict:
    """65..6000 values: the wide expansion kernel's territory (r > 64), sometimes with 0 and
    negatives, steps, or r > 4096 (several candidate chunks)."""
    k = rng.random()
    n = rng.randint(65, 6000)
    if k < 0.6:
        b = rng.randint(1, 3) if rng.random() < 0.7 else rng.randint(-40, 0)
        step = rng.choice([1, 1, 1, 2, 3])
        return interval(b, b + (n - 1) * step, step)
    vals = rng.sample(range(-50, 9000), n)
    return set_(*vals)


def _rand_div_atom(rng: random.Random, refs) -> E:
    """A divisibility conjunct of the shapes the planner compiles to hot atoms (or not)."""
    j = rng.choice(refs)
    c = rng.random()
    if c < 0.35:
        return E(X.code + P(j).code + [OP_DIVIDES])                      # x | p_j
    if c < 0.55:
        return E(X.code + P(j).code + [OP_MULOF])                        # p_j | x
    if c < 0.7:
        return E(X.code + (P(j) * rng.randint(1, 12)).code + [OP_DIVIDES])  # x | c p_j
    if c < 0.8:
        return E((X * rng.randint(1, 4)).code + P(j).code + [OP_DIVIDES])   # (a x) | p_j
    if c < 0.9:
        return E(P(j).code + (C(rng.randint(1, 50)) // X).code + [OP_MULOF])  # (c / x) | p_j
    return E(X.code + (P(j) + rng.randint(-2, 5)).code + [OP_DIVIDES])   # x | (p_j + c)


def random_wide_spec(seed: int) -> Spec:
    """2-3 parameters whose later ranges have 65..6000 values, constrained by divisibility
    atoms (kept selective so the oracle finishes in seconds), optionally ANDed / ORed with a
    random expression.  Pure input generation."""
    rng = random.Random(1_000_003 + seed)
    n = rng.randint(2, 3)
    s = Spec(f"fuzzw_{seed}")
    s.add("p0", interval(rng.randint(-3, 2), rng.randint(3, 200)))
    for i in range(1, n):
        refs = list(range(i))
        cons = _rand_div_atom(rng, refs)
        k = rng.random()
        if k < 0.3:
            cons = cons & _rand_expr(rng, 2, refs, True)
        elif k < 0.4:
            cons = cons | (X.eq(rng.randint(-5, 100)))
        extra = [_rand_div_atom(rng, refs)] if rng.random() < 0.3 else []
        s.add(f"p{i}", _rand_wide_range(rng), cons, *extra)
    return s


def splitmix64_indices(n: int, modulus: int, seed: int, start: int = 0) -> np.ndarray:
    """idx_i = splitmix64(seed + i) mod modulus, i in [start, start+n) (C4 input recipe)."""
    if modulus <= 0:
        raise ValueError("modulus must be positive")
    with np.errstate(over="ignore"):
        z = (np.arange(start, start + n, dtype=np.uint64) + np.uint64(seed)) + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    if modulus >= 1 << 64:
        return z
    return z % np.uint64(modulus)
