"""atfspec — search-space *specifications* (inputs), shared by the oracle tests and the GPU path.

This module is the one thing the oracle (``oracle/``) and the product
(``paper_conf_hpdc_raschg18_b200/``) have in common: it builds parameter
specifications and writes them as JSON.  It holds none of the method's
arithmetic — it never evaluates a constraint, materialises a range, counts or
enumerates anything.  It only *encodes*:

* ranges as ``{"kind": "interval"|"pow2"|"set", ...}``  (§II
  "atf::interval<T>(begin, end, step_size, generator)" and "atf::set(...)");
* constraints as postfix int32 bytecode (SURVEY.md §8(b) opcode table), built
  with a tiny expression DSL mirroring the paper's constraint aliases
  ``divides``, ``is_multiple_of``, ``less_than``, ``greater_than``, ``equal``,
  ``unequal`` combined with ``&&`` / ``||`` (§II Step 1).

Spec JSON layout::

    {"name": str,
     "params": [{"name": str,
                 "range": {"kind": "interval", "begin": b, "end": e, "step": s}
                        | {"kind": "pow2", "begin": b, "end": e, "step": s}
                        | {"kind": "set", "values": [v1, ...]},
                 "constraints": [[word, ...], ...]},   # ANDed, may be empty
                ...]}
"""
from __future__ import annotations

import json
from dataclasses import dataclass, field
from typing import List, Optional, Sequence, Union

# ---- opcodes (SURVEY.md §8(b) "Bytecode (postfix, int32 words, int64 stack)") ----
OP_X, OP_PARAM, OP_CONST = 1, 2, 3
OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_MOD, OP_MIN, OP_MAX = 4, 5, 6, 7, 8, 9, 10
OP_EQ, OP_NE, OP_LT, OP_LE, OP_GT, OP_GE = 11, 12, 13, 14, 15, 16
OP_DIVIDES, OP_MULOF, OP_AND, OP_OR, OP_NOT = 17, 18, 19, 20, 21

OPNAMES = {
    OP_X: "X", OP_PARAM: "PARAM", OP_CONST: "CONST", OP_ADD: "ADD", OP_SUB: "SUB",
    OP_MUL: "MUL", OP_DIV: "DIV", OP_MOD: "MOD", OP_MIN: "MIN", OP_MAX: "MAX",
    OP_EQ: "EQ", OP_NE: "NE", OP_LT: "LT", OP_LE: "LE", OP_GT: "GT", OP_GE: "GE",
    OP_DIVIDES: "DIVIDES", OP_MULOF: "MULOF", OP_AND: "AND", OP_OR: "OR", OP_NOT: "NOT",
}
BINARY_OPS = tuple(range(OP_ADD, OP_OR + 1))


def _split64(v: int) -> List[int]:
    """int64 -> (lo, hi) as two *signed* int32 words (two's complement)."""
    if not (-(1 << 63) <= v < (1 << 63)):
        raise ValueError("constant outside int64")
    u = v & ((1 << 64) - 1)
    lo, hi = u & 0xFFFFFFFF, u >> 32
    to_s = lambda w: w - (1 << 32) if w >= (1 << 31) else w
    return [to_s(lo), to_s(hi)]


class E:
    """A postfix expression.  Python operators build bytecode; nothing is evaluated."""

    __slots__ = ("code",)

    def __init__(self, code: Sequence[int]):
        self.code = list(code)

    # arithmetic
    def _bin(self, other, op, swap=False):
        o = lift(other)
        a, b = (o, self) if swap else (self, o)
        return E(a.code + b.code + [op])

    def __add__(self, o): return self._bin(o, OP_ADD)
    def __radd__(self, o): return self._bin(o, OP_ADD, True)
    def __sub__(self, o): return self._bin(o, OP_SUB)
    def __rsub__(self, o): return self._bin(o, OP_SUB, True)
    def __mul__(self, o): return self._bin(o, OP_MUL)
    def __rmul__(self, o): return self._bin(o, OP_MUL, True)
    def __floordiv__(self, o): return self._bin(o, OP_DIV)      # C truncation (reading #8)
    def __rfloordiv__(self, o): return self._bin(o, OP_DIV, True)
    def __mod__(self, o): return self._bin(o, OP_MOD)
    def __rmod__(self, o): return self._bin(o, OP_MOD, True)
    # comparisons (explicit names: == / != stay Python identity-safe)
    def eq(self, o): return self._bin(o, OP_EQ)
    def ne(self, o): return self._bin(o, OP_NE)
    def __lt__(self, o): return self._bin(o, OP_LT)
    def __le__(self, o): return self._bin(o, OP_LE)
    def __gt__(self, o): return self._bin(o, OP_GT)
    def __ge__(self, o): return self._bin(o, OP_GE)
    # logic: strict, non-short-circuit (reading #7)
    def __and__(self, o): return self._bin(o, OP_AND)
    def __rand__(self, o): return self._bin(o, OP_AND, True)
    def __or__(self, o): return self._bin(o, OP_OR)
    def __ror__(self, o): return self._bin(o, OP_OR, True)
    def __invert__(self): return E(self.code + [OP_NOT])

    def __repr__(self):
        return "E(" + disasm(self.code) + ")"


def lift(v) -> E:
    if isinstance(v, E):
        return v
    if isinstance(v, bool):
        v = int(v)
    if isinstance(v, int):
        return E([OP_CONST] + _split64(v))
    raise TypeError(f"cannot lift {type(v)} into a constraint expression")


X = E([OP_X])


def C(v: int) -> E:
    return lift(v)


def P(j: int) -> E:
    """Value of the already-fixed parameter with id ``j`` (declaration index)."""
    return E([OP_PARAM, int(j)])


def min_(a, b) -> E: return E(lift(a).code + lift(b).code + [OP_MIN])
def max_(a, b) -> E: return E(lift(a).code + lift(b).code + [OP_MAX])
def DIVIDES(a, b) -> E: return E(lift(a).code + lift(b).code + [OP_DIVIDES])  # [a!=0 and b % a == 0]
def MULOF(a, b) -> E: return E(lift(a).code + lift(b).code + [OP_MULOF])      # [b!=0 and a % b == 0]


# ---- the paper's constraint aliases, all relative to the candidate X ----
def divides(e) -> E: return DIVIDES(X, e)          # E % x == 0   ("(N/WPT) % LS == 0")
def is_multiple_of(e) -> E: return MULOF(X, e)     # x % E == 0
def less_than(e) -> E: return X < lift(e)
def greater_than(e) -> E: return X > lift(e)
def equal(e) -> E: return X.eq(e)
def unequal(e) -> E: return X.ne(e)


def disasm(code: Sequence[int]) -> str:
    out, i = [], 0
    while i < len(code):
        op = code[i]
        if op == OP_PARAM:
            out.append(f"PARAM {code[i+1]}"); i += 2
        elif op == OP_CONST:
            lo, hi = code[i+1] & 0xFFFFFFFF, code[i+2] & 0xFFFFFFFF
            v = (hi << 32) | lo
            if v >= 1 << 63:
                v -= 1 << 64
            out.append(f"CONST {v}"); i += 3
        else:
            out.append(OPNAMES.get(op, f"?{op}")); i += 1
    return " ".join(out)


# ---- ranges ----
def interval(begin: int, end: int, step: int = 1) -> dict:
    return {"kind": "interval", "begin": int(begin), "end": int(end), "step": int(step)}


def pow2(begin: int, end: int, step: int = 1) -> dict:
    """``atf::interval<size_t>(begin, end, step, [](i){return pow(2,i);})``."""
    return {"kind": "pow2", "begin": int(begin), "end": int(end), "step": int(step)}


def gen(begin: int, end: int, expr, step: int = 1) -> dict:
    """``atf::interval<T>(begin, end, step, generator)``: values expr(i) for i = begin,
    begin+step, ..., <= end; `expr` is an expression in X (= i) and constants."""
    return {"kind": "gen", "begin": int(begin), "end": int(end), "step": int(step), "code": list(lift(expr).code)}


def set_(*values: int) -> dict:
    return {"kind": "set", "values": [int(v) for v in values]}


def enum(*names: str) -> dict:
    """A named enumeration (S§8(f) NEXT-3): a SET of the integer codes 0..n-1 in the listed
    order (reading #4), with the names kept for display; constraints compare codes
    (e.g. ``equal(enum_code(rng, "local"))``)."""
    if len(set(names)) != len(names):
        raise ValueError("duplicate enum name")  # reading #5
    return {"kind": "set", "values": list(range(len(names))), "names": [str(n) for n in names]}


def enum_code(rng: dict, name: str) -> int:
    return rng["names"].index(name)


def floats(*values: float) -> dict:
    """A float-valued parameter by position index (S§8(f) NEXT-3; P:57 ranges of "arbitrary
    fundamental type T (e.g., bool, integer, or float)"): a SET of the positions 0..n-1 in the
    listed order, the float values kept as the display names (Space.to_named maps positions back).
    Constraints see the position; for an ascending list (float_interval) order comparisons on
    positions equal order comparisons on values (``X <= float_code(rng, 0.5)``)."""
    vals = [float(v) for v in values]
    if len(set(vals)) != len(vals):
        raise ValueError("duplicate float value")  # reading #5
    return {"kind": "set", "values": list(range(len(vals))), "names": vals}


def float_interval(begin: float, end: float, step: float) -> dict:
    """``atf::interval<float>(begin, end, step)``: begin + i * step for i = 0, 1, ... while <= end
    (inclusive, reading #1; a tolerance of 1e-9 * step absorbs the float rounding of the bound)."""
    n = int((end - begin) / step + 1e-9) + 1
    return floats(*[begin + i * step for i in range(max(0, n))])


def float_code(rng: dict, value: float) -> int:
    """Position of `value` in a float parameter's range (exact match)."""
    return rng["names"].index(float(value))


@dataclass
class Param:
    name: str
    range: dict
    constraints: List[List[int]] = field(default_factory=list)


@dataclass
class Spec:
    name: str
    params: List[Param] = field(default_factory=list)

    def add(self, name: str, rng: dict, *constraints: Union[E, Sequence[int], None]) -> int:
        cs = []
        for c in constraints:
            if c is None:
                continue
            cs.append(list(c.code) if isinstance(c, E) else [int(w) for w in c])
        self.params.append(Param(name, rng, cs))
        return len(self.params) - 1

    def id(self, name: str) -> int:
        for i, p in enumerate(self.params):
            if p.name == name:
                return i
        raise KeyError(name)

    def P(self, name: str) -> E:
        return P(self.id(name))

    def to_json(self) -> dict:
        return {"name": self.name,
                "params": [{"name": p.name, "range": p.range, "constraints": p.constraints}
                           for p in self.params]}

    def dumps(self) -> str:
        return json.dumps(self.to_json(), separators=(",", ":"))

    def write(self, path) -> str:
        with open(path, "w") as f:
            f.write(self.dumps())
        return str(path)

    @staticmethod
    def from_json(d: dict) -> "Spec":
        s = Spec(d["name"])
        for p in d["params"]:
            s.params.append(Param(p["name"], dict(p["range"]), [list(c) for c in p.get("constraints", [])]))
        return s

    @staticmethod
    def load(path) -> "Spec":
        with open(path) as f:
            return Spec.from_json(json.load(f))


from .configs import *  # noqa: E402,F401,F403
from .fuzz import random_spec, random_wide_spec  # noqa: E402,F401
