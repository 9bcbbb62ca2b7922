"""Closed forms for search-space sizes — part of the ORACLE (test infrastructure only).

These are the mathematical facts the C++ oracle (atf_oracle.cpp) is pinned to
(SURVEY.md §8(c) "What pins each part").  Each is computed two ways where cheap,
so that a slip in one shows up against the other.

* saxpy: WPT | N and LS | N/WPT.  The pairs (WPT, LS) with
  LS | N/WPT are the pairs (a, b) with b | a | N after a = N/WPT, so
  #pairs = sum_{d | N} tau(d) = prod_i (a_i + 1)(a_i + 2) / 2 for N = prod p_i^a_i.
* interval with divisibility: #{x in [1,R] : x | E} = #{d | E : d <= R};
  #{x in [1,R] : E | x} = floor(R / E).
* divisor chains (C5): #{(x_1..x_k) in [1,R]^k : x_{i+1} | x_i} = D_k(R) =
  sum_{n <= R} d_k(n) (Piltz divisor function), the same for multiple-chains,
  and D_k(R/2) for the even interval(2, R, 2) chain.
"""
from __future__ import annotations

from typing import Dict, List

import numpy as np


def factorize(n: int) -> Dict[int, int]:
    f, p = {}, 2
    while p * p <= n:
        while n % p == 0:
            f[p] = f.get(p, 0) + 1
            n //= p
        p += 1
    if n > 1:
        f[n] = f.get(n, 0) + 1
    return f


def divisors(n: int) -> List[int]:
    return [d for d in range(1, n + 1) if n % d == 0]


def tau(n: int) -> int:
    out = 1
    for a in factorize(n).values():
        out *= a + 1
    return out


def saxpy_size_by_divisor_sum(n: int) -> int:
    return sum(len(divisors(d)) for d in divisors(n))


def saxpy_size_by_exponents(n: int) -> int:
    out = 1
    for a in factorize(n).values():
        out *= (a + 1) * (a + 2) // 2
    return out


def count_divisors_upto(e: int, r: int) -> int:
    """#{x in [1, r] : x | e}  (e != 0)."""
    e = abs(e)
    return sum(1 for d in divisors(e) if d <= r)


def count_multiples_upto(e: int, r: int) -> int:
    """#{x in [1, r] : e | x}  (e > 0)."""
    return r // e


def piltz_table(R: int, kmax: int) -> np.ndarray:
    """D[k][n] = d_k(n) for n <= R (Dirichlet powers of 1), by the recurrence
    d_k = d_{k-1} * 1, i.e. d_k(n) = sum_{m | n} d_{k-1}(m)."""
    d = np.zeros((kmax + 1, R + 1), dtype=np.int64)
    d[1, 1:] = 1
    for k in range(2, kmax + 1):
        for m in range(1, R + 1):
            d[k, m::m] += d[k - 1, m]
    return d


def piltz_D(R: int, kmax: int) -> List[int]:
    """[D_1(R), ..., D_kmax(R)], D_k(R) = sum_{n<=R} d_k(n)."""
    d = piltz_table(R, kmax)
    return [int(d[k, 1:].sum()) for k in range(1, kmax + 1)]


def dirichlet_hyperbola_D2(R: int) -> int:
    """D_2(R) = sum_{d<=R} floor(R/d) — an independent route to the k=2 case."""
    return sum(R // d for d in range(1, R + 1))


def c5_level_sizes(R: int, length: int) -> List[List[int]]:
    """Per-level f_k of the three C5 chains: x (divides), y (multiple-of), z (even, divides)."""
    a = piltz_D(R, length)
    return [a, a, piltz_D(R // 2, length)]


def c1_size() -> int:
    """C1 (configs[0]): TS_M, TS_N powers of two 2^i, 2^j with i, j in [0, 6] and 2^(i+j) <= 1024."""
    return sum(1 for i in range(7) for j in range(7) if i + j <= 10)
