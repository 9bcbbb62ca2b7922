"""Subprocess wrapper around the C++ oracle binary (test infrastructure only)."""
from __future__ import annotations

import json
import os
import subprocess
import tempfile
from typing import Optional

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
BIN = os.path.join(HERE, "atf_oracle")


def build(force: bool = False) -> str:
    src = os.path.join(HERE, "atf_oracle.cpp")
    if force or not os.path.exists(BIN) or os.path.getmtime(BIN) < os.path.getmtime(src):
        subprocess.check_call(["make", "-s", "-C", HERE, "atf_oracle"])
    return BIN


def _spec_path(spec, tmpdir: str) -> str:
    if isinstance(spec, str):
        return spec
    p = os.path.join(tmpdir, "spec.json")
    spec.write(p)
    return p


def _run(args, timeout: Optional[float] = None) -> dict:
    build()
    out = subprocess.run([BIN] + [str(a) for a in args], capture_output=True, text=True, timeout=timeout)
    line = out.stdout.strip().splitlines()[-1] if out.stdout.strip() else ""
    try:
        d = json.loads(line)
    except json.JSONDecodeError:
        raise RuntimeError(f"oracle failed ({out.returncode}): {out.stdout}\n{out.stderr}")
    if "error" in d:
        raise ValueError(d["error"])
    return d


def info(spec, threads: int = 1, hash: bool = False, native: Optional[str] = None,
         native_check: bool = False, timeout=None) -> dict:
    with tempfile.TemporaryDirectory() as td:
        args = ["info", _spec_path(spec, td), "--threads", threads]
        if hash:
            args.append("--hash")
        if native:
            args += ["--native", native]
        if native_check:
            args.append("--native-check")
        return _run(args, timeout)


def width(spec) -> bool:
    """True when some value of the spec lies outside int32: the oracle's row files (o1 / leaves /
    decode output, check input) are then int64 instead of int32 (reading #22)."""
    with tempfile.TemporaryDirectory() as td:
        return bool(_run(["width", _spec_path(spec, td)])["w64"])


def vdtype(spec):
    return np.int64 if width(spec) else np.int32


def o1(spec, timeout=None):
    """Literal brute force over the full product; rows (int32 [S][P], int64 for specs with values
    outside int32) in canonical order."""
    dt = vdtype(spec)
    with tempfile.TemporaryDirectory() as td:
        out = os.path.join(td, "rows.bin")
        d = _run(["o1", _spec_path(spec, td), out], timeout)
        rows = np.fromfile(out, dtype=dt) if os.path.exists(out) else np.zeros(0, dt)
        P = len(spec.params) if not isinstance(spec, str) else None
        return d, (rows.reshape(-1, P) if P else rows)


def leaves(spec, group: int, n_members: int, timeout=None) -> np.ndarray:
    dt = vdtype(spec)
    with tempfile.TemporaryDirectory() as td:
        out = os.path.join(td, "leaves.bin")
        _run(["leaves", _spec_path(spec, td), group, out], timeout)
        return np.fromfile(out, dtype=dt).reshape(-1, n_members)


def decode(spec, indices: np.ndarray, threads: int = 1, want_rows: bool = True, timeout=None):
    """indices (uint64) -> (info, int32 SoA [P][n] or None; int64 for specs with values outside
    int32).  info has 'hash' and 'invalid'."""
    dt = vdtype(spec) if want_rows else None
    with tempfile.TemporaryDirectory() as td:
        idx = os.path.join(td, "idx.bin")
        np.ascontiguousarray(indices, dtype=np.uint64).tofile(idx)
        out = os.path.join(td, "out.bin") if want_rows else "-"
        d = _run(["decode", _spec_path(spec, td), idx, out, "--threads", threads], timeout)
        if not want_rows:
            return d, None
        P = len(spec.params)
        return d, np.fromfile(out, dtype=dt).reshape(P, -1)


def check(spec, rows: np.ndarray, timeout=None, per_row: bool = False) -> dict:
    """Constraint check of configurations rows[n][P] (valid iff every parameter's
    value is in its range and every constraint holds).  per_row: also return "flags", a
    uint8 array with 1 for each valid row."""
    dt = vdtype(spec)
    with tempfile.TemporaryDirectory() as td:
        f = os.path.join(td, "rows.bin")
        np.ascontiguousarray(rows, dtype=dt).tofile(f)
        args = ["check", _spec_path(spec, td), f]
        if per_row:
            args.append(os.path.join(td, "flags.bin"))
        out = _run(args, timeout)
        if per_row:
            out["flags"] = np.fromfile(os.path.join(td, "flags.bin"), dtype=np.uint8)
        return out


def time_sample(spec, threads: int, budget_s: float, timeout=None) -> dict:
    with tempfile.TemporaryDirectory() as td:
        return _run(["time", _spec_path(spec, td), "--threads", threads, "--budget", budget_s], timeout)


def rowhash_rows(rows: np.ndarray, w64: bool = False) -> int:
    """Order-dependent hash H = sum_i rowhash(row_i) * (2i+1) mod 2^64 (same definition as the
    C++ oracle's; used to compare large row sequences without storing them).  w64: the spec has
    values outside int32 and its rows hash their full 64-bit values."""
    rows = np.ascontiguousarray(rows)
    n = rows.shape[0]
    with np.errstate(over="ignore"):
        z = np.full(n, 0x243F6A8885A308D3, dtype=np.uint64)
        for k in range(rows.shape[1]):
            col = rows[:, k].astype(np.int64).astype(np.uint64)
            z ^= col if w64 else col & np.uint64(0xFFFFFFFF)
            z *= np.uint64(0x9E3779B97F4A7C15)
            z ^= z >> np.uint64(32)
        w = np.arange(n, dtype=np.uint64) * np.uint64(2) + np.uint64(1)
        return int((z * w).sum(dtype=np.uint64))
