"""Thin Python front end over the C ABI (argument marshalling only).

``Space`` builds an ``atf_space`` from an :class:`atfspec.Spec` (names, ranges,
constraint bytecode — PAPER.md P:49-59), lets PyTorch provide device memory
(caching allocator) and the CUDA stream, and exposes generate / size / decode.
"""
from __future__ import annotations

import ctypes as C
import json
from typing import Dict, List, Optional

from . import _lib as L


def _range_struct(rng: dict):
    kind = rng["kind"]
    if kind == "interval":
        return L.atf_range(L.ATF_RANGE_INTERVAL, rng["begin"], rng["end"], rng.get("step", 1), None, 0), None
    if kind == "pow2":
        return L.atf_range(L.ATF_RANGE_POW2, rng["begin"], rng["end"], rng.get("step", 1), None, 0), None
    if kind == "gen":
        code = (C.c_int32 * max(1, len(rng["code"])))(*rng["code"])
        return L.atf_range(L.ATF_RANGE_GEN, rng["begin"], rng["end"], rng.get("step", 1),
                           C.cast(code, C.POINTER(C.c_int32)), len(rng["code"])), code
    if kind == "set":
        v = [int(x) for x in rng["values"]]
        if any(x < -2 ** 31 or x >= 2 ** 31 for x in v):  # int64 values (reading #22)
            vals = (C.c_int64 * max(1, len(v)))(*v)
            return L.atf_range(L.ATF_RANGE_SET64, 0, 0, 0, None, len(v), C.cast(vals, C.POINTER(C.c_int64))), vals
        vals = (C.c_int32 * max(1, len(v)))(*v)
        return L.atf_range(L.ATF_RANGE_SET, 0, 0, 0, C.cast(vals, C.POINTER(C.c_int32)), len(v)), vals
    raise ValueError(f"unknown range kind {kind}")


class Space:
    """One search space on one device.

    flags: L.ATF_FLAG_TIMING (per-level device times) | L.ATF_FLAG_GENERIC_ONLY
    (interpret every candidate with the generic bytecode interpreter).
    """

    def __init__(self, spec=None, device: int = 0, stream=None, flags: int = 0, torch_alloc: bool = True,
                 _load_path: Optional[str] = None):
        self._h = C.c_void_p()
        self._bufs: Dict[int, object] = {}
        self._device = device
        self._stream_obj = stream
        stream_ptr = None
        self._alloc_cb = L.ALLOC_FN()
        self._free_cb = L.FREE_FN()
        if torch_alloc or stream is not None:
            import torch
            if torch.cuda.is_available():
                if stream is None:
                    stream = torch.cuda.current_stream(device)
                self._stream_obj = stream
                stream_ptr = stream.cuda_stream
                if torch_alloc:
                    dev = torch.device("cuda", device)

                    def _alloc(nbytes, _stream, _ctx):
                        try:
                            with torch.cuda.stream(self._stream_obj):
                                t = torch.empty(int(nbytes), dtype=torch.uint8, device=dev)
                        except RuntimeError:
                            return None
                        p = t.data_ptr()
                        self._bufs[p] = t
                        return p

                    def _free(ptr, _nbytes, _stream, _ctx):
                        self._bufs.pop(ptr, None)

                    self._alloc_cb = L.ALLOC_FN(_alloc)
                    self._free_cb = L.FREE_FN(_free)
        opts = L.atf_space_opts(device, stream_ptr, self._alloc_cb, self._free_cb, None, flags)
        self.names: List[str] = []
        self._labels: List[Optional[List[str]]] = []  # enum names per parameter (atfspec.enum)
        if _load_path is not None:
            st = L.atf_space_load(C.byref(opts), str(_load_path).encode(), C.byref(self._h))
            if st != L.ATF_OK:
                try:
                    L.check(st, self._h)
                finally:
                    L.atf_space_destroy(self._h)
                    self._h = C.c_void_p()
            n = C.c_int32()
            L.check(L.atf_space_num_params(self._h, C.byref(n)), self._h)
            for p in range(n.value):
                ln = C.c_size_t()
                L.check(L.atf_space_param_name(self._h, p, None, 0, C.byref(ln)), self._h)
                buf = C.create_string_buffer(ln.value + 1)
                L.check(L.atf_space_param_name(self._h, p, buf, ln.value + 1, None), self._h)
                self.names.append(buf.value.decode())
                self._labels.append(None)
            return
        L.check(L.atf_space_create(C.byref(opts), C.byref(self._h)))
        if spec is not None:
            self.add_spec(spec)

    @classmethod
    def load(cls, path, device: int = 0, stream=None, flags: int = 0, torch_alloc: bool = True) -> "Space":
        """A space saved by `save` (checkpoint / resume): GENERATED, ready for decode / encode."""
        return cls(None, device=device, stream=stream, flags=flags, torch_alloc=torch_alloc, _load_path=path)

    def save(self, path) -> None:
        """Write the generated space (spec + level arrays) to `path` (atf_space_save)."""
        L.check(L.atf_space_save(self._h, str(path).encode()), self._h)

    # ---- building
    def add_spec(self, spec) -> None:
        for p in spec.params:
            pid = self.add_param(p.name, p.range)
            for code in p.constraints:
                self.add_constraint(pid, code)

    def add_param(self, name: str, rng: dict) -> int:
        st, keep = _range_struct(rng)
        out = C.c_int32()
        L.check(L.atf_space_add_param(self._h, name.encode(), C.byref(st), C.byref(out)), self._h)
        self.names.append(name)
        self._labels.append(rng.get("names"))
        return out.value

    def add_constraint(self, pid: int, code) -> None:
        arr = (C.c_int32 * len(code))(*[int(w) for w in code])
        L.check(L.atf_space_add_constraint(self._h, pid, arr, len(code)), self._h)

    # ---- planning
    def plan(self) -> None:
        L.check(L.atf_space_plan(self._h), self._h)

    def num_groups(self) -> int:
        out = C.c_int32()
        L.check(L.atf_space_num_groups(self._h, C.byref(out)), self._h)
        return out.value

    def groups(self) -> List[List[int]]:
        res = []
        for g in range(self.num_groups()):
            buf = (C.c_int32 * 64)()
            n = C.c_int32()
            L.check(L.atf_space_group_members(self._h, g, buf, 64, C.byref(n)), self._h)
            res.append(list(buf[: n.value]))
        return res

    def plan_json(self) -> dict:
        n = C.c_size_t()
        L.check(L.atf_space_plan_json(self._h, None, 0, C.byref(n)), self._h)
        buf = C.create_string_buffer(n.value + 1)
        L.check(L.atf_space_plan_json(self._h, buf, n.value + 1, None), self._h)
        return json.loads(buf.value.decode())

    # ---- generation
    def generate(self) -> None:
        L.check(L.atf_space_generate(self._h), self._h)

    def generate_shard(self, rank: int, world: int) -> List[int]:
        cap = 64 * 64
        buf = (C.c_int64 * cap)()
        n = C.c_int32()
        L.check(L.atf_space_generate_shard(self._h, rank, world, buf, cap, C.byref(n)), self._h)
        return list(buf[: n.value])

    def generate_dist(self, rank: int, world: int, allgather) -> None:
        """Balanced multi-GPU generation (atf_space_generate_dist): `allgather(data: bytes) ->
        bytes` must return the concatenation of every rank's `data` in rank order."""
        err = []

        def _cb(send, recv, nbytes, _ctx):
            try:
                out = allgather(C.string_at(send, nbytes))
                assert len(out) == nbytes * world
                C.memmove(recv, out, len(out))
                return 0
            except Exception as ex:  # noqa: BLE001 -- reported through the status code
                err.append(ex)
                return 1

        cb = L.ALLGATHER_FN(_cb)
        st = L.atf_space_generate_dist(self._h, rank, world, cb, None)
        if err:
            raise err[0]
        L.check(st, self._h)

    def dist_round_ms(self) -> List[float]:
        """Device time of each round of the last generate_dist (ATF_FLAG_TIMING)."""
        n = C.c_int32()
        L.check(L.atf_space_dist_round_ms(self._h, None, 0, C.byref(n)), self._h)
        buf = (C.c_float * max(1, n.value))()
        L.check(L.atf_space_dist_round_ms(self._h, buf, n.value, C.byref(n)), self._h)
        return list(buf[: n.value])

    def finalize_shard(self, all_counts: List[List[int]]) -> None:
        world = len(all_counts)
        n = len(all_counts[0])
        flat = (C.c_int64 * (world * n))(*[int(c) for row in all_counts for c in row])
        L.check(L.atf_space_finalize_shard(self._h, flat, world, n), self._h)

    def size(self) -> int:
        lo, hi = C.c_uint64(), C.c_uint64()
        L.check(L.atf_space_size(self._h, C.byref(lo), C.byref(hi)), self._h)
        return (hi.value << 64) | lo.value

    def group_sizes(self) -> List[int]:
        out = []
        for g in range(self.num_groups()):
            v = C.c_uint64()
            L.check(L.atf_space_group_size(self._h, g, C.byref(v)), self._h)
            out.append(v.value)
        return out

    def num_levels(self, g: int) -> int:
        v = C.c_int32()
        L.check(L.atf_space_num_levels(self._h, g, C.byref(v)), self._h)
        return v.value

    def level_sizes(self, g: int) -> List[int]:
        out = []
        for k in range(self.num_levels(g)):
            v = C.c_uint64()
            L.check(L.atf_space_level_size(self._h, g, k, C.byref(v)), self._h)
            out.append(v.value)
        return out

    def level_view(self, g: int, k: int) -> dict:
        v = L.atf_level_view()
        L.check(L.atf_space_level_view(self._h, g, k, C.byref(v)), self._h)
        return {f: getattr(v, f) for f, _ in L.atf_level_view._fields_}

    def level_tensors(self, g: int, k: int):
        """Zero-copy torch views of level k of group g: (records int32 [n, words], csr int64 [n+1] or
        None for the leaf level).  Valid until the space is regenerated or closed."""
        import torch
        v = self.level_view(g, k)

        class _CAI:
            def __init__(self, ptr, shape, typestr):
                self.__cuda_array_interface__ = {"shape": shape, "typestr": typestr, "data": (ptr, False),
                                                 "version": 3}

        dev = torch.device("cuda", self._device)
        n, W = v["n_nodes"], v["words"]
        rec = (torch.as_tensor(_CAI(v["records"], (n, W), "<i4"), device=dev) if n and v["records"]
               else torch.zeros((0, W), dtype=torch.int32, device=dev))
        nc = v["csr_nodes"]
        csr = torch.as_tensor(_CAI(v["csr"], (nc + 1,), "<i8"), device=dev) if v["csr"] else None
        return rec, csr

    def stats(self) -> List[dict]:
        n = C.c_int32()
        L.check(L.atf_space_stats(self._h, None, 0, C.byref(n)), self._h)
        arr = (L.atf_level_stats * max(1, n.value))()
        L.check(L.atf_space_stats(self._h, arr, n.value, C.byref(n)), self._h)
        return [{f: getattr(arr[i], f) for f, _ in L.atf_level_stats._fields_} for i in range(n.value)]

    # ---- decode (device tensors in, device tensor out)
    def value_bits(self) -> int:
        """32 if every parameter value fits int32, else 64 (configurations are then int64)."""
        b = C.c_int32()
        L.check(L.atf_space_value_bits(self._h, C.byref(b)), self._h)
        return b.value

    def _out(self, out, P, n, device):
        import torch
        if out is not None:
            return out, out.dtype == torch.int64
        w64 = self.value_bits() == 64
        return torch.empty((P, n), dtype=torch.int64 if w64 else torch.int32, device=device), w64

    def decode(self, idx, out=None, stream=None):
        """idx: CUDA tensor of uint64/int64 indices [n] -> int32 tensor [P, n] (SoA); int64 for a
        space with values outside int32 (or when `out` is int64)."""
        n = idx.numel()
        out, w64 = self._out(out, len(self.names), n, idx.device)
        sp = stream.cuda_stream if stream is not None else None
        fn = L.atf_space_decode_indices_i64 if w64 else L.atf_space_decode_indices
        L.check(fn(self._h, idx.data_ptr(), n, out.data_ptr(), out.stride(0), sp), self._h)
        return out

    def decode_range(self, first: int, n: int, out=None, stream=None):
        """The n consecutive indices first, first + 1, ... (any S, u128 in the library) ->
        int32 tensor [P, n] (int64 as for decode)."""
        import torch
        out, w64 = self._out(out, len(self.names), n, torch.device("cuda", self._device))
        sp = stream.cuda_stream if stream is not None else None
        fn = L.atf_space_decode_range_i64 if w64 else L.atf_space_decode_range
        L.check(fn(self._h, first & ((1 << 64) - 1), first >> 64, n, out.data_ptr(), out.stride(0), sp), self._h)
        return out

    def decode128(self, idx_lo, idx_hi, out=None, stream=None):
        """u128 indices hi * 2^64 + lo (CUDA int64 tensors holding the u64 halves) -> int32 [P, n]."""
        import torch
        n = idx_lo.numel()
        P = len(self.names)
        if out is None:
            out = torch.empty((P, n), dtype=torch.int32, device=idx_lo.device)
        idx_lo, idx_hi = idx_lo.contiguous(), idx_hi.contiguous()
        sp = stream.cuda_stream if stream is not None else None
        L.check(L.atf_space_decode_indices128(self._h, idx_lo.data_ptr(), idx_hi.data_ptr(), n, out.data_ptr(),
                                              out.stride(0), sp), self._h)
        return out

    def decode_digits(self, digits, out=None, stream=None):
        """digits: CUDA tensor [G, n] of per-group indices -> int32 tensor [P, n] (int64 as for
        decode)."""
        n = digits.shape[1]
        out, w64 = self._out(out, len(self.names), n, digits.device)
        digits = digits.contiguous()
        sp = stream.cuda_stream if stream is not None else None
        fn = L.atf_space_decode_digits_i64 if w64 else L.atf_space_decode_digits
        L.check(fn(self._h, digits.data_ptr(), n, out.data_ptr(), out.stride(0), sp), self._h)
        return out

    # ---- encode (inverse of decode; membership)
    def encode(self, values, stream=None):
        """values: int32 CUDA tensor [P, n] (SoA, one configuration per column) -> int64
        tensor [n] of 0-based indices, -1 where the configuration is not in the space
        (requires S < 2^64)."""
        import torch
        values = values.to(torch.int32)
        if values.stride(1) != 1:
            values = values.contiguous()
        n = values.shape[1]
        G = self.num_groups()
        dig = torch.empty((G, n), dtype=torch.int64, device=values.device)
        idx = torch.empty(n, dtype=torch.int64, device=values.device)
        sp = stream.cuda_stream if stream is not None else None
        L.check(L.atf_space_encode_indices(self._h, values.data_ptr(), n, values.stride(0), dig.data_ptr(),
                                           idx.data_ptr(), sp), self._h)
        return idx  # UINT64_MAX reads as -1 in int64

    def encode_digits(self, values, stream=None):
        """values: int32 CUDA tensor [P, n] -> int64 tensor [G, n] of per-group leaf indices
        (-1 where the group's values are not a valid path); works for any S."""
        import torch
        values = values.to(torch.int32)
        if values.stride(1) != 1:
            values = values.contiguous()
        n = values.shape[1]
        dig = torch.empty((self.num_groups(), n), dtype=torch.int64, device=values.device)
        sp = stream.cuda_stream if stream is not None else None
        L.check(L.atf_space_encode_digits(self._h, values.data_ptr(), n, values.stride(0), dig.data_ptr(), sp),
                self._h)
        return dig

    def filter_product(self):
        """CLTune-style baseline: count the valid tuples of the FULL cartesian
        product on the GPU (every tuple enumerated, every constraint interpreted).
        Returns (valid tuples = S, product size)."""
        cnt, tot = C.c_uint64(), C.c_uint64()
        L.check(L.atf_space_filter_product(self._h, C.byref(cnt), C.byref(tot)), self._h)
        return cnt.value, tot.value

    def neighbors(self, values, seed: int, max_tries: int = 16, stream=None):
        """values: int32 CUDA tensor [P, n] of valid configurations -> (int32 [P, n] neighbours,
        int32 [n] changed parameter id or -1); one parameter re-drawn per row."""
        import torch
        values = values.to(torch.int32)
        if values.stride(1) != 1:
            values = values.contiguous()
        P, n = values.shape
        out = torch.empty((P, n), dtype=torch.int32, device=values.device)
        moved = torch.empty(n, dtype=torch.int32, device=values.device)
        sp = stream.cuda_stream if stream is not None else None
        L.check(L.atf_space_neighbors(self._h, values.data_ptr(), values.stride(0), n, seed & ((1 << 64) - 1),
                                      max_tries, out.data_ptr(), out.stride(0), moved.data_ptr(), sp), self._h)
        return out, moved

    def to_named(self, configs) -> List[dict]:
        """Decoded configurations (int32 [P, n]) -> one dict per configuration, parameter name ->
        value, with the names of enum parameters (atfspec.enum) in place of their codes.
        Host-side formatting for display / logging."""
        cols = configs.cpu().numpy() if hasattr(configs, "cpu") else configs
        names = self._labels
        out = []
        for j in range(cols.shape[1]):
            row = {}
            for p, nm in enumerate(self.names):
                v = int(cols[p, j])
                row[nm] = names[p][v] if names[p] is not None else v
            out.append(row)
        return out

    def close(self) -> None:
        if self._h:
            L.atf_space_destroy(self._h)
            self._h = C.c_void_p()
            self._bufs.clear()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
