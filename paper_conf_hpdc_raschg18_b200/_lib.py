"""ctypes binding of libatfgen.so — the C ABI declared in include/atfgen.h.

Argument marshalling only: every step of the generation and decode path runs in
the library's sm_100a kernels.  The functions below have the C names.  There is
no fallback: if the shared library is missing, importing this module raises.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ATF_LIB_PATH") or os.path.join(HERE, "libatfgen.so")  # override: A/B builds

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'` "
                      f"(or `make -C {os.path.join(HERE, 'csrc')}`)")

lib = C.CDLL(LIB_PATH)

# ---- status codes (include/atfgen.h) ----
ATF_OK = 0
STATUS = {0: "ATF_OK", -1: "ATF_ERR_INVALID_ARG", -2: "ATF_ERR_OOM", -3: "ATF_ERR_CUDA", -4: "ATF_ERR_STATE",
          -5: "ATF_ERR_BYTECODE", -6: "ATF_ERR_FORWARD_REF", -7: "ATF_ERR_OVERFLOW", -8: "ATF_ERR_INDEX",
          -9: "ATF_ERR_DUPLICATE", -10: "ATF_ERR_LIMIT"}
ATF_RANGE_INTERVAL, ATF_RANGE_POW2, ATF_RANGE_SET, ATF_RANGE_GEN, ATF_RANGE_SET64 = 0, 1, 2, 3, 4
ATF_FLAG_TIMING, ATF_FLAG_GENERIC_ONLY, ATF_FLAG_LEGACY_WIDE, ATF_FLAG_NO_JIT, ATF_FLAG_SERIAL_GROUPS = 1, 2, 8, 16, 32
ATF_FLAG_NO_SEG_BOUNDS = 64
ATF_FLAG_NO_TAIL = 128
ATF_FLAG_NO_REPLAY = 256
ATF_FLAG_DIST_SUBSETS = 512        # default since round 2 (no-op)
ATF_FLAG_DIST_NO_SUBSETS = 1024


class atf_range(C.Structure):
    _fields_ = [("kind", C.c_int32), ("begin", C.c_int64), ("end", C.c_int64), ("step", C.c_int64),
                ("values", C.POINTER(C.c_int32)), ("n_values", C.c_int64), ("values64", C.POINTER(C.c_int64))]


ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
ALLGATHER_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p)


class atf_space_opts(C.Structure):
    _fields_ = [("device", C.c_int32), ("stream", C.c_void_p), ("alloc", ALLOC_FN), ("free", FREE_FN),
                ("alloc_ctx", C.c_void_p), ("flags", C.c_uint32)]


class atf_level_view(C.Structure):
    _fields_ = [("records", C.c_void_p), ("csr", C.c_void_p), ("n_nodes", C.c_uint64), ("offset", C.c_uint64),
                ("words", C.c_int32), ("param", C.c_int32), ("field_word", C.c_int32),
                ("field_shift", C.c_int32), ("field_bits", C.c_int32), ("csr_offset", C.c_uint64),
                ("csr_nodes", C.c_uint64)]


class atf_level_stats(C.Structure):
    _fields_ = [("group", C.c_int32), ("level", C.c_int32), ("param", C.c_int32), ("r", C.c_int64),
                ("evals", C.c_uint64), ("f", C.c_uint64), ("ms", C.c_float), ("path", C.c_int32),
                ("expand_ms", C.c_float), ("kernel", C.c_int32),
                ("pairs", C.c_uint64), ("cpt", C.c_int32), ("nseg", C.c_int32), ("launches", C.c_int32)]


SP = C.c_void_p  # atf_space*
_st = C.c_int32

_SIGS = {
    "atf_space_create": (_st, [C.POINTER(atf_space_opts), C.POINTER(SP)]),
    "atf_space_add_param": (_st, [SP, C.c_char_p, C.POINTER(atf_range), C.POINTER(C.c_int32)]),
    "atf_space_add_constraint": (_st, [SP, C.c_int32, C.POINTER(C.c_int32), C.c_int32]),
    "atf_space_plan": (_st, [SP]),
    "atf_space_num_params": (_st, [SP, C.POINTER(C.c_int32)]),
    "atf_space_num_groups": (_st, [SP, C.POINTER(C.c_int32)]),
    "atf_space_group_members": (_st, [SP, C.c_int32, C.POINTER(C.c_int32), C.c_int32, C.POINTER(C.c_int32)]),
    "atf_space_plan_json": (_st, [SP, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
    "atf_space_generate": (_st, [SP]),
    "atf_space_generate_shard": (_st, [SP, C.c_int32, C.c_int32, C.POINTER(C.c_int64), C.c_int32,
                                       C.POINTER(C.c_int32)]),
    "atf_space_finalize_shard": (_st, [SP, C.POINTER(C.c_int64), C.c_int32, C.c_int32]),
    "atf_space_size": (_st, [SP, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]),
    "atf_space_group_size": (_st, [SP, C.c_int32, C.POINTER(C.c_uint64)]),
    "atf_space_num_levels": (_st, [SP, C.c_int32, C.POINTER(C.c_int32)]),
    "atf_space_level_size": (_st, [SP, C.c_int32, C.c_int32, C.POINTER(C.c_uint64)]),
    "atf_space_level_view": (_st, [SP, C.c_int32, C.c_int32, C.POINTER(atf_level_view)]),
    "atf_space_decode_indices": (_st, [SP, C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_space_decode_indices128": (_st, [SP, C.c_void_p, C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_space_decode_range": (_st, [SP, C.c_uint64, C.c_uint64, C.c_int64, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_space_decode_digits": (_st, [SP, C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_space_decode_indices_i64": (_st, [SP, C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_space_decode_digits_i64": (_st, [SP, C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_space_decode_range_i64": (_st, [SP, C.c_uint64, C.c_uint64, C.c_int64, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_space_value_bits": (_st, [SP, C.POINTER(C.c_int32)]),
    "atf_space_save": (_st, [SP, C.c_char_p]),
    "atf_space_load": (_st, [C.POINTER(atf_space_opts), C.c_char_p, C.POINTER(SP)]),
    "atf_space_param_name": (_st, [SP, C.c_int32, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
    "atf_space_encode_digits": (_st, [SP, C.c_void_p, C.c_int64, C.c_int64, C.c_void_p, C.c_void_p]),
    "atf_space_encode_indices": (_st, [SP, C.c_void_p, C.c_int64, C.c_int64, C.c_void_p, C.c_void_p, C.c_void_p]),
    "atf_space_filter_product": (_st, [SP, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]),
    "atf_space_neighbors": (_st, [SP, C.c_void_p, C.c_int64, C.c_int64, C.c_uint64, C.c_int32, C.c_void_p, C.c_int64,
                                  C.c_void_p, C.c_void_p]),
    "atf_space_stats": (_st, [SP, C.POINTER(atf_level_stats), C.c_int32, C.POINTER(C.c_int32)]),
    "atf_space_generate_dist": (_st, [SP, C.c_int32, C.c_int32, ALLGATHER_FN, C.c_void_p]),
    "atf_space_dist_round_ms": (_st, [SP, C.POINTER(C.c_float), C.c_int32, C.POINTER(C.c_int32)]),
    "atf_space_destroy": (None, [SP]),
    "atf_status_str": (C.c_char_p, [_st]),
    "atf_space_last_error": (C.c_char_p, [SP]),
    # include/atfgen_test.h
    "atf_test_divisible16": (_st, [C.POINTER(C.c_uint64)]),
    "atf_test_set_tail_stage": (_st, [C.c_int32]),
    "atf_test_set_geometry": (_st, [C.c_int32, C.c_int32]),
    "atf_test_set_direct_tiles": (_st, [C.c_int32]),
    "atf_test_set_tail_product": (_st, [C.c_int32]),
    "atf_test_set_async_rounds": (_st, [C.c_int32]),
    "atf_test_set_tail_leaf_direct": (_st, [C.c_int32]),
    "atf_test_set_wide_group": (_st, [C.c_int32]),
    "atf_test_jit_source": (_st, [SP, C.c_int32, C.c_int32, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
    "atf_test_tail_source": (_st, [SP, C.c_int32, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t),
                                   C.POINTER(C.c_int32)]),
    "atf_test_exclusive_scan_u32": (_st, [C.c_void_p, C.c_void_p, C.c_int64, C.c_void_p]),
    "atf_test_shard_slice": (_st, [C.POINTER(C.c_uint64), C.c_uint64, C.c_int32, C.c_int32,
                                   C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]),
    "atf_test_shard_offsets": (_st, [C.POINTER(C.c_int64), C.c_int32, C.c_int32, C.c_int32,
                                     C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]),
}

EXPORTED = tuple(_SIGS)

for _name, (_res, _args) in _SIGS.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args
    globals()[_name] = _f


class AtfError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def check(status: int, space=None) -> None:
    if status != ATF_OK:
        msg = atf_space_last_error(space).decode() if space else atf_status_str(status).decode()
        raise AtfError(status, msg)
