"""Checkpoint / resume of a generated space (atf_space_save / atf_space_load).

CPU part: argument / state / file validation without a GPU.  GPU part: save -> load round trips
whose sizes, level sizes and every decoded configuration equal the original space's and the
oracle's; corrupted and truncated files are rejected.
"""
import os

import numpy as np
import pytest

import atfspec as A
from oracle import run as orc


def _status(fn):
    from paper_conf_hpdc_raschg18_b200 import AtfError
    with pytest.raises(AtfError) as e:
        fn()
    return e.value.status


# ---------------------------------------------------------------- CPU
def test_save_needs_a_generated_space(tmp_path):
    from paper_conf_hpdc_raschg18_b200 import Space
    sp = Space(A.c1_toy(), torch_alloc=False)
    assert _status(lambda: sp.save(tmp_path / "x.atf")) == -4          # ATF_ERR_STATE
    sp.plan()
    assert _status(lambda: sp.save(tmp_path / "x.atf")) == -4
    sp.close()


def test_load_rejects_missing_and_foreign_files(tmp_path):
    from paper_conf_hpdc_raschg18_b200 import Space
    assert _status(lambda: Space.load(tmp_path / "missing.atf", torch_alloc=False)) == -1
    bad = tmp_path / "bad.atf"
    bad.write_bytes(b"not a checkpoint at all")
    assert _status(lambda: Space.load(bad, torch_alloc=False)) == -1
    wrong = tmp_path / "v9.atf"
    wrong.write_bytes(b"ATFSPC01" + (9).to_bytes(4, "little") + bytes(16))
    assert _status(lambda: Space.load(wrong, torch_alloc=False)) == -1   # unsupported version


def test_param_names_abi():
    import ctypes as C
    from paper_conf_hpdc_raschg18_b200 import Space, _lib as L
    sp = Space(A.c3_xgemm("IS1"), torch_alloc=False)
    ln = C.c_size_t()
    L.check(L.atf_space_param_name(sp._h, 0, None, 0, C.byref(ln)), sp._h)
    assert ln.value == 3
    buf = C.create_string_buffer(3)   # truncated to cap - 1
    L.check(L.atf_space_param_name(sp._h, 0, buf, 3, None), sp._h)
    assert buf.value == b"MW"
    assert L.atf_space_param_name(sp._h, 99, None, 0, None) == -1
    sp.close()


# ---------------------------------------------------------------- GPU
def _specs():
    import sys
    sys.path.insert(0, os.path.dirname(__file__))
    from test_int64_values import mixed_groups64
    return {"C1": A.c1_toy(), "fig1": A.fig1(), "C2-16": A.c2_xgemm_direct(16), "C3-IS1": A.c3_xgemm("IS1"),
            "C5-300x4": A.c5_chains(300, 4), "mixed64": mixed_groups64(), "saxpy360": A.saxpy(360)}


@pytest.fixture(scope="module")
def GSpace():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpdc_raschg18_b200 import Space
    return Space


@pytest.mark.gpu
@pytest.mark.parametrize("name", sorted(_specs()))
def test_save_load_round_trip(GSpace, name, tmp_path):
    import torch
    spec = _specs()[name]
    path = tmp_path / f"{name}.atf"
    with GSpace(spec) as sp:
        sp.generate()
        sp.save(path)
        S, gs = sp.size(), sp.group_sizes()
        lv = [sp.level_sizes(g) for g in range(sp.num_groups())]
        n = min(S, 1 << 16)
        idx = torch.arange(n, dtype=torch.int64, device="cuda") * max(1, S // max(n, 1))
        want = sp.decode(idx).cpu().numpy()
    with GSpace.load(path) as ld:
        assert ld.names == [p.name for p in spec.params]
        assert ld.size() == S and ld.group_sizes() == gs
        assert [ld.level_sizes(g) for g in range(ld.num_groups())] == lv
        got = ld.decode(idx).cpu().numpy()
        assert np.array_equal(got, want)
        # the oracle agrees on the loaded space (every configuration of small spaces)
        if S <= 200_000:
            _, ref = orc.decode(spec, np.arange(S, dtype=np.uint64))
            allrows = ld.decode(torch.arange(S, dtype=torch.int64, device="cuda")).cpu().numpy()
            assert np.array_equal(allrows, ref)
        if ld.value_bits() == 32 and S:
            # encode walks the loaded CSR: decode -> encode is the identity
            back = ld.encode(ld.decode(idx))
            assert torch.equal(back.cpu(), idx.cpu())
        # a loaded space regenerates normally
        ld.generate()
        assert ld.size() == S and np.array_equal(ld.decode(idx).cpu().numpy(), want)


@pytest.mark.gpu
def test_load_rejects_corrupted_and_truncated(GSpace, tmp_path):
    path = tmp_path / "c5.atf"
    with GSpace(A.c5_chains(300, 3)) as sp:
        sp.generate()
        sp.save(path)
        sizes = sp.group_sizes()
    data = bytearray(path.read_bytes())
    flipped = tmp_path / "flipped.atf"
    bad = bytearray(data)
    bad[len(bad) // 2] ^= 0x40
    flipped.write_bytes(bytes(bad))
    assert _status(lambda: GSpace.load(flipped)) == -1
    cut = tmp_path / "cut.atf"
    cut.write_bytes(bytes(data[: len(data) - 100]))
    assert _status(lambda: GSpace.load(cut)) == -1
    with GSpace.load(path) as ld:   # the intact file still loads
        assert ld.group_sizes() == sizes
