"""Host-side checks of the C-ABI boundary (no GPU needed, no compute calls)."""
import os
import re

import numpy as np
import pytest

import graphgen as gg
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _lib():
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    return asc


def test_library_exports_every_declared_symbol():
    asc = _lib()
    hdr = open(os.path.join(ROOT, "include", "ascetic.h")).read()
    declared = set(re.findall(r"\b(ascetic_[a-z_0-9]+)\s*\(", hdr))
    assert declared, "no declarations parsed"
    for name in declared:
        assert hasattr(asc._lib, name), f"{name} declared in ascetic.h but not exported"
    assert declared <= set(asc.EXPORTS)
    assert "sm_100a" in asc.version()


def test_state_machine_without_gpu():
    asc = _lib()
    asc.unload()
    with pytest.raises(asc.AsceticError) as e:
        asc.run("bfs", 0)
    assert e.value.code == asc.ESTATE
    with pytest.raises(asc.AsceticError) as e:
        asc.set_budget(1 << 20)
    assert e.value.code == asc.ESTATE
    with pytest.raises(asc.AsceticError) as e:
        asc.stats()
    assert e.value.code == asc.ESTATE


def test_load_csr_validation_without_gpu():
    asc = _lib()
    nbr = np.array([1, 0], dtype=np.uint32)
    for bad in ([1, 1, 2], [0, 2, 1], [0, 1, 3]):
        with pytest.raises(asc.AsceticError) as e:
            asc.load_csr(np.array(bad, dtype=np.uint64), nbr)
        assert e.value.code == asc.EINVAL
    with pytest.raises(asc.AsceticError) as e:
        asc.load_csr(np.array([0, 1, 2], dtype=np.uint64), np.array([1, 5], dtype=np.uint32), validate=True)
    assert e.value.code == asc.EINVAL
    with pytest.raises(TypeError):
        asc.load_csr(np.array([0, 1, 2], dtype=np.int64), nbr)


@pytest.mark.parametrize("b_e", [4, 8])
def test_library_placer_matches_oracle(b_e):
    """The library's placer (its own C++ code) agrees with the oracle's Eq. 2 placer everywhere."""
    asc = _lib()
    g = gg.rmat(13, seed=5)
    D = b_e * g.m
    for budget in [0, 1, 16383, 16384, 100_000, D // 10, D // 4, D // 2, D - 1, D, 2 * D]:
        for frac in [-1.0, 0.0, 0.25, 0.97, 1.0]:
            mine = asc.place(g.off, b_e, budget, frac)
            ref = oracle.placer(g.off, b_e, budget, frac)
            for k in ["R", "D", "B", "Ms", "s", "static_bytes", "C", "cap"]:
                assert mine[k] == getattr(ref, k), (budget, frac, k)


def test_place_rejects_bad_fraction():
    asc = _lib()
    off = np.array([0, 4], dtype=np.uint64)
    for f in [1.5, float("nan")]:
        with pytest.raises(asc.AsceticError) as e:
            asc.place(off, 4, 1 << 20, f)
        assert e.value.code == asc.EINVAL


def test_binding_mirrors_header_enums_and_structs():
    """The ctypes binding's option ids, load flags and stats fields follow include/ascetic.h."""
    asc = _lib()
    hdr = open(os.path.join(ROOT, "include", "ascetic.h")).read()
    opts = {m.group(1).lower(): int(m.group(2)) for m in re.finditer(r"ASCETIC_OPT_([A-Z_0-9]+)\s*=\s*(\d+)", hdr)}
    assert opts == asc.OPTIONS
    flags = {m.group(1): int(m.group(2)) for m in re.finditer(r"ASCETIC_([A-Z]+)\s*=\s*(\d+)u", hdr)}
    assert flags == {"SYMMETRIC": asc.SYMMETRIC, "COPY": asc.COPY, "VALIDATE": asc.VALIDATE, "PAIRS": asc.PAIRS,
                     "SORTED": asc.SORTED}
    body = hdr[hdr.index("typedef struct {\n    int32_t algo;"):hdr.index("} ascetic_stats_t;")]
    names = re.findall(r"^\s*(?:u?int(?:32|64)_t|double)\s+([a-z_0-9, ]+);", body, re.M)
    fields = [f.strip() for grp in names for f in grp.split(",")]
    assert fields == [f for f, _ in asc.Stats._fields_]
