"""The C-ABI library builds, loads without a GPU and exports every entry point include/sieve.h
declares; host-only utilities work.  (No compute call is made here: there is no GPU.)"""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from tools.build_native import build_lib
    build_lib()
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    return sieve


def _declared():
    src = open(os.path.join(ROOT, "include", "sieve.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sieve_[a-z0-9_]+)\s*\(", src)) -
                  {"sieve_alloc_fn", "sieve_free_fn"})


def test_exports_every_declared_symbol(lib):
    L = ctypes.CDLL(lib.LIB_PATH)
    names = _declared()
    assert len(names) >= 20
    for n in names:
        assert hasattr(L, n), n
    assert sorted(lib.EXPORTED) == names


def test_version_and_limbs(lib):
    assert "sm_100a" in lib.version()
    for v in [0, 1, (1 << 64) - 1, 1 << 64, (1 << 128) - 1, 0x0123456789ABCDEF_FEDCBA9876543210]:
        limbs = lib.u128_to_limbs(v)
        assert all(0 <= l < (1 << 32) for l in limbs)
        assert lib.limbs_to_u128(limbs) == v
    # lane sums of many ranks' limbs normalise back to the exact sum
    vals = [(1 << 128) // 7 - 12345, (1 << 100) + 3, (1 << 127) // 5]
    lanes = [sum(l) for l in zip(*[lib.u128_to_limbs(v) for v in vals])]
    assert lib.limbs_to_u128(lanes) == sum(vals)


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ispass_naderantahanse23_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                s = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", s).lower().replace("oracle/ ", ""), f


def test_stratum_struct_size(lib):
    assert lib.STRATUM_DTYPE.itemsize == 96


def test_binding_validates_before_the_library_reads():
    """the binding rejects arguments the library would read out of bounds"""
    import numpy as np
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    kid = np.zeros(10, np.uint32)
    x = np.ones(9, np.uint64)

    class _Ctx:  # no GPU needed: the checks run before any library call
        device = 0
        _h = None
    with pytest.raises(ValueError):
        sieve.load_trace(_Ctx(), kid, x, num_kernels=1)
    with pytest.raises(ValueError):
        sieve.load_trace(_Ctx(), kid, np.ones(10, np.uint64), num_kernels=1, cycles=np.ones(3, np.uint64))

    class _Trace:
        n = 10
        ctx = _Ctx()
    with pytest.raises(TypeError):
        sieve.sieve._check_sid(torch.zeros(10, dtype=torch.int32), _Trace())   # host tensor

    class _Strata:
        _h = None

        def __len__(self):
            return 5
    with pytest.raises(ValueError):
        sieve.predict(_Strata(), _Trace(), rep_cycles=np.ones(4, np.uint64))
