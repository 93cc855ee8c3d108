"""C-ABI library checks that need no GPU: it loads, exports every symbol include/mf.h declares,
and its host-only logic (parameter defaults, strata planner) is right."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_hpdc_xietfl17_b200 import build, mf

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    build.build()
    return mf.lib()


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "mf.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(mf_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol(L):
    names = declared_symbols()
    assert "mf_train_epoch" in names and "mf_create" in names and len(names) >= 15
    for name in names:
        assert hasattr(L, name), name
    assert set(names) <= set(mf.EXPORTED)


def test_python_binding_has_every_abi_name(L):
    """The binding is thin and named like the boundary: one same-named Python callable per
    include/mf.h entry point (argument marshalling only)."""
    for name in declared_symbols():
        assert callable(getattr(mf, name, None)), name
    assert mf.mf_abi_version() == L.mf_abi_version()
    assert mf.mf_status_string(-6) == "MF_E_RANGE"
    assert mf.mf_params_default().batch_f == 256


def test_abi_version_and_status_strings(L):
    hdr = open(os.path.join(ROOT, "include", "mf.h")).read()
    assert L.mf_abi_version() == int(re.search(r"#define MF_ABI_VERSION (\d+)", hdr).group(1))
    assert L.mf_status_string(-6) == b"MF_E_RANGE"


def test_params_default_and_struct_size(L):
    p = mf.Params()
    assert L.mf_params_default(ctypes.byref(p)) == 0
    assert p.struct_size == ctypes.sizeof(mf.Params)
    # Table 3 Netflix and Table 2 k
    assert (p.k, round(p.lambda_p, 6), round(p.alpha, 6), round(p.beta, 6)) == (128, 0.05, 0.08, 0.3)
    assert p.batch_f == 256 and p.world == 1


def test_create_rejects_bad_params_before_touching_a_device(L):
    p = mf.Params()
    L.mf_params_default(ctypes.byref(p))
    h = ctypes.c_void_p()
    p.m, p.n = 100, 100
    p.k = 48
    assert L.mf_create(ctypes.byref(p), ctypes.byref(h)) == -7      # k not supported
    p.k = 16
    p.storage = 5
    assert L.mf_create(ctypes.byref(p), ctypes.byref(h)) == -1
    p.storage = 0
    p.world, p.grid_a = 3, 8                                         # a % world != 0
    assert L.mf_create(ctypes.byref(p), ctypes.byref(h)) == -1
    p.world, p.grid_a = 1, 32                                        # a / world > 16 blocks
    assert L.mf_create(ctypes.byref(p), ctypes.byref(h)) == -1
    p.grid_a = 0
    p.q_cache = 2                                                    # q_cache in {0, 1}
    assert L.mf_create(ctypes.byref(p), ctypes.byref(h)) == -1
    p.q_cache = 0
    bad = mf.Params()
    assert L.mf_create(ctypes.byref(bad), ctypes.byref(h)) == -1     # struct_size unset
    assert not h.value


def test_create_refuses_combinations_no_kernel_implements(L):
    """Options that have no kernel instantiation are refused with MF_E_UNSUPPORTED at create
    (never silently run as another variant)."""
    def refused(**kw):
        p = mf.Params()
        L.mf_params_default(ctypes.byref(p))
        p.m, p.n = 1000, 800
        for kk, vv in kw.items():
            setattr(p, kk, vv)
        h = ctypes.c_void_p()
        return L.mf_create(ctypes.byref(p), ctypes.byref(h)) == -7 and not h.value
    assert refused(rating_stage=1, exact_order=1)
    assert refused(rating_stage=2, lr_rule=1)
    assert refused(rating_stage=1, schedule=1)                        # wavefront
    assert refused(rating_stage=2, k=256, storage=0)                  # 32-B lane slices
    assert refused(rating_stage=2, prefetch=2)
    assert refused(rating_stage=1, batch_f=100)                       # f % 64 != 0
    assert refused(group_cols=1, schedule=1)
    assert refused(staged=2, world=2, grid_a=8, rank=0)
    assert refused(grid_cols=1, grid_a=4, schedule=1)                # a x 1: Hogwild only
    assert refused(grid_cols=1, grid_a=4, lr_rule=1)
    assert refused(grid_cols=1, grid_a=8, world=2, rank=0)


def test_strata_holders_partition_and_rotation(L):
    """A: in sub-epoch j segment J is held by the owner of row (J - pi_t[j]) mod a; each rank
    holds exactly a/G segments per sub-epoch; pi_t is the oracle's strata order."""
    from oracle import pyoracle as po
    a = 8
    for G in (1, 2, 4, 8):
        for t in range(3):
            o = po.Oracle(16, 16, 2, [0], [0], [1.0], seed=42, grid_a=a)
            pi = o.export("strata", t)
            for j in range(a):
                h = mf.strata_holders(42, a, G, t, j)
                assert sorted(np.bincount(h, minlength=G).tolist()) == [a // G] * G
                for J in range(a):
                    r = (J - pi[j]) % a
                    assert h[J] == r // (a // G)
    with pytest.raises(mf.MFError):
        mf.strata_holders(42, 8, 3, 0, 0)


def test_comm_selftest_rejects_bad_arguments_before_touching_a_device(L):
    buf = ctypes.create_string_buffer(128)
    out = ctypes.create_string_buffer(64)
    assert L.mf_comm_selftest(None, 1, 0, 0, 0, out, 64) == -1
    assert L.mf_comm_selftest(buf, 2, 2, 0, 0, out, 64) == -1          # rank >= world
    assert L.mf_comm_selftest(buf, 1, 0, 0, 3, out, 64) == -1          # transport
    assert out.value == b"bad arguments"
