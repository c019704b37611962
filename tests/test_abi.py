"""The C-ABI library loads without a GPU, exports every symbol include/xk.h declares, and
performs argument checking (BLAS XERBLA numbering, same codes as the oracle) before it
needs a device.  Also: the product package never imports the oracle (task framing ③)."""
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_sc_gautierl21_b200 as xk
from paper_conf_sc_gautierl21_b200 import _abi

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "xk.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(xk_[a-z0-9_]+)\s*\(", src)))


def test_every_declared_symbol_is_exported():
    L = xk.lib()
    decl = declared_symbols()
    assert len(decl) >= 30
    missing = [s for s in decl if getattr(L, s, None) is None]
    assert not missing, missing
    assert sorted(_abi.SYMBOLS) == decl  # the binding mirrors the header exactly


def test_not_initialized_is_an_error_not_a_crash():
    A = np.zeros((4, 4), order="F")
    with pytest.raises(xk.XKError) as e:
        xk.dgemm("N", "N", 4, 4, 4, 1.0, A, 4, A, 4, 0.0, A, 4)
    assert e.value.code == _abi.XK_ERR_NOT_INITIALIZED
    with pytest.raises(xk.XKError):
        xk.sync()


def test_argument_errors_match_oracle_codes():
    A = np.zeros((4, 4), order="F")
    cases = [("X", "N", 2, 2, 2, 4, 4, 4), ("N", "Q", 2, 2, 2, 4, 4, 4), ("N", "N", -1, 2, 2, 4, 4, 4),
             ("N", "N", 2, -1, 2, 4, 4, 4), ("N", "N", 2, 2, -1, 4, 4, 4), ("N", "N", 5, 2, 2, 4, 4, 5),
             ("T", "N", 2, 2, 5, 4, 5, 4), ("N", "N", 2, 2, 5, 4, 4, 4), ("N", "N", 5, 2, 2, 5, 4, 4)]
    for (ta, tb, m, n, k, lda, ldb, ldc) in cases:
        want = oracle.dgemm(ta, tb, m, n, k, 1.0, A, A, 0.0, A, lda=lda, ldb=ldb, ldc=ldc)
        assert want < 0
        assert xk.dgemm(ta, tb, m, n, k, 1.0, A, lda, A, ldb, 0.0, A, ldc) == want
        assert xk.dgemm_async(ta, tb, m, n, k, 1.0, A, lda, A, ldb, 0.0, A, ldc) == want
    # quick returns succeed without touching anything (even uninitialised)
    assert xk.dgemm("N", "N", 0, 4, 4, 1.0, A, 4, A, 4, 0.0, A, 4) == 0
    assert xk.dgemm("N", "N", 4, 4, 4, 0.0, A, 4, A, 4, 1.0, A, 4) == 0
    # other routines share the XERBLA numbering with the oracle
    assert xk.dsyrk("L", "N", 5, 2, 1.0, A, 4, 0.0, A, 5) == oracle.dsyrk("L", "N", 5, 2, 1.0, A, 0.0, A, lda=4, ldc=5)
    assert xk.dsyr2k("L", "N", 4, 2, 1.0, A, 4, A, 4, 0.0, A, 3) == -12
    assert xk.dsymm("L", "X", 2, 2, 1.0, A, 4, A, 4, 0.0, A, 4) == -2
    for f, of in ((xk.dtrmm, oracle.dtrmm), (xk.dtrsm, oracle.dtrsm)):
        assert f("L", "L", "N", "X", 2, 2, 1.0, A, 4, A, 4) == of("L", "L", "N", "X", 2, 2, 1.0, A, A) == -4
        assert f("L", "L", "N", "N", 4, 2, 1.0, A, 4, A, 3) == -11
    # xk_distribute_2dbc_async: argument codes checked before the library state
    assert xk.lib().xk_distribute_2dbc_async(-1, 2, None, 4, 1, 1, 1, 1) == -1
    assert xk.lib().xk_distribute_2dbc_async(2, -1, None, 4, 1, 1, 1, 1) == -2
    assert xk.lib().xk_distribute_2dbc_async(5, 2, None, 4, 1, 1, 1, 1) == -4
    assert xk.lib().xk_distribute_2dbc_async(4, 2, None, 4, 0, 1, 1, 1) == -5
    assert xk.lib().xk_distribute_2dbc_async(4, 2, None, 4, 1, 0, 1, 1) == -6
    assert xk.lib().xk_distribute_2dbc_async(4, 2, None, 4, 1, 1, 0, 1) == -7
    assert xk.lib().xk_distribute_2dbc_async(4, 2, None, 4, 1, 1, 1, 0) == -8


def test_product_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sc_gautierl21_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cpp", ".cu", ".h")):
                txt = open(os.path.join(dirpath, fn)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, fn
                assert "oracle.h" not in txt and "liboracle" not in txt, fn


def test_c_example_builds_against_the_header():
    """The C ABI is usable from plain C: examples/xk_dgemm_example.c compiles and links."""
    from tools.build_native import build_example
    assert os.path.exists(build_example())
