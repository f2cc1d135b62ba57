"""CPU checks of the boundary: the C-ABI library loads and exports every symbol include/sepo.h
declares; the binding names match; the budget arithmetic is consistent. No compute calls."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "sepo.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sepo_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    L = sepo.lib()
    decl = declared_symbols()
    assert len(decl) >= 14
    for name in decl:
        assert hasattr(L, name), name
    assert sorted(sepo.EXPORTS) == decl


def test_version_and_budget_arithmetic():
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    assert b"sm_100a" in sepo.lib().sepo_version()
    b1 = sepo.budget_for(1 << 20, 65536, 100)
    b2 = sepo.budget_for(1 << 20, 65536, 101)
    assert b2 - b1 == 65536 + 10
    assert sepo.budget_for(1 << 21, 65536, 100) - b1 == 4 << 20


def test_no_cpu_fallback_without_gpu():
    import torch
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(RuntimeError):
        sepo.Table(1 << 26, 1 << 16, 65536)


def test_product_does_not_import_oracle_or_gen():
    pkg = os.path.join(ROOT, "paper_conf_ipps_mokhtaris17_b200")
    for dp, _, fns in os.walk(pkg):
        for f in fns:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                s = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", s).lower() or f.endswith(".md"), f
                assert "import gen" not in s and "gen_common" not in s, f
