"""The C-ABI library builds, loads without a GPU and exports every symbol include/gmpsvm.h
declares; argument validation happens before any CUDA call (CPU, -m "not gpu")."""
import ctypes as ct
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def gm():
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as m

    return m


def _declared():
    src = open(os.path.join(ROOT, "include", "gmpsvm.h")).read()
    return sorted(set(re.findall(r"GMPSVM_API\s+[\w\s\*]*?\b(gmpsvm_\w+)\s*\(", src)))


def test_header_symbols_exported(gm):
    names = _declared()
    assert len(names) >= 20
    L = ct.CDLL(gm._lib.LIB_PATH)
    for n in names:
        assert hasattr(L, n), n
    assert gm.lib().gmpsvm_abi_version() == 1


def test_binding_covers_header(gm):
    assert set(_declared()) <= set(gm._lib._SIGS)


def test_struct_layouts_match_header(gm):
    # sizes of the ctypes mirrors == the C structs (offsets checked via sizeof)
    o = gm._lib.Options()
    gm.lib().gmpsvm_options_init(ct.byref(o))
    assert o.struct_size == ct.sizeof(gm._lib.Options)


def test_invalid_arguments_rejected_without_gpu(gm):
    X = np.zeros((4, 2), np.float32)
    y = np.array([0, 1, 0, 1], np.int32)
    for args in [(X, y, 1, 1.0, 0.5, 1e-3), (X, y, 2, -1.0, 0.5, 1e-3), (X, y, 2, 1.0, 0.0, 1e-3),
                 (X, y, 2, 1.0, 0.5, float("nan")), (X[:1], y[:1], 2, 1.0, 0.5, 1e-3)]:
        with pytest.raises(gm.GmpsvmError) as e:
            gm.train(*args)
        assert e.value.code == gm.EINVAL
    with pytest.raises(gm.GmpsvmError) as e:
        gm.train(X, y, 2, 1.0, 0.5, 1e-3, ws_size=3)
    assert e.value.code == gm.EINVAL


def test_deserialize_rejects_garbage(gm):
    with pytest.raises(gm.GmpsvmError) as e:
        gm.Model.deserialize(b"not a model at all")
    assert e.value.code == gm.EFORMAT


def test_product_package_does_not_import_oracle():
    import ast

    pkg = os.path.join(ROOT, "paper_conf_icde_wenshcc19_b200")
    for f in os.listdir(pkg):
        if f.endswith(".py"):
            tree = ast.parse(open(os.path.join(pkg, f)).read())
            for node in ast.walk(tree):
                if isinstance(node, (ast.Import, ast.ImportFrom)):
                    mods = [a.name for a in node.names] if isinstance(node, ast.Import) else [node.module or ""]
                    assert not any(m.split(".")[0] == "oracle" for m in mods), f
    for f in os.listdir(os.path.join(pkg, "csrc")):
        for line in open(os.path.join(pkg, "csrc", f)):
            if line.lstrip().startswith("#include"):
                assert "oracle" not in line, (f, line)
