"""The product path is the native library only: no product module imports the oracle, the oracle
imports nothing of the product, bench.py touches the oracle only inside its baseline legs, and the
binding fails loudly when libaegkv.so is missing instead of falling back to anything."""
import ast
import os

import pytest

import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sosp_xiang0qyzyzl0025_b200")


def _is_oracle(m):
    return m == "oracle" or m.startswith("oracle.")


def _imports(tree):
    for node in ast.walk(tree):
        if isinstance(node, ast.Import):
            for a in node.names:
                yield a.name
        elif isinstance(node, ast.ImportFrom) and node.module:
            yield node.module


def _py_files(*dirs):
    for d in dirs:
        for dp, _, fs in os.walk(d):
            for f in fs:
                if f.endswith(".py"):
                    yield os.path.join(dp, f)


def _tree(p):
    return ast.parse(open(p).read(), p)


def test_product_does_not_import_the_oracle():
    bad = [(os.path.relpath(p, ROOT), m) for p in _py_files(PKG, os.path.join(ROOT, "aeg_inputs"))
           for m in _imports(_tree(p)) if _is_oracle(m)]
    assert not bad, bad
    # the native sources include nothing from oracle/
    for dp, _, fs in os.walk(os.path.join(PKG, "csrc")):
        for f in fs:
            for line in open(os.path.join(dp, f), errors="replace"):
                assert not (line.lstrip().startswith("#include") and "oracle" in line), (f, line)


def test_oracle_does_not_import_the_product():
    bad = [(os.path.relpath(p, ROOT), m) for p in _py_files(os.path.join(ROOT, "oracle"))
           for m in _imports(_tree(p)) if m.startswith("paper_conf") or m.startswith("aeg_inputs")]
    assert not bad, bad


def test_bench_uses_the_oracle_only_in_its_baseline_legs():
    tree = _tree(os.path.join(ROOT, "bench.py"))
    assert not [n for n in tree.body if isinstance(n, (ast.Import, ast.ImportFrom))
                and any(_is_oracle(m) for m in _imports(n))], "module-level oracle import"
    users = {fn.name for fn in tree.body if isinstance(fn, (ast.FunctionDef, ast.ClassDef))
             and any(_is_oracle(m) for m in _imports(fn))}
    assert users <= {"OracleSample"}, users


def test_binding_fails_loudly_without_the_library(monkeypatch, tmp_path):
    monkeypatch.setattr(aeg, "_L", None)
    monkeypatch.setattr(aeg, "LIB_PATH", str(tmp_path / "libaegkv.so"))
    with pytest.raises(aeg.AegError, match="missing"):
        aeg.lib()
    with pytest.raises(aeg.AegError, match="missing"):
        aeg.Context(0)
