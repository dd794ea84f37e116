"""The oracle and the CUDA path share no code: neither imports the other, and
the product never loads anything under oracle/ (DESIGN.md §Oracle)."""
import ast
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = "paper_conf_ppopp_prajapatirradg17_b200"


def _imports(path):
    tree = ast.parse(open(path).read())
    names = set()
    for n in ast.walk(tree):
        if isinstance(n, ast.Import):
            names |= {a.name.split(".")[0] for a in n.names}
        elif isinstance(n, ast.ImportFrom) and n.module:
            names.add(n.module.split(".")[0])
    return names


def _files(d, exts):
    for root, _, fs in os.walk(os.path.join(ROOT, d)):
        for f in fs:
            if f.endswith(exts):
                yield os.path.join(root, f)


def test_product_does_not_import_oracle():
    for f in _files(PKG, (".py",)):
        assert "oracle" not in _imports(f), f
    for f in _files(PKG, (".cu", ".cpp", ".h")):
        src = open(f).read()
        assert "oracle/" not in src and "stencil_oracle" not in src, f


def test_oracle_does_not_import_product():
    for f in _files("oracle", (".py",)):
        assert PKG not in _imports(f), f
    src = open(os.path.join(ROOT, "oracle", "stencil_oracle.c")).read()
    includes = [l for l in src.splitlines() if l.startswith("#include")]
    assert all("<" in l for l in includes), includes          # system headers only


def test_synth_has_no_method_arithmetic():
    imps = _imports(os.path.join(ROOT, "synth", "__init__.py"))
    assert imps <= {"__future__", "numpy", "torch"}
