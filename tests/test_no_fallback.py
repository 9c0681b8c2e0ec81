"""The product path has no CPU fallback (task rule; include/idg.h): a missing library raises instead of
computing anything, and nothing in the package imports or executes the oracle (test infrastructure)."""
import ast
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_veenboerpr17_b200")


def test_missing_library_raises():
    code = ("import paper_conf_ipps_veenboerpr17_b200.idg as b\n"
            "b._LIB_PATH = '/nonexistent/libidg_b200.so'; b._lib = None\n"
            "try:\n    b.lib()\nexcept ImportError as e:\n    print('RAISED', e)\n")
    out = subprocess.run([sys.executable, "-c", code], cwd=ROOT, capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stderr
    assert "RAISED" in out.stdout and "no fallback" in out.stdout


def _imports(path):
    tree = ast.parse(open(path).read(), filename=path)
    for node in ast.walk(tree):
        if isinstance(node, ast.Import):
            yield from (a.name for a in node.names)
        elif isinstance(node, ast.ImportFrom):
            yield node.module or ""


def test_package_never_imports_the_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith(".py"):
                mods = list(_imports(os.path.join(dirpath, f)))
                assert not any(m == "oracle" or m.startswith("oracle.") for m in mods), (f, mods)
    for f in os.listdir(os.path.join(PKG, "csrc")):
        src = open(os.path.join(PKG, "csrc", f), errors="replace").read()
        assert "idg_oracle" not in src and "oracle/" not in src, f
