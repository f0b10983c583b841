"""The committed golden file (SURVEY §8(c) P0 values from the survey author's independent script)
is reproduced, value by value, by scripts/make_golden.py: a plain-Python brute force that restates
fmix32 / fmix64 / pair_hash and the nested-loop join from their definitions and imports neither
oracle/ nor the CUDA package."""
import ast
import importlib.util
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCRIPT = os.path.join(ROOT, "scripts", "make_golden.py")


def _load():
    spec = importlib.util.spec_from_file_location("make_golden", SCRIPT)
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_script_is_independent_of_oracle_and_product():
    tree = ast.parse(open(SCRIPT).read())
    mods = {a.name.split(".")[0] for n in ast.walk(tree) if isinstance(n, ast.Import) for a in n.names}
    mods |= {n.module.split(".")[0] for n in ast.walk(tree) if isinstance(n, ast.ImportFrom) and n.module}
    assert mods <= {"json", "os", "sys"}, mods


def test_script_reproduces_committed_golden():
    m = _load()
    g = m.build()
    f = json.load(open(m.GOLDEN))
    for k in ("tiny", "all_equal", "fmix32", "pair_hash"):
        assert g[k] == f[k], k
