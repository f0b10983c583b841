"""CPU checks of the C-ABI boundary: libgsh.so loads, exports every symbol include/gsh.h
declares, reports argument errors before any launch, and the Python binding mirrors the
header's structs.  No compute calls (no GPU here)."""
import ctypes
import os
import re
import subprocess
import tempfile

import pytest

import paper_conf_icde_caic24_b200 as gsh
from paper_conf_icde_caic24_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    txt = open(_lib.HEADER_PATH).read()
    return sorted(set(re.findall(r"GSH_API\s+[\w\s\*]*?\b(gsh_\w+)\s*\(", txt)))


def test_library_exports_every_header_symbol():
    lib = _lib.load()
    names = header_functions()
    assert len(names) >= 15
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(_lib.EXPORTED) == names


def test_compiled_for_sm100a():
    lib = _lib.load()
    assert lib.gsh_compiled_arch() == 100
    assert lib.gsh_version() >= 1
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_status_strings_and_struct_sizes():
    lib = _lib.load()
    assert lib.gsh_status_string(0) == b"GSH_OK"
    assert lib.gsh_status_string(1) == b"GSH_ERR_INVALID"
    # the ctypes mirrors match the C compiler's layout of include/gsh.h field by field
    src = "#include <stdio.h>\n#include <stddef.h>\n#include \"gsh.h\"\nint main(void){\n"
    structs = (("gsh_config", _lib.GshConfig), ("gsh_result", _lib.GshResult),
               ("gsh_shard_params", _lib.GshShardParams), ("gsh_comm", _lib.GshComm),
               ("gsh_sharded_result", _lib.GshShardedResult))
    for cname, cls in structs:
        src += f'printf("%zu\\n", sizeof({cname}));\n'
        for f, _ in cls._fields_:
            src += f'printf("%zu\\n", offsetof({cname}, {f}));\n'
    src += "return 0;}\n"
    with tempfile.TemporaryDirectory() as d:
        c, exe = os.path.join(d, "sz.c"), os.path.join(d, "sz")
        open(c, "w").write(src)
        subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        got = [int(x) for x in subprocess.check_output([exe]).split()]
    want = []
    for _, cls in structs:
        want.append(ctypes.sizeof(cls))
        want += [getattr(cls, f).offset for f, _ in cls._fields_]
    assert got == want
    cfg = _lib.default_config()
    assert list(cfg.pass_bits) == [-1, -1] and cfg.capacity == 0


def test_workspace_sizing_is_monotone_and_rejects_bad_config():
    a = gsh.workspace_bytes(1 << 10, 1 << 10)
    b = gsh.workspace_bytes(1 << 20, 1 << 20)
    assert 0 < a < b
    # ~20 B per tuple plus tables
    assert b >= 20 * (2 << 20)
    with pytest.raises(ValueError):
        gsh.workspace_bytes(100, 100, gsh.make_config(pass_bits=(9, 1)))
    with pytest.raises(ValueError):
        gsh.workspace_bytes(100, 100, gsh.make_config(force_all_heavy=True, force_all_normal=True))
    with pytest.raises(ValueError):
        gsh.workspace_bytes(100, 100, gsh.make_config(prepass_bits=9))
    with pytest.raises(ValueError):   # pre-pass bits stack on the routing bits (<= 16 in total)
        gsh.workspace_bytes(100, 100, gsh.make_config(prepass_bits=2, route_bits=15))


def test_prepass_workspace_adds_split_copies():
    """The pre-partition pass (gsh_config.prepass_bits) needs the sub-problem workspace plus SoA
    copies of both sides (16 B per tuple); auto mode adds it only beyond 2^28 tuples per side."""
    n = 1 << 20
    plain = gsh.workspace_bytes(n, n, gsh.make_config(prepass_bits=-1))
    assert gsh.workspace_bytes(n, n) == plain
    forced = gsh.workspace_bytes(n, n, gsh.make_config(prepass_bits=2))
    assert forced >= plain + 16 * n
    big = 1 << 29
    assert gsh.workspace_bytes(big, big) >= gsh.workspace_bytes(big, big, gsh.make_config(prepass_bits=-1)) + 16 * big


def test_argument_errors_before_any_launch():
    lib = _lib.load()
    res = _lib.GshResult()
    R = _lib.GshRelation(None, None, 10)  # NULL with n > 0
    S = _lib.GshRelation(None, None, 0)
    st = lib.gsh_join(ctypes.byref(R), ctypes.byref(S), 0, None, None, 0, None, None, ctypes.byref(res))
    assert st == _lib.GSH_ERR_INVALID
    assert b"invalid relation" in lib.gsh_last_error()
    R = _lib.GshRelation(None, None, 0)
    st = lib.gsh_join(ctypes.byref(R), ctypes.byref(S), 1, None, None, 0, None, None, ctypes.byref(res))
    assert st == _lib.GSH_ERR_INVALID  # MATERIALIZE without output
    st = lib.gsh_join(ctypes.byref(R), ctypes.byref(S), 0, None, None, 0, None, None, None)
    assert st == _lib.GSH_ERR_INVALID  # res NULL
    R = _lib.GshRelation(None, None, 1 << 32)
    st = lib.gsh_join(ctypes.byref(R), ctypes.byref(S), 0, None, None, 0, None, None, ctypes.byref(res))
    assert st == _lib.GSH_ERR_INVALID  # n >= 2^32


def test_gbase_argument_errors_before_any_launch():
    lib = _lib.load()
    res = _lib.GshResult()
    R = _lib.GshRelation(None, None, 10)
    S = _lib.GshRelation(None, None, 0)
    assert lib.gsh_join_gbase(ctypes.byref(R), ctypes.byref(S), 0, None, None, 0, None, None,
                              ctypes.byref(res)) == _lib.GSH_ERR_INVALID
    R = _lib.GshRelation(None, None, 0)
    assert lib.gsh_join_gbase(ctypes.byref(R), ctypes.byref(S), 1, None, None, 0, None, None,
                              ctypes.byref(res)) == _lib.GSH_ERR_INVALID   # MATERIALIZE without output
    big = _lib.GshRelation(1, 1, (1 << 28) + 1)   # never dereferenced: refused first
    assert lib.gsh_join_gbase(ctypes.byref(big), ctypes.byref(S), 0, None, None, 0, None, None,
                              ctypes.byref(res)) == _lib.GSH_ERR_INVALID
    assert b"2^28" in lib.gsh_last_error()


def test_gbase_workspace_sizing():
    # bucket pools: larger than GSH's workspace, growing with n; refused beyond 2^28 per side
    lib = _lib.load()
    a, b = gsh.gbase_workspace_bytes(1 << 20, 1 << 20), gsh.gbase_workspace_bytes(1 << 27, 1 << 27)
    assert 0 < a < b and b > gsh.workspace_bytes(1 << 27, 1 << 27)
    assert lib.gsh_gbase_workspace_bytes((1 << 28) + 1, 10, None) == 0
    with pytest.raises(ValueError):
        gsh.gbase_workspace_bytes((1 << 28) + 1, 10)


def test_hybrid_config_validation():
    lib = _lib.load()
    assert gsh.workspace_bytes(1 << 20, 1 << 20, gsh.make_config(hybrid=True)) > \
        gsh.workspace_bytes(1 << 20, 1 << 20)
    cfg = gsh.make_config()
    cfg.hybrid = 2
    assert lib.gsh_workspace_bytes(1000, 1000, ctypes.byref(cfg)) == 0
    cfg = gsh.make_config(hybrid=True, hybrid_share=257)
    assert lib.gsh_workspace_bytes(1000, 1000, ctypes.byref(cfg)) == 0


def test_product_path_refuses_cpu_tensors():
    import torch
    k = torch.zeros(4, dtype=torch.int32)
    with pytest.raises(ValueError, match="CUDA"):
        gsh.join(k, k, k, k)


def test_product_does_not_import_oracle():
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    pkg = os.path.join(root, "paper_conf_icde_caic24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "join_oracle" not in txt, f
