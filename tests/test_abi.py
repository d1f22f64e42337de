"""CPU-only checks of the boundary: the C-ABI library builds for sm_100a, loads,
exports every symbol include/*.h declares, and agrees with the oracle's layout
(each side defines its constants independently)."""
import ctypes
import os
import re
import subprocess

import oracle
import paper_conf_ppopp_geladog19_b200 as ga

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = set()
    for h in ("ga.h", "ga_bench.h", "ga_rcu.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        names |= set(re.findall(r"^\s*(?:ga_status|const char\*)\s+(ga_\w+)\s*\(", src, re.M))
    return names


def test_library_exports_every_declared_symbol():
    L = ga.lib()
    declared = _declared()
    assert len(declared) >= 20
    assert declared == set(ga.EXPORTED)
    for name in declared:
        assert hasattr(L, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", ga._build.LIB], capture_output=True, text=True).stdout
    for name in declared:
        assert re.search(rf"\bT {name}\b", out), name


def test_library_is_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", ga._build.LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings_and_layout():
    assert ga.ga_status_str(0) == "ok"
    assert "invalid" in ga.ga_status_str(1)
    lay = ga.ga_layout()
    b = oracle.BUILD
    assert lay["page"] == b["page"] and lay["chunk_pages"] == b["chunk_pages"]
    assert lay["min_class"] == b["min_class"] and lay["bin_max"] == b["bin_max"]
    assert lay["n_classes"] == 8 and lay["bitmap_bits"] == 256


def test_invalid_arguments_rejected_without_gpu():
    L = ga.lib()
    h = ctypes.c_void_p()
    # fewer than one chunk -> GA_EINVAL before touching the device
    assert L.ga_heap_create(0, None, None, 1000, 0, ctypes.byref(h)) == 1
    assert L.ga_heap_create(0, None, None, 1 << 20, 0, None) == 1
    assert L.ga_heap_destroy(None) == 1
    assert L.ga_stats(None, None, None) == 1


def test_oracle_and_cuda_path_share_no_code():
    """Neither side imports or includes the other."""
    csrc = os.path.join(ROOT, "paper_conf_ppopp_geladog19_b200")
    for dirpath, _, files in os.walk(csrc):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in re.sub(r"#.*|//.*", "", txt).lower() or f == "__init__.py" and \
                    "import oracle" not in txt, f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert "paper_conf_ppopp_geladog19_b200" not in txt.replace(
                "(paper_conf_ppopp_geladog19_b200/csrc)", "").replace(
                "(``paper_conf_ppopp_geladog19_b200``)", ""), f
            assert "#include \"ga" not in txt
