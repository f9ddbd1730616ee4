"""CPU-side checks of the C ABI: the library builds for sm_100a, loads, and exports every
symbol include/harmonia.h declares; the product package does not import the oracle."""
import os
import re
import subprocess

import pytest

from conftest import ROOT


def _declared():
    src = open(os.path.join(ROOT, "include", "harmonia.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(harmonia_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    import paper_conf_ppopp_yanlpz19_b200 as hm

    L = hm.lib()
    names = _declared()
    assert len(names) >= 18
    for n in names:
        assert hasattr(L, n), n
    assert L.harmonia_abi_version() == 2


def test_sass_is_sm100a_and_uses_bulk_copy():
    from paper_conf_ppopp_yanlpz19_b200 import _build

    out = subprocess.run(["cuobjdump", "-lelf", _build.LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", _build.LIB], capture_output=True, text=True).stdout
    assert "UBLKCP" in sass  # TMA bulk copy staging of the PS / top levels
    assert "VOTE" in sass    # ballot-based in-node rank


def test_status_strings_and_psa_bits():
    import paper_conf_ppopp_yanlpz19_b200 as hm

    L = hm.lib()
    for s in range(8):
        assert L.harmonia_status_string(s)
    assert hm.psa_bits_auto(1 << 23) == 19  # Eq 2
    assert hm.psa_bits_auto(1 << 16) == 12
    assert hm.psa_bits_auto(10) == 0


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ppopp_yanlpz19_b200")
    for dp, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cc")):
                s = open(os.path.join(dp, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", s, re.M), f
                assert "oracle.h" not in s and "liboracle" not in s, f


def test_null_and_invalid_args_without_gpu():
    """Argument validation happens before any CUDA call."""
    import ctypes as C

    import paper_conf_ppopp_yanlpz19_b200 as hm

    L = hm.lib()
    assert L.harmonia_search_batch(None, None, 5, None, None, 0, None, None) == 1
    assert L.harmonia_get_info(None, None) == 1
    bo = hm.BuildOpts(3, 1.0, 0, 0)  # fanout not a power of two
    h = C.c_void_p()
    assert L.harmonia_build(None, None, 0, C.byref(bo), None, C.byref(h)) == 1


def test_struct_layouts_match_the_header(tmp_path):
    """The ctypes mirrors of the ABI structs have the header's size and field offsets (compiled
    with gcc against include/harmonia.h; no GPU)."""
    import ctypes as C

    import paper_conf_ppopp_yanlpz19_b200 as hm

    structs = {"harmonia_build_opts": hm.BuildOpts, "harmonia_query_opts": hm.QueryOpts,
               "harmonia_plan": hm.PlanInfo, "harmonia_info": hm.Info}
    lines = ['#include <stdio.h>', '#include "harmonia.h"', "int main(void) {"]
    for cname, py in structs.items():
        lines.append(f'  printf("{cname} size %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'  printf("{cname} {f} %zu\\n", offsetof({cname}, {f}));')
    lines += ["  return 0;", "}"]
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    got = {}
    for line in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.splitlines():
        s, f, v = line.split()
        got[(s, f)] = int(v)
    for cname, py in structs.items():
        assert got[(cname, "size")] == C.sizeof(py), cname
        for f, _ in py._fields_:
            assert got[(cname, f)] == getattr(py, f).offset, (cname, f)


def test_sass_uses_blackwell_memory_instructions():
    """The search kernel's 256-bit leaf-block loads, the TMA bulk stores of the PSA write-outs
    and the warp shuffles of the window rank are in the built library."""
    from paper_conf_ppopp_yanlpz19_b200 import _build

    sass = subprocess.run(["cuobjdump", "-sass", _build.LIB], capture_output=True, text=True).stdout
    assert "LDG.E.ENL2.256" in sass  # ld.global.nc.v4.u64 (sm_100a 256-bit load)
    assert "UBLKCP.G.S" in sass      # cp.async.bulk shared -> global (TMA store)
    assert "SHFL.IDX" in sass
