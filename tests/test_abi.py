"""CPU-side checks of the boundary: the C-ABI library builds for sm_100a, loads, and exports
every symbol include/tid.h declares; the header and the binding agree.  No compute calls."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "tid.h")


def _declared():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:tid_status|const char\*)\s+(tid_\w+)\s*\(", src, re.M)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icpp_wangzll21_b200 import build
    build.build()
    import paper_conf_icpp_wangzll21_b200 as tid
    return tid.load_library()


def test_header_declares_boundary():
    names = _declared()
    for need in ("tid_index_create", "tid_add_references", "tid_verify", "tid_search", "tid_index_destroy",
                 "tid_last_error"):
        assert need in names


def test_library_exports_every_declared_symbol(lib):
    out = subprocess.check_output(["nm", "-D", "--defined-only", lib._name]).decode()
    exported = set(re.findall(r" T (tid_\w+)", out))
    missing = [n for n in _declared() if n not in exported]
    assert not missing, f"declared in tid.h but not exported: {missing}"
    import paper_conf_icpp_wangzll21_b200 as tid
    assert sorted(tid.EXPORTS) == _declared()


def test_library_is_sm100a_native(lib):
    sass = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "-sass", lib._name]).decode()
    assert "sm_100a" in subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "-lelf", lib._name]).decode()
    assert "UTCIMMA" in sass, "tcgen05.mma kind::i8 missing from SASS"
    assert "LDTM" in sass, "tcgen05.ld missing from SASS"
    assert "UTMALDG" in sass, "TMA tensor load missing from SASS"
    assert not re.search(r"\s(HMMA|IMMA)\.", sass), "legacy mma.sync path present"


def test_errors_without_gpu(lib):
    """No GPU here: create must fail loudly (never fall back to the CPU)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import paper_conf_icpp_wangzll21_b200 as tid
    with pytest.raises(tid.TidError):
        tid.Index(ref_kp=256)
    assert lib.tid_last_error() != b""


def test_config_struct_matches_header():
    import paper_conf_icpp_wangzll21_b200 as tid
    src = open(HEADER).read()
    body = re.search(r"typedef struct \{(.*?)\} tid_config;", src, re.S).group(1)
    fields = re.findall(r"^\s*(?:const\s+)?\w+\*?\s+\*?(\w+)(?:,\s*(\w+))?;", body, re.M)
    names = [x for f in fields for x in f if x]
    assert names == [f for f, _ in tid.Config._fields_]


def test_struct_sizes_match_the_c_compiler(tmp_path):
    """Every struct the binding mirrors has the size and field offsets gcc gives the header's."""
    import paper_conf_icpp_wangzll21_b200 as tid
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    structs = {"tid_config": tid.Config, "tid_info": tid.Info, "tid_stats": tid.Stats, "tid_tuning": tid.Tuning,
               "tid_geom_params": tid.GeomParams}
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "tid.h"', "int main(void) {"]
    for cname, py in structs.items():
        lines.append(f'  printf("{cname} %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'  printf("{cname}.{f} %zu\\n", offsetof({cname}, {f}));')
    lines.append("  return 0;\n}")
    src = tmp_path / "sizes.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "sizes"
    subprocess.check_call(["gcc", "-I", os.path.join(root, "include"), str(src), "-o", str(exe)])
    got = dict(l.split() for l in subprocess.check_output([str(exe)], text=True).splitlines())
    for cname, py in structs.items():
        assert int(got[cname]) == ctypes.sizeof(py), cname
        for f, _ in py._fields_:
            assert int(got[f"{cname}.{f}"]) == getattr(py, f).offset, (cname, f)


def test_plain_c_example_compiles_and_links(tmp_path):
    """include/tid.h is valid C and libtid.so links from a plain C program (examples/search_example.c;
    running it needs a GPU)."""
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    lib_dir = os.path.join(root, "paper_conf_icpp_wangzll21_b200")
    out = tmp_path / "search_example"
    subprocess.check_call(["gcc", "-O2", "-Wall", "-Werror", "-I", os.path.join(root, "include"),
                           os.path.join(root, "examples", "search_example.c"), "-L", lib_dir, "-ltid",
                           f"-Wl,-rpath,{lib_dir}", "-o", str(out)])
    assert out.exists()


def test_binding_checks_output_buffers():
    """Caller-supplied outputs are checked, never converted: a wrong dtype / shape, a
    non-contiguous or read-only array, or a CUDA tensor on another device raises before any
    library call (an int32 ids buffer would otherwise be overrun by the int64 writes)."""
    import numpy as np
    import pytest
    import torch
    from paper_conf_icpp_wangzll21_b200 import _out_ptr, _ptr
    ok = np.empty((3, 5), np.int64)
    assert _out_ptr(ok, (3, 5), np.int64, 0, "ids") == ok.ctypes.data
    with pytest.raises(TypeError):
        _out_ptr(np.empty((3, 5), np.int32), (3, 5), np.int64, 0, "ids")
    with pytest.raises(TypeError):
        _out_ptr(np.empty((3, 4), np.int64), (3, 5), np.int64, 0, "ids")
    with pytest.raises(ValueError):
        _out_ptr(np.empty((5, 3), np.int64).T, (3, 5), np.int64, 0, "ids")
    ro = np.empty((3, 5), np.int64)
    ro.flags.writeable = False
    with pytest.raises(ValueError):
        _out_ptr(ro, (3, 5), np.int64, 0, "ids")
    with pytest.raises(TypeError):
        _out_ptr(torch.empty((3, 5), dtype=torch.int32), (3, 5), np.int64, 0, "ids")
    t = torch.empty((3, 5), dtype=torch.int64)
    assert _out_ptr(t, (3, 5), np.int64, 0, "ids") == t.data_ptr()
    with pytest.raises(TypeError):
        _out_ptr([0] * 15, (15,), np.int64, 0, "ids")
    # inputs: torch tensors must already have the right dtype (no silent reinterpretation)
    with pytest.raises(TypeError):
        _ptr(torch.zeros((2, 3, 128), dtype=torch.int32), np.uint8)
    p, keep = _ptr(np.zeros((2, 3, 128), np.int64), np.uint8)  # numpy inputs are converted
    assert keep.dtype == np.uint8
