"""The C-ABI library builds, loads without a GPU, and exports every symbol include/vf.h declares."""
import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_asplos_zhangar21_b200 import vf

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "vf.h")


def declared():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = set(re.findall(r"\b(vf_[a-z0-9_]+)\s*\(", src))
    names.discard("vf_strip")  # static inline helper, not exported
    return names


def test_header_declares_expected_entry_points():
    names = declared()
    for must in ("vf_alloc_typed", "vf_alloc_typed_batch", "vf_alloc_cuda", "vf_dispatch_cuda",
                 "vf_dispatch_sharedoa", "vf_dispatch_coal", "vf_dispatch_typeptr", "vf_range_table",
                 "vf_resolve", "vf_verify_types"):
        assert must in names


def test_library_exports_every_declared_symbol():
    L = vf.lib()
    missing = [n for n in sorted(declared()) if not hasattr(L, n)]
    assert not missing, missing
    assert set(vf.SYMBOLS) == declared()


def test_exported_symbols_are_c_linkage():
    out = subprocess.run(["nm", "-D", "--defined-only", vf.SO], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\s[TW]\s(vf_\w+)$", out, flags=re.M))
    assert declared() <= exported


def test_status_strings_and_app_info():
    L = vf.lib()
    assert L.vf_status_str(0) == b"VF_OK"
    assert L.vf_status_str(4) == b"VF_ERR_TAG_BITS"
    nt, sizes, nm = vf.app_info(vf.APP_MICRO)
    assert nt == 32 and nm == 2 and set(sizes) == {16}
    nt, sizes, nm = vf.app_info(vf.APP_GOL)
    assert nt == 2 and sizes == [16, 16]
    with pytest.raises(vf.VFError):
        vf.app_info(99)


def test_tuning_validation():
    with pytest.raises(vf.VFError):
        vf.set_tuning("unroll", 3)
    with pytest.raises(vf.VFError):
        vf.set_tuning("nope", 1)
    vf.set_tuning("unroll", -1)
    vf.set_tuning("prefetch", -1)


def test_create_without_gpu_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    L = vf.lib()
    h = ctypes.c_void_p()
    st = L.vf_create(None, ctypes.byref(h))
    assert st != 0 and not h.value
    assert L.vf_dispatch(None, 0, 0, 0, None, 0, None, 0, None) == 1  # null ctx -> VF_ERR_INVALID


def test_product_path_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_asplos_zhangar21_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle.h" not in txt and "liboracle" not in txt, f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".cpp", ".h")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert not re.search(r"^\s*(from|import)\s+paper_conf", txt, flags=re.M), f
            assert not re.search(r'#include\s+[<"].*vf(_internal)?\.h', txt), f


def test_header_is_plain_c():
    """include/vf.h compiles as C (and as C++) with no CUDA headers: the boundary
    is plain pointers and sizes."""
    for lang, std in (("c", "-std=c11"), ("c++", "-std=c++17")):
        r = subprocess.run(["gcc", "-fsyntax-only", "-x", lang, std, "-Wall", "-Werror", HDR],
                           capture_output=True, text=True)
        assert r.returncode == 0, r.stderr


def test_arg_struct_layouts_match_header(tmp_path):
    """The ctypes mirrors of the method-argument structs have the C sizes and
    field offsets of include/vf.h (compiled here with gcc)."""
    import ctypes
    structs = {"vf_graph_en_bfs_args": vf.graph_en_bfs_args, "vf_graph_en_cc_args": vf.graph_en_cc_args,
               "vf_graph_en_pr_args": vf.graph_en_pr_args, "vf_edge_args": vf.edge_args,
               "vf_edge_resolver": vf.edge_resolver, "vf_graph_bfs_args": vf.graph_bfs_args,
               "vf_graph_cc_args": vf.graph_cc_args, "vf_graph_pr_args": vf.graph_pr_args,
               "vf_graph_bfs_bits_args": vf.graph_bfs_bits_args, "vf_collide_near_entry": vf.collide_near_entry}
    lines = ['#include <stdio.h>', '#include <stddef.h>', f'#include "{HDR}"', "int main(void) {"]
    for cname, py in structs.items():
        lines.append(f'  printf("{cname} %zu\\n", sizeof({cname}));')
        for fname, _ in py._fields_:
            lines.append(f'  printf("{cname}.{fname} %zu\\n", offsetof({cname}, {fname}));')
    lines.append("  return 0;\n}")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-std=c11", "-o", str(exe), str(src)], check=True)
    got = dict(l.split() for l in subprocess.run([str(exe)], capture_output=True, text=True,
                                                  check=True).stdout.splitlines())
    for cname, py in structs.items():
        assert int(got[cname]) == ctypes.sizeof(py), cname
        for fname, _ in py._fields_:
            assert int(got[f"{cname}.{fname}"]) == getattr(py, fname).offset, f"{cname}.{fname}"


def test_graph_en_app_info():
    nt, sizes, nm = vf.app_info(vf.APP_GRAPH_EN)
    assert nt == 4 and nm == 4 and sizes == [16, 16, 16, 16]
    nt, sizes, nm = vf.app_info(vf.APP_EDGE)
    assert nt == 2 and nm == 3 and sizes == [32, 32]
