"""CPU checks of the boundary: libowl.so loads and exports every symbol include/owl.h declares (no compute
calls without a GPU), the binding fails loudly without a device, and the product never reaches the oracle."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_dsn_zhaoxcqzj24_b200")


def _declared():
    src = open(os.path.join(ROOT, "include", "owl.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(owl_[a-z0-9_]+)\s*\(", src)))


def test_every_declared_symbol_is_exported():
    lib = ctypes.CDLL(os.path.join(PKG, "libowl.so"))
    names = _declared()
    assert len(names) >= 20, names
    for n in names:
        assert hasattr(lib, n), f"libowl.so does not export {n}"
    from paper_conf_dsn_zhaoxcqzj24_b200 import _lib
    assert set(_lib.SIGNATURES) == set(names), set(names) ^ set(_lib.SIGNATURES)


def test_library_is_sm100a():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", os.path.join(PKG, "libowl.so")],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out, out


def test_no_device_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_dsn_zhaoxcqzj24_b200 import api
    with pytest.raises(api.OwlError, match="OWL_ERR_CUDA"):
        api.Context(0)
    from paper_conf_dsn_zhaoxcqzj24_b200 import _lib
    L = _lib.load()
    assert L.owl_version().decode().startswith("owl-b200")
    assert L.owl_ctx_destroy(None) == 0
    assert L.owl_build_adcfg(None, None, 0, None) == 1  # OWL_ERR_INVALID_ARG
    assert b"NULL" in L.owl_last_error()


def test_product_never_imports_the_oracle():
    for d, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                txt = open(os.path.join(d, f)).read()
                assert not re.search(r"^\s*(import|from)\s+(oracle|tracegen)\b", txt, flags=re.M), f
                assert not re.search(r"#include\s+[<\"][^>\"]*(oracle|owl_gen)", txt), f
                assert "liboracle" not in txt and "libowlgen" not in txt, f
    head = open(os.path.join(ROOT, "oracle", "owl_oracle.cpp")).read(600)
    assert "TEST INFRASTRUCTURE ONLY" in head


def test_oracle_shares_no_header_with_product():
    src = open(os.path.join(ROOT, "oracle", "owl_oracle.cpp")).read()
    includes = re.findall(r'#include\s+[<"]([^>"]+)[>"]', src)
    assert all("/" not in i and not i.startswith("owl") for i in includes), includes


def test_binding_layouts_match_header(tmp_path):
    """The ctypes structs and numpy row dtypes of the binding have the header's sizes and field offsets."""
    import subprocess
    from paper_conf_dsn_zhaoxcqzj24_b200 import _lib, api
    c = tmp_path / "sz.c"
    c.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "owl.h"\nint main(void){printf("%zu %zu %zu %zu %zu '
                 '%zu %zu %zu\\n", sizeof(owl_config), offsetof(owl_config, hcf_reading), sizeof(owl_segment), '
                 'sizeof(owl_adcfg_info), sizeof(owl_diff), sizeof(owl_leak), sizeof(owl_ks_row), '
                 'offsetof(owl_ks_row, D));return 0;}\n')
    exe = tmp_path / "sz"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), str(c), "-o", str(exe)], check=True)
    got = [int(v) for v in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split()]
    assert got == [ctypes.sizeof(_lib.OwlConfig), _lib.OwlConfig.hcf_reading.offset, ctypes.sizeof(_lib.OwlSegment),
                   ctypes.sizeof(_lib.OwlAdcfgInfo), api.DIFF_DTYPE.itemsize, api.LEAK_DTYPE.itemsize,
                   api.KS_DTYPE.itemsize, api.KS_DTYPE.fields["D"][1]]
