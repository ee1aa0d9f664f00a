"""CPU-only checks of the C-ABI boundary: libsf.so builds for sm_100a, loads,
and exports every function include/sf.h declares; the Python binding mirrors
them; the product path has no CPU fallback (no device -> SF_ERR_CUDA)."""
import os
import re
import subprocess

import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import build, sf

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared():
    txt = open(os.path.join(ROOT, "include", "sf.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(sf_[a-z_0-9]+)\s*\(", txt)))


@pytest.fixture(scope="module")
def libpath():
    return build.build()


def test_header_declares_north_star_entry_points():
    names = declared()
    for n in ["sf_level_create", "sf_apply_bc", "sf_apply_op", "sf_smooth_gsrb", "sf_residual",
              "sf_restrict", "sf_interpolate", "sf_vcycle"]:
        assert n in names


def test_library_exports_every_declared_symbol(libpath):
    out = subprocess.run(["nm", "-D", "--defined-only", libpath], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r" T (sf_[a-z_0-9]+)$", out, flags=re.M))
    missing = [n for n in declared() if n not in exported]
    assert not missing, missing


def test_binding_mirrors_header(libpath):
    L = sf.lib()
    for n in declared():
        getattr(L, n)
    assert set(declared()) == set(sf.EXPORTS)


def test_sm100a_sass_present(libpath):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", libpath],
                         capture_output=True, text=True, check=True).stdout
    assert "sm_100a" in out


def test_no_cpu_fallback_without_device(libpath):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(sf.SfError) as e:
        sf.sf_level_create(16, 16, 16, 1 / 16)
    assert e.value.status == sf.SF_ERR_CUDA


def test_argument_errors_are_synchronous(libpath):
    with pytest.raises(sf.SfError) as e:
        sf.sf_level_bytes_needed(1, 16, 16)
    assert e.value.status == sf.SF_ERR_SHAPE
    c = sf.Comm.local(3)
    with pytest.raises(sf.SfError) as e:
        sf.sf_level_bytes_needed(16, 16, 16, c.h)   # 16 % 3 != 0
    assert e.value.status == sf.SF_ERR_SHAPE
    assert sf.sf_level_bytes_needed(16, 16, 18, c.h) > 0
    c.close()


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_zhangdmwbf17_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert not re.search(r"(^\s*(from|import)\s+oracle)|liboracle|\bor_[a-z_]+\(", txt,
                                     flags=re.M), f
