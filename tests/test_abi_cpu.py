"""C-ABI contract checks that need no GPU: the library loads and exports every symbol include/*.h declares, and the
host-side error paths answer without touching a device."""
import ctypes
import glob
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        src = open(h).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names |= set(re.findall(r"\b(starsim_[a-z_]+)\s*\(", src))
    return sorted(names)


@pytest.fixture(scope="module")
def lib():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_ipps_lizzh12_b200 import starsim
    return starsim.lib()


def test_header_declares_the_boundary():
    names = declared_functions()
    for want in ["starsim_create", "starsim_destroy", "starsim_last_error", "starsim_render", "starsim_render_band",
                 "starsim_render_gray", "starsim_render_atomic", "starsim_upload_aos", "starsim_quantize",
                 "starsim_get_bins", "starsim_profile", "starsim_kernel_times", "starsim_set_psf",
                 "starsim_set_tile_kernel", "starsim_set_binning", "starsim_set_roi",
                 "starsim_render_band_to", "starsim_render_lut"]:
        assert want in names


def test_library_exports_every_declared_symbol(lib):
    for name in declared_functions():
        assert hasattr(lib, name), name


def test_library_is_sm100a_only():
    import subprocess
    from paper_conf_ipps_lizzh12_b200 import starsim
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", starsim.LIB_PATH],
                         capture_output=True, text=True).stdout
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


def test_null_ctx_is_einval(lib):
    vp = ctypes.c_void_p
    assert lib.starsim_render(None, None, None, None, 0, 16, 16, 1.0, 5, 1.0, vp(1), None) == -1
    assert lib.starsim_render_band(None, None, None, None, 0, 16, 16, 0, 16, 1.0, 5, 1.0, vp(1), None) == -1
    assert lib.starsim_render_atomic(None, None, None, None, 0, 16, 16, 1.0, 5, 1.0, vp(1), None) == -1
    assert lib.starsim_quantize(None, None, 0, 8, None, None) == -1
    assert lib.starsim_upload_aos(None, None, 0, None, None, None, None) == -1
    for fn in (lib.starsim_set_psf, lib.starsim_set_roi, lib.starsim_set_tile_kernel, lib.starsim_set_binning):
        fn.argtypes = [ctypes.c_void_p, ctypes.c_int32]
        assert fn(None, 0) == -1
    assert lib.starsim_profile(None, 1) == -1
    lib.starsim_destroy(None)   # NULL-safe


def test_create_without_gpu_reports_enodev(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    h = ctypes.c_void_p()
    rc = lib.starsim_create(ctypes.byref(h), 0)
    assert rc == -4 and not h.value
    assert lib.starsim_last_error(None)
