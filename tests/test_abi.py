"""Host-side checks of the C-ABI library (no GPU needed): it loads, exports every
symbol include/mars.h declares, and refuses to compute without a device (no
CPU fallback)."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_icpp_lancl21_b200 as mars

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "mars.h")


def _declared():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^MARS_API\s+[\w\s\*]+?\b(mars_\w+)\s*\(", src, re.M)))


def test_header_declares_the_boundary():
    names = _declared()
    for n in ("mars_graph_load", "mars_dgi_create", "mars_dgi_step", "mars_encode", "mars_free"):
        assert n in names
    assert len(names) >= 19


def test_library_exports_every_declared_symbol():
    L = mars.lib()
    for n in _declared():
        assert hasattr(L, n), n
    assert set(_declared()) == set(mars.SIGNATURES), "binding and header disagree"


def test_version_and_param_count():
    assert "sm_100a" in mars.version()
    assert mars.num_params(64, 256) == 64 * 256 + 3 * 256 * 256 + 3


def test_config_default():
    c = mars.config_default()
    assert (c.in_dim, c.hidden_dim, c.num_layers, c.world_size) == (64, 256, 3, 1)
    assert abs(c.lr - 1e-3) < 1e-9 and abs(c.beta2 - 0.999) < 1e-7


def test_free_null_and_bad_handles_are_safe():
    mars.lib().mars_free(None)
    bogus = (ctypes.c_uint64 * 4)(1, 2, 3, 4)
    mars.lib().mars_free(ctypes.cast(bogus, ctypes.c_void_p))   # wrong tag: ignored
    st = mars.lib().mars_graph_info(ctypes.cast(bogus, ctypes.c_void_p), None, None, None, None)
    assert st == mars.mars.MARS_ESTATE


def test_sass_is_sm100a():
    """The shared object carries sm_100a SASS (cuobjdump), not PTX-only."""
    import shutil
    import subprocess
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(exe):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([exe, "--list-elf", mars.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


@pytest.mark.skipif(__import__("torch").cuda.is_available(), reason="CPU-only check")
def test_no_cpu_fallback():
    class G:
        num_nodes = 2
        indptr = np.array([0, 1, 1], np.int64)
        indices = np.array([1], np.int32)
        features = np.zeros((2, 16), np.float32)
    with pytest.raises(mars.MarsError) as e:
        mars.graph_load([G()])
    assert e.value.status == mars.mars.MARS_ECUDA
    with pytest.raises(mars.MarsError) as e:
        mars.dgi_create(in_dim=16, hidden_dim=32)
    assert e.value.status == mars.mars.MARS_ECUDA
