"""The C-ABI library loads on a CPU-only box and exports every symbol include/olap.h
declares; without a GPU its compute entry points fail loudly (no CPU fallback)."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    txt = open(os.path.join(ROOT, "include", "olap.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(olap_[a-z_]+)\s*\(", txt)))


def test_header_declares_the_boundary():
    names = _declared()
    for must in ("olap_cube_create", "olap_cube_load", "olap_dict_build", "olap_dict_translate",
                 "olap_query_batch", "olap_query_batch_device", "olap_query_partials_device",
                 "olap_finalize_device", "olap_last_error"):
        assert must in names


def test_library_exports_every_declared_symbol():
    import paper_conf_ipps_malikrse12_b200 as olap
    raw = ctypes.CDLL(olap.LIB_PATH)
    for name in _declared():
        assert hasattr(raw, name), f"{name} declared in olap.h but not exported"
    # the binding wires exactly the declared set
    assert set(olap.EXPORTS) == set(_declared())
    assert b"sm_100a" in olap.lib.olap_version()


def test_sm100a_code_in_library():
    import subprocess
    import paper_conf_ipps_malikrse12_b200 as olap
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", olap.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_no_cpu_fallback_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import paper_conf_ipps_malikrse12_b200 as olap
    with pytest.raises(olap.OlapError) as ei:
        olap.Cube((4, 4), np.int32)
    assert ei.value.status == olap.E_CUDA
    with pytest.raises(olap.OlapError):
        olap.Dict(["a", "b"])


def test_layout_arguments_validated_before_the_device():
    """olap_cube_create_layout rejects an unknown layout and bricked shapes outside ndims 3-6
    with OLAP_E_INVALID on any box (argument checks come before any CUDA call)."""
    import paper_conf_ipps_malikrse12_b200 as olap
    for ext, layout in (((4, 4, 4), 7), ((10, 20), olap.LAYOUT_BRICK), ((2,) * 7, olap.LAYOUT_BRICK),
                        ((4, 0, 4), olap.LAYOUT_BRICK), ((10, 20), olap.LAYOUT_BRICK3),
                        ((2,) * 7, olap.LAYOUT_BRICK3), ((0, 4, 4), olap.LAYOUT_BRICK3)):
        with pytest.raises(olap.OlapError) as ei:
            olap.Cube(ext, np.float32, layout=layout)
        assert ei.value.status == olap.E_INVALID, (ext, layout)
