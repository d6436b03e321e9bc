"""C-ABI boundary checks that need no GPU: libhq.so loads, exports every
symbol include/hq.h declares, its struct layouts match the Python mirrors,
and without a device every entry point fails loudly (no CPU fallback)."""
import ctypes
import os
import re

import pytest

from paper_conf_sigmod_funkebnmt18_b200 import hq

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_functions():
    src = open(os.path.join(ROOT, "include", "hq.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:hq_status|const char\*|int32_t|size_t)\s+(hq_\w+)\s*\(", src, flags=re.M)))


def test_library_exports_every_declared_symbol():
    names = _declared_functions()
    assert len(names) >= 20
    L = hq.lib()
    for n in names:
        assert hasattr(L, n), n
    assert sorted(hq.EXPORTS) == names


def test_struct_layouts_match():
    L = hq.lib()
    assert L.hq_abi_version() == 1
    for name, S in hq.STRUCTS.items():
        assert L.hq_sizeof(name.encode()) == ctypes.sizeof(S), name


def test_no_device_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a device is present")
    with pytest.raises(hq.HQError) as e:
        hq.Context(0, stream=0)
    assert e.value.code == hq.HQ_ERR_NO_DEVICE


def test_null_arguments_rejected():
    L = hq.lib()
    assert L.hq_run_pipeline(None, None, None) == hq.HQ_ERR_ARG
    assert L.hq_fetch_result(None, None, None, 0, None) == hq.HQ_ERR_ARG
    assert L.hq_last_error()
