import json
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import hqgen  # noqa: E402

GOLDEN = os.path.join(ROOT, "tests", "golden")

_DTYPES = {}
for _schema in hqgen.SCHEMAS.values():
    for _name, _dt in _schema:
        _DTYPES.setdefault(_name, np.dtype(_dt))


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200) and the built libhq.so")


def load_golden(name):
    """Load a tests/golden fixture; tables become dicts of typed numpy columns."""
    with open(os.path.join(GOLDEN, name)) as f:
        fx = json.load(f)
    tables = {}
    for t, cols in fx.get("tables", {}).items():
        tables[t] = {c: np.asarray(v, dtype=_DTYPES[c]) for c, v in cols.items()}
    fx["tables"] = tables
    return fx


@pytest.fixture(scope="session")
def golden():
    return load_golden
