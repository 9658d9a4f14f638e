import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (run with -m gpu under gpurun)")
    config.addinivalue_line("markers", "slow: full-size cases (minutes on CPU)")


def pytest_collection_modifyitems(config, items):
    try:
        import torch
        has_gpu = torch.cuda.is_available()
    except Exception:  # pragma: no cover
        has_gpu = False
    if has_gpu:
        return
    skip = pytest.mark.skip(reason="no CUDA device")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)


def read_golden(name):
    """Parse a tests/golden/*.txt fixture: '# comments', 'key v v v' lines and a
    'rows' section of whitespace-separated column lists (empty line = empty row)."""
    path = os.path.join(ROOT, "tests", "golden", name)
    out, rows, in_rows = {}, [], False
    with open(path) as f:
        for raw in f:
            line = raw.rstrip("\n")
            if line.startswith("#"):
                continue
            if line.strip() == "rows":
                in_rows = True
                continue
            parts = line.split()
            if in_rows and parts and parts[0].lstrip("-").isdigit():
                rows.append([int(x) for x in parts])
                continue
            in_rows = False
            if not parts:
                continue
            out[parts[0]] = [int(x) if x.lstrip("-").isdigit() else x for x in parts[1:]]
    out["rows"] = rows
    return out
