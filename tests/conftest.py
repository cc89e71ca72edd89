import os
import sys
from pathlib import Path

import pytest

ROOT = Path(__file__).resolve().parent.parent
if str(ROOT) not in sys.path:
    sys.path.insert(0, str(ROOT))

GOLDEN = Path(__file__).resolve().parent / "golden"


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200, sm_100a) and the built libsat.so")
    config.addinivalue_line("markers", "slow: long-running (full-size) test")


def _cuda_available() -> bool:
    try:
        import torch

        return torch.cuda.is_available()
    except Exception:
        return False


def pytest_collection_modifyitems(config, items):
    if _cuda_available():
        return
    skip = pytest.mark.skip(reason="no CUDA device in this container (run with -m gpu on a B200)")
    for item in items:
        if "gpu" in item.keywords:
            item.add_marker(skip)


def read_golden_blocks(name: str) -> dict:
    """Parse a golden fixture: '#' comments, '[section]' headers, whitespace-separated int rows."""
    blocks, cur = {}, None
    for line in (GOLDEN / name).read_text().splitlines():
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        if line.startswith("[") and line.endswith("]"):
            cur = line[1:-1]
            blocks[cur] = []
            continue
        blocks.setdefault(cur, []).append([int(x) for x in line.split()])
    return blocks


@pytest.fixture(scope="session")
def golden():
    return read_golden_blocks
