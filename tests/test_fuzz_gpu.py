"""A short randomised GPU-vs-oracle sweep (scripts/fuzz_parity.py, 20 s): random shapes,
batch sizes, value ranges, tie-heavy epochs, forced kernel paths, constrained and pruned
calls -- every result bit-exact against the CPU oracle. Run with ``pytest -m gpu``."""
from __future__ import annotations

import json
import os
import subprocess
import sys

import pytest

from conftest import cuda_available

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_fuzz_parity_short():
    if not cuda_available():
        pytest.fail("no CUDA device: the -m gpu tests must run on a GPU box")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "fuzz_parity.py"), "20", "2024"],
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    summary = json.loads(r.stdout.strip().splitlines()[-1])
    assert summary["cases"] > 200, summary
    assert summary["failures"] == 0, r.stdout[-2000:]
