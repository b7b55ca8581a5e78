"""examples/search_example.c on the GPU: index create, song_search and
song_search_pipelined from plain C; the full-queue search equals brute force."""
import subprocess

import pytest

pytestmark = pytest.mark.gpu

from test_abi import _build_c_example  # noqa: E402


def test_c_example_runs(tmp_path):
    exe = _build_c_example(tmp_path)
    res = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert res.returncode == 0, res.stdout + res.stderr
    assert "exact top-K ok" in res.stdout
