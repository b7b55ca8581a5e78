"""Host logic of bench.py that decides what is measured (no GPU): the
operating-point grid and the GPU-local host-core parsing."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_grid_starts_at_K_and_is_ascending():
    for K in (1, 10, 100, 127, 1000):
        g = bench.grid_for(K)
        assert g[0] == K
        assert g == sorted(set(g))
        assert all(L >= K for L in g)
        # every grid point at or above K is offered
        assert set(L for L in bench.GRID if L >= K) <= set(g)


def test_grid_for_K10_is_the_plain_grid():
    assert bench.grid_for(10) == bench.GRID


def test_gpu_local_cpus_without_gpu_is_empty():
    import torch
    if torch.cuda.is_available():
        return
    assert bench.gpu_local_cpus(0) == set()


def test_graph_choice_and_builder_params_per_config():
    from workloads.synth import CONFIGS
    assert bench.default_graph(CONFIGS["sift1m"]) == "batched"
    assert bench.default_graph(CONFIGS["nytimes256"]) == "batched"
    assert bench.default_graph(CONFIGS["gist1m"]) == "exact"
    assert bench.default_graph(CONFIGS["glove200"]) == "exact"
    for name in ("sift1m", "nytimes256"):
        b = bench.build_params(CONFIGS[name])
        assert b == bench.BUILD
        assert b["queue_len"] == 128 and b["batch_shift"] == 2 and b["prefix"] == 1 << 16
