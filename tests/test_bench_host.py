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
    for name in ("sift1m", "nytimes256", "gist1m", "glove200"):
        assert bench.default_graph(CONFIGS[name]) == "mixed"
        chain = bench.MIXED[name]
        assert isinstance(chain[0], str) and len(chain) >= 2
        for spec, take in chain[1:]:
            assert 0 < take < CONFIGS[name].degree
            assert spec.split(":")[0] in ("exact", "batched")
    assert bench.MIXED["glove200"][0] == "exact:ip"  # the IP graph's links first ...
    assert bench.MIXED["glove200"][1][0].startswith("batched:cosine")  # ... then angular ones
    assert bench.default_graph(CONFIGS["scaleout100m"]) == "batched"  # R15 is O(n^2)
    for name in ("sift1m", "nytimes256"):
        b = bench.build_params(CONFIGS[name])
        assert b == bench.BUILD
        assert b["queue_len"] == 128 and b["batch_shift"] == 2 and b["prefix"] == 1 << 16


def test_gpus_flag_launches_ranks_gloo():
    """`bench.py --gpus 2` without a torchrun environment re-launches itself
    under torch.distributed.run with 2 ranks (CPU: gloo); rank 0 reports the
    world it saw."""
    import json
    import subprocess
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    env["SONG_BENCH_BACKEND"] = "gloo"
    env["CUDA_VISIBLE_DEVICES"] = ""
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2",
                          "--launch-check"], capture_output=True, text=True, env=env, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [json.loads(l) for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    assert lines[0]["n_gpus"] == 2 and lines[0]["backend"] == "gloo"
    assert lines[0]["rank_sum"] == 3.0  # ranks 0 and 1 both joined


def test_parity_gate_bars():
    import numpy as np
    gi = np.arange(2000).reshape(200, 10).astype(np.int32)
    gd = np.linspace(1, 2, 2000).reshape(200, 10).astype(np.float32)
    gc = np.ones((200, 2), np.int64)
    truth = gi.copy()
    ok = bench.parity_gate(gi, gd, gc, gi.copy(), gd.copy(), gc.copy(), truth, exact=True)
    assert ok["ok"] and ok["ids_equal"] == 1.0
    # one query of 200 differs: 0.995 passes the float bar, never the integer one
    oi = gi.copy()
    oi[0, 9] = 99999
    f = bench.parity_gate(gi, gd, gc, oi, gd.copy(), gc.copy(), truth, exact=False)
    assert f["ok"] and f["ids_equal"] == 0.995
    assert not bench.parity_gate(gi, gd, gc, oi, gd.copy(), gc.copy(), truth, exact=True)["ok"]
    oi[1, 9] = 99999  # two of 200: below 0.995
    assert not bench.parity_gate(gi, gd, gc, oi, gd.copy(), gc.copy(), truth, exact=False)["ok"]
    # a distance off by more than rtol 1e-5 fails
    od = gd.copy()
    od[5, 3] *= 1.001
    assert not bench.parity_gate(gi, gd, gc, gi.copy(), od, gc.copy(), truth, exact=False)["ok"]
