"""Where does the end-to-end step (song_search with host buffers) spend its
time beyond the device step?  Times, on the bench workload: the pinned HtoD
copy of the query batch alone, the DtoH of the results alone, the device step
(CUDA events), and the whole song_search call (wall clock).

    python tools/e2e_probe.py
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def main():
    import numpy as np
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS
    cfg = CONFIGS["sift1m"]
    dev = torch.device("cuda", 0)
    x, q0, q, adj = bench.build_workload(cfg, dev, 0, print)
    idx = song.SongIndex(x, adj)
    L = 32
    qh = q.cpu().pin_memory()
    ih = torch.empty((q.shape[0], 10), dtype=torch.int32).pin_memory()
    dh = torch.empty((q.shape[0], 10), dtype=torch.float32).pin_memory()
    qd = torch.empty_like(q)
    res = {}

    def wall(fn, n=20):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(n):
            t = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t)
        return float(np.median(ts)) * 1e3

    res["h2d_5MB_ms"] = wall(lambda: qd.copy_(qh, non_blocking=True))
    od = torch.empty((q.shape[0], 10), dtype=torch.int32, device=dev)
    res["d2h_0.4MB_ms"] = wall(lambda: ih.copy_(od, non_blocking=True))
    out = (torch.empty((q.shape[0], 10), dtype=torch.int32, device=dev),
           torch.empty((q.shape[0], 10), dtype=torch.float32, device=dev), None)
    p = song.Params(K=10, queue_len=L)
    res["device_step_wall_ms"] = wall(lambda: idx.search(q, params=p, out=out))
    res["song_search_ms"] = wall(lambda: idx.search_host_into(qh, 10, L, ih, dh))
    print(res)


if __name__ == "__main__":
    main()
