"""Where does the end-to-end step (song_search with host buffers) spend its
time beyond the device step?  Times, on the bench workload: the pinned HtoD
copy of the query batch alone, the DtoH of the results alone, the device step
(CUDA events), and the whole song_search call (wall clock).

    python tools/e2e_probe.py
"""
import json
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
    # as bench.py's e2e loop: a 512 MiB L2 flush + synchronize before each call
    flush = torch.empty(128 << 20, dtype=torch.float32, device=dev)

    def flushed(fn, n=20):
        ts = []
        for i in range(n + 3):
            flush.zero_()
            torch.cuda.synchronize()
            t = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            if i >= 3:
                ts.append(time.perf_counter() - t)
        return [round(float(np.percentile(ts, k)) * 1e3, 4) for k in (0, 50, 100)]

    res["device_step_wall_flushed_ms_min_med_max"] = flushed(
        lambda: idx.search(q, params=p, out=out))
    res["song_search_flushed_ms_min_med_max"] = flushed(
        lambda: idx.search_host_into(qh, 10, L, ih, dh))
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]

    def dev_timed_call():
        ev[0].record()
        idx.search_host_into(qh, 10, L, ih, dh)
        ev[1].record()

    # the call on the device clock (events on torch's stream bracket the
    # library's stream work because song_search synchronizes before returning)
    ts = []
    for i in range(23):
        flush.zero_()
        torch.cuda.synchronize()
        dev_timed_call()
        torch.cuda.synchronize()
        if i >= 3:
            ts.append(ev[0].elapsed_time(ev[1]))
    res["song_search_flushed_event_ms_min_med_max"] = [round(float(np.percentile(ts, k)), 4)
                                                       for k in (0, 50, 100)]
    print(json.dumps(res))
    if len(sys.argv) > 1:
        with open(sys.argv[1], "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
