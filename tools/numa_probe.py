"""Does the host NUMA node matter for the e2e step's copies?  Times a pinned
5.12 MB HtoD (the SIFT1M batch) and an 0.8 MB DtoH (its results) with the
process bound to each NUMA node's cores in turn, the pinned buffers allocated
under that binding.

    python tools/numa_probe.py [--out gpurun_out/numa_probe.json]
"""
import argparse
import glob
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def cpulist(text):
    out = set()
    for part in text.strip().split(","):
        if "-" in part:
            a, b = part.split("-")
            out.update(range(int(a), int(b) + 1))
        elif part:
            out.add(int(part))
    return out


def main():
    import torch
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    dev = torch.cuda.current_device()
    allc = os.sched_getaffinity(0)
    nodes = {}
    for d in sorted(glob.glob("/sys/devices/system/node/node[0-9]*")):
        with open(os.path.join(d, "cpulist")) as f:
            c = cpulist(f.read()) & allc
        if c:
            nodes[os.path.basename(d)] = c
    local = bench.gpu_local_cpus(dev)
    res = {"gpu_local_cpus": len(local), "nodes": {}}
    src = torch.randn(10000, 128, device="cuda")
    for name, cpus in list(nodes.items()) + [("all", allc)]:
        os.sched_setaffinity(0, cpus)
        qh = torch.empty(src.shape, dtype=torch.float32, pin_memory=True)
        oh = torch.empty((10000, 20), dtype=torch.float32, pin_memory=True)
        dq = torch.empty_like(src)
        do = torch.empty((10000, 20), device="cuda")
        ts = {"h2d": [], "d2h": []}
        for i in range(25):
            torch.cuda.synchronize()
            t = time.perf_counter()
            dq.copy_(qh, non_blocking=True)
            torch.cuda.synchronize()
            t1 = time.perf_counter()
            oh.copy_(do, non_blocking=True)
            torch.cuda.synchronize()
            t2 = time.perf_counter()
            if i >= 5:
                ts["h2d"].append((t1 - t) * 1e3)
                ts["d2h"].append((t2 - t1) * 1e3)
        res["nodes"][name] = {
            "cores": len(cpus), "gpu_local": bool(cpus & local) if name != "all" else None,
            "h2d_ms_median": sorted(ts["h2d"])[10], "d2h_ms_median": sorted(ts["d2h"])[10]}
        del qh, oh
    os.sched_setaffinity(0, allc)
    print(json.dumps(res, indent=1))
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
