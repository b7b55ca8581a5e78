"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list: time
and share of the timed region per kernel.

    python tools/launch_summary.py gpurun_out/x_launches.csv "header line"
"""
import collections
import csv
import sys


def main():
    path = sys.argv[1]
    head = sys.argv[2] if len(sys.argv) > 2 else ""
    rows = [r for r in csv.reader(open(path)) if r]
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    ik, im, iv = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    tot = collections.OrderedDict()
    cnt = collections.Counter()
    for r in rows[hdr + 1:]:
        if len(r) <= iv or r[im] != "gpu__time_duration.sum":
            continue
        v = float(r[iv].replace(",", ""))
        tot[r[ik]] = tot.get(r[ik], 0.0) + v
        cnt[r[ik]] += 1
    allns = sum(tot.values())
    if head:
        print(f"# {head}")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        print(f"{k[:60]:60s} launches={cnt[k]:3d} total_ns={v:12.0f} share={v / allns:.3f}")


if __name__ == "__main__":
    main()
