"""Attribute ncu per-instruction counts (instructions executed, stall samples)
to CUDA source lines using nvdisasm line info of the same kernel.

usage: python tools/sass_by_line.py <report.ncu-rep> <libsong.so> <kernel-mangled-substring>
"""
import collections, csv, io, re, subprocess, sys, tempfile, os

rep, lib, kname = sys.argv[1], sys.argv[2], sys.argv[3]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]; data = rows[2:]
iex = hdr.index("Instructions Executed"); ist = hdr.index("Warp Stall Sampling (All Samples)")
isrc = hdr.index("Source")
# extract cubin and disassemble with line info
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=tmp, capture_output=True)
cubins = [os.path.join(tmp, f) for f in os.listdir(tmp) if f.endswith(".cubin")]
text = ""
for c in cubins:
    full = subprocess.run(["nvdisasm", "-g", "-c", c], capture_output=True, text=True).stdout
    # keep only the .text section of the requested kernel
    keep = False
    for l in full.splitlines():
        if l.startswith("//--------------------- .text."):
            keep = kname in l
        if keep:
            text += l + "\n"
    if text:
        break
# parse: lines "//## File "...", line N" followed by instructions "/*0120*/ OPC ..."
line_of = []
cur = None
for l in text.splitlines():
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    m = re.match(r'\s+/\*([0-9a-f]{4,})\*/\s+(.*)', l)
    if m:
        line_of.append((cur, m.group(2).strip()))
print(f"disassembled instructions {len(line_of)}, profiled {len(data)}")
te = sum(float(r[iex] or 0) for r in data); ts = sum(float(r[ist] or 0) for r in data)
agg = collections.defaultdict(lambda: [0.0, 0.0])
for k, r in enumerate(data):
    if k >= len(line_of):
        break
    agg[line_of[k][0]][0] += float(r[iex] or 0)
    agg[line_of[k][0]][1] += float(r[ist] or 0)
src = {}
for (f, n), (e, s) in sorted(agg.items(), key=lambda x: -x[1][0])[:(100000 if "--all" in sys.argv else 60)]:
    path = None
    for root in ("paper_conf_icde_zhaotl20_b200/csrc",):
        p = os.path.join(root, f) if f else None
        if p and os.path.exists(p):
            path = p
    txt = ""
    if path:
        if path not in src:
            src[path] = open(path).read().splitlines()
        txt = src[path][n - 1].strip()[:70] if n - 1 < len(src[path]) else ""
    print(f"{100*e/te:5.1f}%i {100*s/ts:5.1f}%s  {f}:{n}  {txt}")
