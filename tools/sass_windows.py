"""Instruction / stall share by SASS window (where the time goes)."""
import csv, subprocess, io, sys
from collections import Counter
rep = sys.argv[1]; W = int(sys.argv[2]) if len(sys.argv) > 2 else 24
thr = float(sys.argv[3]) if len(sys.argv) > 3 else 0.012
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out))); hdr=rows[1]; data=rows[2:]
isrc=hdr.index("Source"); ist=hdr.index("Warp Stall Sampling (All Samples)"); iex=hdr.index("Instructions Executed")
ts=sum(float(r[ist] or 0) for r in data); te=sum(float(r[iex] or 0) for r in data)
print(f"instructions {te:.4g}  stall samples {ts:.0f}")
for w in range(0,len(data),W):
    ch=data[w:w+W]; s=sum(float(r[ist] or 0) for r in ch); e=sum(float(r[iex] or 0) for r in ch)
    if s/ts>thr or e/te>thr:
        ops=[(r[isrc].split()[1] if r[isrc].strip().startswith('@') else r[isrc].split()[0]) for r in ch if r[isrc].strip()]
        c=Counter(o.split('.')[0] for o in ops).most_common(6)
        print(f"{w:5d} i={100*e/te:5.1f}% s={100*s/ts:5.1f}%  {c}")
