"""Group per-line instruction/stall attribution (tools/sass_by_line.py) into
the kernel's stages, by line ranges of search_kernel.cuh."""
import re, subprocess, sys, collections
rep, lib, kname = sys.argv[1], sys.argv[2], sys.argv[3]
src = open("paper_conf_icde_zhaotl20_b200/csrc/search_kernel.cuh").read().splitlines()
def find(pat):
    for i, l in enumerate(src):
        if re.search(pat, l):
            return i + 1
    return None
marks = [
    ("hash probes", find(r"^struct HashSet")), ("bloom", find(r"^struct BloomSet")),
    ("sorting nets", find(r"^template <bool DESC>")), ("count_below", find(r"number of elements of sorted")),
    ("transpose reduce", find(r"^// Transposed butterfly")), ("reg queues", find(r"^// --------------------------------------------------- register queues")),
    ("merge", find(r"^// Bitonic merge of the sorted queue")), ("distance", find(r"^// ------------------------------------------------------- bulk distance")),
    ("kernel prologue", find(r"^// ---------------------------------------------------------- the kernel")),
    ("a3 pop/topk", find(r"// ---- a3:")), ("a4 locate", find(r"// ---- a4:")), ("a5 distance call", find(r"// ---- a5:")),
    ("a6 maintain", find(r"// ---- a6:")), ("a7 output", find(r"// ---- a7:")),
]
marks = [(n, l) for n, l in marks if l]
marks.sort(key=lambda x: x[1])
def stage_of(f, n):
    if f != "search_kernel.cuh":
        return "intrinsics (" + f + ")"
    cur = "top"
    for name, l in marks:
        if n >= l:
            cur = name
    return cur
out = subprocess.run([sys.executable, "tools/sass_by_line.py", rep, lib, kname, "--all"], capture_output=True, text=True).stdout
agg = collections.defaultdict(lambda: [0.0, 0.0])
for l in out.splitlines():
    m = re.match(r"\s*([\d.]+)%i\s+([\d.]+)%s\s+(\S+):(\d+)", l)
    if m:
        agg[stage_of(m.group(3), int(m.group(4)))][0] += float(m.group(1))
        agg[stage_of(m.group(3), int(m.group(4)))][1] += float(m.group(2))
for k, (i, s) in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{i:5.1f}% instr  {s:5.1f}% stall  {k}")
