"""Attribute an ncu report's per-SASS instruction counts and stall samples to CUDA source
lines (nvdisasm -g line info of the same libgfsl.so build).
python tools/sass_lines.py REPORT.ncu-rep KERNEL_MANGLED_PREFIX NCU_NAME_REGEX [lib.so]
(SRC_DIR = the csrc/ tree the library was built from, default the working tree)"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, kname, nregex = sys.argv[1], sys.argv[2], sys.argv[3]
lib = sys.argv[4] if len(sys.argv) > 4 else "paper_conf_ppopp_moscovicicp17_b200/libgfsl.so"
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=tmp, capture_output=True)
sass, start = None, None
for cubin in sorted(f for f in os.listdir(tmp) if f.endswith(".cubin")):
    lines = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(tmp, cubin)], capture_output=True,
                           text=True).stdout.split("\n")
    hits = [i for i, l in enumerate(lines) if l.startswith(".text." + kname)]
    if hits:
        sass, start = lines, hits[0]
        break
cur, off2line = None, {}
for l in sass[start + 1:]:
    if l.startswith(".text."):
        break
    m = re.search(r'## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (m.group(1).split("/")[-1], int(m.group(2)))
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/", l)
    if m:
        off2line[int(m.group(1), 16)] = cur
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", "regex:" + nregex],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
hi = [i for i, x in enumerate(r) if x and x[0] == "Address"][0]
h = r[hi]
rows = [x for x in r[hi + 1:] if len(x) == len(h) and x[0].startswith("0x")]


def I(v):
    try:
        return int(v)
    except ValueError:
        return 0


ii, si = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
base = int(rows[0][0], 16)
agg, st, seen = collections.Counter(), collections.Counter(), set()
for x in rows:
    a = int(x[0], 16)
    if a in seen:
        continue
    seen.add(a)
    ln = off2line.get(a - base)
    agg[ln] += I(x[ii])
    st[ln] += I(x[si])
tot, stt = sum(agg.values()), max(1, sum(st.values()))
print(f"total warp instructions {tot}, stall samples {stt}")
srcs = {}
for ln, c in agg.most_common(45):
    s = ""
    if ln:
        p = os.path.join(os.environ.get("SRC_DIR", "paper_conf_ppopp_moscovicicp17_b200/csrc"), ln[0])
        if os.path.exists(p):
            srcs.setdefault(p, open(p).read().split("\n"))
            s = srcs[p][ln[1] - 1].strip()[:80]
    print(f"{c:10d} {100 * c / tot:5.1f}%  stall {100 * st[ln] / stt:5.1f}%  {ln}  {s}")
