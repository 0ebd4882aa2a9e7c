"""Per-source-line instruction and stall-sample totals of one kernel of an ncu capture.

usage: python scripts/sass_lines.py <prof.ncu-rep> <object.o> <mangled-kernel-substring> [top]
Joins `ncu --page source --print-source sass` (per-SASS-instruction counters) with
`nvdisasm -g` line info of the same build (instruction i <-> offset 16 i), and prints
source lines by executed warp instructions (with inline frames attributed to the
innermost line, as nvdisasm reports them).
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, obj, kname = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 60
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
data = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr)]
with tempfile.TemporaryDirectory() as td:
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=td,
                   capture_output=True)
    cub = [f for f in os.listdir(td) if f.endswith(".cubin")][0]
    sass = subprocess.run(["nvdisasm", "-g", os.path.join(td, cub)], capture_output=True,
                          text=True).stdout
lines = sass.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith(".text.") and kname in l)
line_of = {}
cur = None
for l in lines[start + 1:]:
    if l.startswith("//---------------------"):
        break
    m = re.match(r'\s*//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m:
        line_of[int(m.group(1), 16) // 16] = cur
inst = collections.Counter()
samp = collections.Counter()
tot_i = tot_s = 0
for i, r in enumerate(data):
    n = int(r["Instructions Executed"] or 0)
    s = int(r["# Samples"] or 0)
    key = line_of.get(i, ("?", 0))
    inst[key] += n
    samp[key] += s
    tot_i += n
    tot_s += s
src = {}
def text(f, n):
    if f not in src:
        p = os.path.join(os.path.dirname(os.path.abspath(__file__)), "..",
                         "paper_conf_ipps_zhangwlf14_b200", "csrc", f)
        src[f] = open(p).read().splitlines() if os.path.exists(p) else []
    return src[f][n - 1].strip()[:70] if 0 < n <= len(src[f]) else ""
print(f"instructions executed {tot_i:.3e}, samples {tot_s}")
for key, n in inst.most_common(top):
    print(f"{key[0][:12]:12s}:{key[1]:4d} inst {100 * n / tot_i:5.1f}% samp "
          f"{100 * samp[key] / max(tot_s, 1):5.1f}%  {text(*key)}")
if os.environ.get("TOP_INSTR"):
    # the instructions with the most stall samples, with their source line
    order = sorted(range(len(data)), key=lambda i: -int(data[i]["# Samples"] or 0))
    print("--- top instructions by stall samples")
    for i in order[:int(os.environ["TOP_INSTR"])]:
        r = data[i]
        key = line_of.get(i, ("?", 0))
        print(f"{100 * int(r['# Samples'] or 0) / max(tot_s, 1):5.1f}%  {r['Source'][:44]:44s} "
              f"{key[0][:12]}:{key[1]} {text(*key)[:60]}")
