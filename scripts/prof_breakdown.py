"""Instruction / stall-sample breakdown of the block kernel by code region.
usage: python scripts/prof_breakdown.py <prof.ncu-rep> [kernel-substring]"""
import collections, os, re, subprocess, sys
rep = sys.argv[1]
kern = sys.argv[2] if len(sys.argv) > 2 else "search_block_kernelILb0ELi3ELb0E"
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
obj = os.path.join(root, "paper_conf_ipps_zhangwlf14_b200", "build", "search_block.cu.o")
out = subprocess.run([sys.executable, os.path.join(root, "scripts", "sass_lines.py"), rep, obj, kern,
                      "100000"], capture_output=True, text=True).stdout
src = open(os.path.join(root, "paper_conf_ipps_zhangwlf14_b200", "csrc", "search_block.cu")).read().split("\n")
# regions by markers in search_block.cu
# line numbers of the build the capture was taken with: STRIP_REGIONS=1 when
# that build predates the REGION marker lines (they are pure insertions)
strip = os.environ.get("STRIP_REGIONS") == "1"
marks = {}
n = 0
for l in src:
    if "REGION:" in l:
        marks[n + 1 if strip else n + 1] = l.split("REGION:")[1].strip().split()[0]
        if strip:
            continue
    n += 1
starts = sorted(marks)
def region(ln):
    r = "other"
    for s in starts:
        if s <= ln:
            r = marks[s]
    return r
tot = collections.Counter(); samp = collections.Counter()
for l in out.split("\n"):
    m = re.match(r'(\S+)\s*:\s*(\d+) inst\s+([\d.]+)% samp\s+([\d.]+)%', l)
    if not m:
        continue
    f, ln, ip, sp = m.group(1), int(m.group(2)), float(m.group(3)), float(m.group(4))
    if f.startswith("search_commo"):
        cat = "xdrop" if 26 <= ln <= 180 else "common"
    elif f.startswith("search_block"):
        cat = region(ln)
    else:
        cat = "intrinsics"
    tot[cat] += ip; samp[cat] += sp
print(out.split("\n")[0])
for k, v in tot.most_common():
    print(f"{k:14s} inst {v:5.1f}%  stall samples {samp[k]:5.1f}%")
