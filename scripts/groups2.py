import sys
FILE = __import__("os").environ.get("SRCFILE", "search.cu")
exec(open('/tmp/agg.py').read().split("tot_i = ")[0])
tot_i = sum(v[0] for v in by_line.values()); tot_s = sum(v[1] for v in by_line.values())
import re
src_lines = open('/root/repo/paper_conf_ipps_zhangwlf14_b200/csrc/search.cu').read().split('\n')
groups = [(a,b,n) for a,b,n in [tuple(x.split(':')) for x in sys.argv[2].split(',')]]
for a,b,n in groups:
    a=int(a); b=int(b)
    i = sum(v[0] for k,v in by_line.items() if k[0].startswith(FILE) and a<=k[1]<=b)
    s = sum(v[1] for k,v in by_line.items() if k[0].startswith(FILE) and a<=k[1]<=b)
    print(f"{n:28s} L{a}-{b} instr {100*i/tot_i:5.1f}%  samples {100*s/tot_s:5.1f}%")
i = sum(v[0] for k,v in by_line.items() if not k[0].startswith(FILE)); s = sum(v[1] for k,v in by_line.items() if k[0]!="search.cu")
print(f"{'intrinsics(other files)':28s} instr {100*i/tot_i:5.1f}%  samples {100*s/tot_s:5.1f}%")
