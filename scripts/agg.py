import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = None; cur_file = "?"; cur_line = None
by_line = collections.defaultdict(lambda: [0,0, collections.Counter()]); src = {}
for r in rows:
    if not r: continue
    if r[0] == "File Path": cur_file = r[1].split("/")[-1]; continue
    if r[0] == "Function Name": continue
    if r[0] == "Line No": hdr = r; ie = hdr.index("Instructions Executed"); samp = hdr.index("Warp Stall Sampling (All Samples)"); stall_cols = [i for i,h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]; continue
    if hdr is None or len(r) < len(hdr): continue
    if r[0]:
        cur_line = (cur_file, int(r[0])); src[cur_line] = r[1]
    if not r[2] or r[2] == "...": continue
    try:
        by_line[cur_line][0] += int(r[ie] or 0)
        by_line[cur_line][1] += int(r[samp] or 0)
        for c in stall_cols:
            v = int(r[c] or 0)
            if v: by_line[cur_line][2][hdr[c]] += v
    except ValueError:
        pass
tot_i = sum(v[0] for v in by_line.values()); tot_s = sum(v[1] for v in by_line.values())
print("total instr", tot_i, "samples", tot_s)
for ln, (i, s, st) in sorted(by_line.items(), key=lambda kv: -kv[1][1])[:int(sys.argv[2]) if len(sys.argv)>2 else 40]:
    top = ", ".join(f"{k[6:]}:{v*100//max(s,1)}%" for k, v in st.most_common(3))
    print(f"{ln[0][:10]}:{ln[1]:4d} instr {100*i/tot_i:5.1f}% samp {100*s/tot_s:5.1f}%  {src.get(ln,'').strip()[:58]:58s} | {top}")
groups = {"xdrop(84-119)": (84,119), "successor(123-140)":(120,141), "trace":(142,152), "flush(157-230)":(157,232), "kernel-setup(233-268)":(233,268), "iter-load+lookup(269-300)":(269,301), "helpers(301-340)":(301,341), "fill(341-346)":(341,346), "passA(347-357)":(347,357), "passB(358-375)":(358,375), "passC(376-389)":(376,389), "slow(390-430)":(390,430), "tail(430-440)":(430,440)}
print()
for g,(a,b) in groups.items():
    i = sum(v[0] for k,v in by_line.items() if k[0]=="search.cu" and a<=k[1]<=b)
    s = sum(v[1] for k,v in by_line.items() if k[0]=="search.cu" and a<=k[1]<=b)
    print(f"{g:28s} instr {100*i/tot_i:5.1f}%  samples {100*s/tot_s:5.1f}%")
i = sum(v[0] for k,v in by_line.items() if k[0]!="search.cu"); s = sum(v[1] for k,v in by_line.items() if k[0]!="search.cu")
print(f"{'intrinsics(other files)':28s} instr {100*i/tot_i:5.1f}%  samples {100*s/tot_s:5.1f}%")
