import csv, sys, collections
path = sys.argv[1]
rows = list(csv.reader(open(path)))
cur_file = None; hdr = None; out = []
for r in rows:
    if not r: continue
    if r[0] == "File Path": cur_file = r[1].split('/')[-1]; continue
    if r[0] == "Function Name": continue
    if r[0] == "Line No": hdr = r; continue
    if hdr and len(r) == len(hdr) and r[0].isdigit():
        d = dict(zip(hdr, r))
        try: ins = int(d["Instructions Executed"]); s = int(d["Warp Stall Sampling (All Samples)"])
        except: continue
        out.append((cur_file, int(r[0]), ins, s, r[1]))
groups = eval(sys.argv[2])  # list of (name, file, lo, hi)
agg = collections.defaultdict(lambda: [0,0]); tot=[0,0]
for f,l,i,s,src in out:
    tot[0]+=i; tot[1]+=s
    for name, gf, lo, hi in groups:
        if f == gf and lo <= l <= hi: agg[name][0]+=i; agg[name][1]+=s; break
    else: agg['other:'+f][0]+=i; agg['other:'+f][1]+=s
for k,v in sorted(agg.items(), key=lambda kv:-kv[1][0]):
    print(f"{k:30s} instr {100*v[0]/tot[0]:5.1f}%  samples {100*v[1]/tot[1]:5.1f}%")
