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
        try:
            s = int(d["Warp Stall Sampling (All Samples)"]); ins = int(d["Instructions Executed"])
        except: continue
        out.append((ins, s, cur_file, int(r[0]), r[1][:100]))
tot_i = sum(o[0] for o in out)
print("total warp instr", tot_i)
for o in sorted(out, reverse=True)[:int(sys.argv[2])]:
    print(f"{100*o[0]/tot_i:5.1f}%  {o[2]}:{o[3]}  {o[4]}")
