"""Per-source-line instruction / stall-sample shares from an ncu report (source page).  usage: python tools/ncu_lines.py REPORT.ncu-rep [N]"""
import csv, subprocess, sys
rep, n = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
cur = hdr = None; out = []
for r in csv.reader(txt.splitlines()):
    if not r: continue
    if r[0] == "File Path": cur = r[1].split('/')[-1]; continue
    if r[0] == "Function Name": continue
    if r[0] == "Line No": hdr = r; continue
    if hdr and r[0].isdigit():
        try: s = int(r[4]); ins = int(r[7])
        except ValueError: continue
        out.append((ins, s, cur, int(r[0]), r[1][:100]))
ti = sum(o[0] for o in out); ts = sum(o[1] for o in out)
print("warp instr", ti, "stall samples", ts)
for o in sorted(out, reverse=True)[:n]:
    print(f"{100*o[0]/ti:5.1f}% {100*o[1]/ts:5.1f}%  {o[2]}:{o[3]}  {o[4]}")
