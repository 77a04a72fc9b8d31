"""Top CUDA source lines of an ncu report by warp-stall samples (aggregated over their SASS),
plus the hottest SASS instructions. Usage: ncu_hot.py REPORT [N]"""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]; n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
def num(x):
    try: return float(x.replace(",", ""))
    except: return 0.0
agg = defaultdict(lambda: [0.0, 0.0, ""]); sass = []; fname = "?"; hdr = None
for r in csv.reader(io.StringIO(out)):
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or len(r) < len(hdr) or not r[2].startswith("0x"): continue
    st = num(r[4]); ins = num(r[7])
    key = f"{fname}:{r[0]}"
    a = agg[key]; a[0] += st; a[1] += ins; a[2] = a[2] or r[1].strip()
    sass.append((st, ins, key, r[3].strip()))
tot = sum(v[0] for v in agg.values()) or 1
print("== source lines by stall samples")
for k, (st, ins, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:n]:
    print(f"{st/tot*100:5.1f}%  inst {ins:>11.0f}  {k:16s} {src[:90]}")
print("== SASS by stall samples")
for st, ins, key, s in sorted(sass, key=lambda t: -t[0])[:n]:
    print(f"{st/tot*100:5.1f}%  inst {ins:>11.0f}  {key:16s} {s[:80]}")
