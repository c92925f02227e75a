"""Per-source-line instruction counts from an ncu report (cuda,sass view)."""
import csv, subprocess, sys, collections
rep = sys.argv[1]; units = float(sys.argv[2]); top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout.splitlines()
f = None; res = []
hdr = None
for r in csv.reader(out):
    if not r: continue
    if r[0] == "File Path": f = r[1].split('/')[-1]; continue
    if r[0] == "Function Name": continue
    if r[0] == "Line No": hdr = r; continue
    if hdr and r[0]:  # a source line row (aggregated)
        try:
            ie = int(r[hdr.index("Instructions Executed")]); st = int(r[hdr.index("Warp Stall Sampling (All Samples)")])
        except Exception:
            continue
        res.append((ie, st, f, r[0], r[1].strip()[:90]))
res.sort(reverse=True)
tot = sum(x[0] for x in res); tst = sum(x[1] for x in res)
print(f"total {tot/units:.1f} per unit")
for ie, st, f, ln, src in res[:top]:
    print(f"{ie/units:7.1f} {100*st/max(tst,1):5.1f}%  {f}:{ln}  {src}")
