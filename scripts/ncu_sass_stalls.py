"""Per-SASS-instruction stall reasons of an ncu report (top instructions by
samples), with L1 shared wavefronts: where the kernel waits and on what."""
import csv, subprocess, sys
rep = sys.argv[1]; units = float(sys.argv[2]); top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
rows = list(csv.reader(subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                                      capture_output=True, text=True).stdout.splitlines()))
h = rows[1]
ix = {k: h.index(k) for k in h}
reasons = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
res = []
tot = 0
for r in rows[2:]:
    if len(r) < len(h):
        continue
    s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    tot += s
    rs = sorted(((int(r[ix[k]] or 0), k[6:]) for k in reasons), reverse=True)[:3]
    res.append((s, r[ix["Address"]][-5:], r[ix["Source"]].strip()[:60], int(r[ix["Instructions Executed"]] or 0) / units,
                r[ix["L1 Wavefronts Shared"]], rs))
res_sorted = sorted(res, reverse=True)[:top]
for s, a, src, ie, wf, rs in res_sorted:
    print(f"{100*s/tot:5.1f}% {a} {ie:5.2f} wf={wf:>8} {src:60s} " + " ".join(f"{k}={v}" for v, k in rs if v))
