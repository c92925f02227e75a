"""Summarise an ncu report: instruction mix per work unit, stalls, key metrics."""
import csv, collections, re, subprocess, sys
rep = sys.argv[1]
units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                     capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(src))
h = rows[1]
iS, iE, iW = h.index('Source'), h.index('Instructions Executed'), h.index('Warp Stall Sampling (All Samples)')
op, stall = collections.Counter(), collections.Counter()
tot = tots = 0
for r in rows[2:]:
    if len(r) < len(h) or not r[iE].isdigit():
        continue
    m = re.match(r'(@!?U?P\w+\s+)?([A-Z0-9_.]+)', r[iS].strip())
    o = (m.group(2) if m else r[iS]).split('.')[0]
    e, w = int(r[iE] or 0), int(r[iW] or 0)
    op[o] += e; stall[o] += w; tot += e; tots += w
print(f"instructions {tot}  per unit {tot/units:.1f}")
for o, c in op.most_common(int(sys.argv[3]) if len(sys.argv) > 3 else 16):
    print(f"  {o:10s} {c/units:8.1f}  stall {100*stall[o]/max(tots,1):5.1f}%")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout.splitlines()
r = list(csv.reader(raw)); hh, vv = r[0], r[2]
want = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'launch__registers_per_thread', 'launch__occupancy_limit_registers',
        'launch__occupancy_limit_shared_mem', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'l1tex__t_sector_hit_rate.pct',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed']
for k, x in zip(hh, vv):
    if k in want:
        print(f"{k} = {x}")
st = [(k, x) for k, x in zip(hh, vv) if 'pcsamp_warps_issue_stalled' in k and not k.endswith('not_issued')]
st = sorted(((float(x), k.replace('smsp__pcsamp_warps_issue_stalled_', '')) for k, x in st if x), reverse=True)[:8]
print("stalls:", ", ".join(f"{k}={int(v)}" for v, k in st))
