"""Summarise gpurun_out/prof_round into profiles/ (tracked)."""
import csv, collections, json, os, shutil, subprocess, sys
R = sys.argv[1] if len(sys.argv) > 1 else "r01"
src = "gpurun_out/prof_round"
dst = "profiles"
os.makedirs(dst, exist_ok=True)
for f in ["bench.jsonl", "bench_reference.jsonl", "pcg.jsonl", "coverage.jsonl", "gpu.csv",
          "bench_27pt128.jsonl", "bench_27pt256.jsonl", "bench_rmat20.jsonl", "bench_5pt64.jsonl",
          "bench_rmat24.jsonl", "compare_7pt128.jsonl", "compare_27pt128.jsonl",
          "compare_rmat20.jsonl", "compare_5pt64.jsonl"]:
    p = os.path.join(src, f)
    if os.path.exists(p):
        lines = [l for l in open(p) if l.strip().startswith("{") or f.endswith(".csv")]
        open(os.path.join(dst, f"{R}_{f}"), "w").writelines(lines)
# launch list: per-kernel totals and shares
rows = [r for r in csv.reader(open(os.path.join(src, "launches.csv"))) if len(r) > 5]
h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value")
tot = collections.defaultdict(float); cnt = collections.Counter()
for r in rows[1:]:
    tot[r[ki]] += float(r[vi].replace(",", "")); cnt[r[ki]] += 1
all_ns = sum(tot.values())
with open(os.path.join(dst, f"{R}_launches_summary.txt"), "w") as f:
    f.write("ncu --metrics gpu__time_duration.sum --clock-control none (bench.py --steps 5 --warmup 3)\n")
    f.write("cold-cache, serialised launches: compare shares, not absolute times\n\n")
    f.write(f"{'launches':>8} {'avg us':>10} {'share':>7}  kernel\n")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        f.write(f"{cnt[k]:8d} {v / cnt[k] / 1e3:10.2f} {100 * v / all_ns:6.1f}%  {k[:90]}\n")
shutil.copy(os.path.join(src, "launches.csv"), os.path.join(dst, f"{R}_launches.csv"))
# full capture summary + traffic per launch for bench.py's roofline
rep = os.path.join(src, "k_lean.ncu-rep")
out = subprocess.run([sys.executable, "scripts/ncu_summary.py", rep, "65536", "30"],
                     capture_output=True, text=True).stdout
lines = subprocess.run([sys.executable, "scripts/ncu_lines.py", rep, "65536", "30"],
                       capture_output=True, text=True).stdout
open(os.path.join(dst, f"{R}_k_lean_ncu_summary.txt"), "w").write(
    "ncu --set full --clock-control none -k regex:k_lean (bench workload 7pt128, k_lean<CHECK, SHORT>)\n"
    "per-unit counts are per 32-row group (65536 groups)\n\n" + out + "\nper source line:\n" + lines)
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout.splitlines()
r = list(csv.reader(raw)); hh = r[0]; units = r[1]
res = []
for row in r[2:]:
    d = dict(zip(hh, row))
    u = dict(zip(hh, units))
    def mb(k):
        v = float(d[k].replace(",", "")); un = u.get(k, "")
        return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(un, 1)
    res.append({"kernel": d.get("Kernel Name"), "dram_read": mb("dram__bytes_read.sum"),
                "dram_write": mb("dram__bytes_write.sum")})
prot = [x for x in res if "(bool)1" in (x["kernel"] or "") or "<1," in (x["kernel"] or "")]
pick = prot[0] if prot else res[0]
json.dump({"source": f"profiles/{R}_k_lean_ncu_summary.txt (ncu --set full capture)",
           "kernel": pick["kernel"], "dram_bytes_per_launch": pick["dram_read"] + pick["dram_write"],
           "all": res}, open(os.path.join(dst, "traffic_7pt128.json"), "w"), indent=1)
print(open(os.path.join(dst, f"{R}_launches_summary.txt")).read())
print(out)
