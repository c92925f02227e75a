"""Key per-unit metrics of an ncu report: LSU wavefronts, issue, stalls, DRAM."""
import csv, re, subprocess, sys
rep = sys.argv[1]; units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines())); h, v = r[0], r[2]
d = dict(zip(h, v))
def f(k):
    try: return float(d[k].replace(',', ''))
    except Exception: return float('nan')
cyc = f('sm__cycles_elapsed.avg')
print(f"time_us {f('gpu__time_duration.sum'):.2f}  cycles/SM {cyc:.0f}")
for k in ['l1tex__data_pipe_lsu_wavefronts_mem_shared.sum', 'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum',
          'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum', 'l1tex__t_output_wavefronts_pipe_lsu_mem_global_op_ld.sum',
          'smsp__inst_executed.sum', 'dram__bytes_read.sum']:
    print(f"{k:70s} {f(k)/units:10.1f} /unit")
for k in ['l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed',
          'smsp__issue_active.avg.pct_of_peak_sustained_active', 'sm__warps_active.avg.pct_of_peak_sustained_active',
          'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'launch__registers_per_thread',
          'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active', 'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active',
          'l1tex__t_sector_hit_rate.pct', 'lts__t_sector_hit_rate.pct']:
    print(f"{k:70s} {d.get(k)}")
st = {k.split('warp_issue_stalled_')[1].split('_per')[0]: f(k) for k in h
      if k.startswith('smsp__average_warp_latency_issue_stalled_') and k.endswith('.ratio')} if False else {}
st = {}
for k in h:
    m = re.match(r'smsp__pcsamp_warps_issue_stalled_(\w+)$', k)
    if m and not m.group(1).endswith('not_issued'):
        st[m.group(1)] = f(k)
tot = sum(x for x in st.values() if x == x)
print('stalls:', ', '.join(f"{k}={100*x/tot:.1f}%" for k, x in sorted(st.items(), key=lambda t: -t[1])[:9]))
