"""Key metrics of an assign_tc ncu capture (per 128-point tile): python scripts/km_ncu_summary.py REP"""
import csv, subprocess, sys, io, collections
rep = sys.argv[1]
raw = list(csv.reader(io.StringIO(subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout)))
h, v = raw[0], raw[2]
m = {h[i]: v[i] for i in range(len(h))}
def g(k): return float(m[k].replace(',', ''))
tiles = float(sys.argv[2]) if len(sys.argv) > 2 else 44400.0  # 5683200 points / 128 (scripts/km_prof)
sms = 148
print(f"duration {g('gpu__time_duration.sum') if 'gpu__time_duration.sum' in m else 0} tiles {tiles:.0f}  cycles/tile/SM {g('sm__cycles_elapsed.max') * sms / tiles:.0f}")
for k in ['sm__inst_executed.sum', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum', 'l1tex__data_pipe_tc_wavefronts_mem_shared.sum',
          'l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum', 'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum',
          'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum']:
    if k in m: print(f"  {k:60s} {g(k) / tiles:10.1f} per tile (per SM)" if 'sum' in k else '')
for k in ['sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active', 'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active',
          'sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active', 'sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active',
          'sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active',
          'smsp__issue_active.avg.pct_of_peak_sustained_active', 'l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed',
          'l1tex__data_pipe_tc_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed', 'launch__registers_per_thread']:
    if k in m: print(f"  {k:60s} {m[k]}")
src = list(csv.reader(io.StringIO(subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'], capture_output=True, text=True).stdout)))
hd = src[1]; ix = hd.index('Instructions Executed')
op = collections.Counter()
for x in src[2:]:
    try: n = int(x[ix])
    except Exception: continue
    t = x[1].split(); o = t[1] if t[0].startswith('@') else t[0]
    op[o.split('.')[0]] += n
print('  per-tile SASS mix:', ', '.join(f"{k} {c / tiles:.0f}" for k, c in op.most_common(24)))
