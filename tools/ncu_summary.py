"""Summarise an ncu --set full report: headline metrics, pipe use, stalls, and the
basic blocks by stall share.  usage: ncu_summary.py REPORT SIMS_PER_LAUNCH [N_BLOCKS]"""
import csv, sys, subprocess
from collections import Counter
rep = sys.argv[1]; sims = float(sys.argv[2]) / 32
raw = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines())); h = r[0]; v = r[2]
H0, V0 = h, v
want = ['gpu__time_duration.sum', 'sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active', 'sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active', 'smsp__issue_active.avg.pct_of_peak_sustained_active', 'smsp__warps_active.avg.per_cycle_active', 'smsp__warps_eligible.avg.per_cycle_active', 'smsp__inst_executed.sum', 'launch__registers_per_thread', 'sass__inst_executed_local_loads', 'sass__inst_executed_local_stores', 'dram__bytes_read.sum', 'dram__bytes_write.sum']
for i, name in enumerate(h):
    if name in want: print(name, v[i])
for i, name in enumerate(h):
    if 'issue_stalled' in name and 'per_issue_active.ratio' in name and float(v[i] or 0) > 0.05:
        print('  stall', name.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', ''), v[i])
src = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'], capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines())); h = rows[1]; ix = {k: i for i, k in enumerate(h)}
items = []
for rr in rows[2:]:
    if len(rr) < len(h): continue
    try: a = int(rr[ix['Address']], 16)
    except: continue
    items.append((a, int(rr[ix['Instructions Executed']] or 0), int(rr[ix['Warp Stall Sampling (All Samples)']] or 0), rr[ix['Source']]))
items.sort(); base = items[0][0]
blocks = []; cur = None
for a, n, s, x in items:
    if cur and n == cur[1]: cur[2].append(x); cur[3] += s
    else: cur = [a, n, [x], s]; blocks.append(cur)
tot = sum(n for a, n, s, x in items); tots = sum(s for a, n, s, x in items)
print('instr/sim %.1f' % (tot / sims))
for a, n, ss, st in sorted(blocks, key=lambda b: -b[3])[:int(sys.argv[3]) if len(sys.argv) > 3 else 10]:
    c = Counter(x.split()[0] if not x.startswith('@') else x.split()[1] for x in ss)
    print(hex(a - base), 'per-sim %.3f' % (n / sims), 'len', len(ss), 'inst %.1f%% stall %.1f%%' % (n * len(ss) / tot * 100, st / tots * 100), dict(c.most_common(6)))

# --json OUT: the per-launch figures bench.py attaches to its roofline object
if '--json' in sys.argv:
    import json
    out = sys.argv[sys.argv.index('--json') + 1]
    g = {name: V0[i] for i, name in enumerate(H0)}
    f = lambda k: float(g[k]) if g.get(k) not in (None, '') else None
    rec = {'report': rep.split('/')[-1], 'kernel': g.get('Kernel Name'),
           'dram_bytes_per_launch': (f('dram__bytes_read.sum') or 0) + (f('dram__bytes_write.sum') or 0),
           'gpu_time_ms': f('gpu__time_duration.sum'),
           'issue_active_pct': f('smsp__issue_active.avg.pct_of_peak_sustained_active'),
           'alu_pipe_pct': f('sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active'),
           'fmaheavy_pipe_pct': f('sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed'),
           'warps_active_per_smsp': f('smsp__warps_active.avg.per_cycle_active'),
           'instr_per_sim': tot / sims, 'registers': f('launch__registers_per_thread')}
    json.dump(rec, open(out, 'w'), indent=1)
    print('wrote', out)
