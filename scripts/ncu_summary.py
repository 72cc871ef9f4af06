"""Summarise ncu outputs (launch list CSV + --set full report) into profiles/.

    python scripts/ncu_summary.py --launches gpurun_out/launches_r01.csv \
        --full gpurun_out/ncu_full_r01.ncu-rep --out profiles/r01
"""
import argparse, csv, io, json, statistics, subprocess
from collections import defaultdict

ap = argparse.ArgumentParser()
ap.add_argument('--launches')
ap.add_argument('--full')
ap.add_argument('--out', required=True)
ap.add_argument('--only', help="regex: keep only matching kernels in the launch table (e.g. the apply's kernels)")
ap.add_argument('--traffic-key', help="also write profiles/ncu_traffic.json[key] = per-pass DRAM bytes")
a = ap.parse_args()
summary = {}
if a.launches:
    rows = list(csv.reader(open(a.launches)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == 'ID')
    hdr = rows[start]
    ix = {h: i for i, h in enumerate(hdr)}
    per = defaultdict(dict)
    for r in rows[start + 1:]:
        if len(r) < len(hdr):
            continue
        per[r[ix['ID']]]['name'] = r[ix['Kernel Name']]
        v = r[ix['Metric Value']].replace(',', '')
        try:
            v = float(v)
        except ValueError:
            pass
        unit = r[ix['Metric Unit']]
        if unit in ('Kbyte',): v *= 1e3
        if unit in ('Mbyte',): v *= 1e6
        if unit in ('Gbyte',): v *= 1e9
        if unit in ('usecond',): v *= 1e3
        if unit in ('msecond',): v *= 1e6
        per[r[ix['ID']]][r[ix['Metric Name']]] = v
    agg = defaultdict(lambda: defaultdict(list))
    for d in per.values():
        nm = d['name'].split('(')[0].replace('void ', '')[:90]
        if a.only and not __import__('re').search(a.only, nm):
            continue
        for k, v in d.items():
            if k != 'name' and isinstance(v, float):
                agg[nm][k].append(v)
    tot = sum(sum(v.get('gpu__time_duration.sum', [0])) for v in agg.values())
    lines = ['| kernel | launches | mean ns | share of GPU time | mean DRAM read MB | mean DRAM write MB |', '|---|---|---|---|---|---|']
    ks = {}
    for nm, m in sorted(agg.items(), key=lambda x: -sum(x[1].get('gpu__time_duration.sum', [0]))):
        t = m.get('gpu__time_duration.sum', [0])
        rd = m.get('dram__bytes_read.sum', [0]); wr = m.get('dram__bytes_write.sum', [0])
        ks[nm] = {'launches': len(t), 'mean_ns': statistics.mean(t), 'share': sum(t) / tot,
                  'dram_read_B': statistics.mean(rd), 'dram_write_B': statistics.mean(wr)}
        lines.append(f"| `{nm}` | {len(t)} | {statistics.mean(t):.0f} | {sum(t)/tot:.1%} | {statistics.mean(rd)/1e6:.2f} | {statistics.mean(wr)/1e6:.2f} |")
    summary['launches'] = ks
    open(a.out + '_launches.md', 'w').write('\n'.join(lines) + '\n')
if a.full:
    raw = subprocess.run(['ncu', '-i', a.full, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    keys = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
            'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'lts__t_bytes.sum',
            'l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum',
            'l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum',
            'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum', 'smsp__inst_executed.sum',
            'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
            'launch__grid_size', 'launch__block_size', 'sm__cycles_active.avg']
    kern = []
    for vals in rows[2:]:
        d = dict(zip(hdr, vals))
        u = dict(zip(hdr, units))
        e = {'kernel': d.get('Kernel Name', '')[:120]}
        for k in keys:
            if k in d:
                e[k] = f"{d[k]} {u.get(k, '')}".strip()
        stalls = []
        for h, v in d.items():
            if 'average_warps_issue_stalled' in h and h.endswith('per_issue_active.ratio'):
                try:
                    stalls.append((float(v), h.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', '')))
                except ValueError:
                    pass
        e['top_stalls'] = {n: round(v, 2) for v, n in sorted(stalls, reverse=True)[:6]}
        kern.append(e)
    summary['full'] = kern
    if a.traffic_key:
        import os, re
        tp = os.path.join(os.path.dirname(os.path.abspath(__file__)), '..', 'profiles', 'ncu_traffic.json')
        tj = json.load(open(tp)) if os.path.exists(tp) else {}
        ent = {}
        for e in kern:
            m = re.search(r'row_pass_tlc_kernel<(\d+), (\d+)', e['kernel'])
            if not m:
                continue
            kind = {'1': 'R1', '2': 'R2', '0': 'R3'}[m.group(2)]
            def num(x):
                v, u = x.split(' ', 1) if ' ' in x else (x, '')
                v = float(v.replace(',', ''))
                return v * {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}.get(u.strip(), 1)
            ent[kind] = num(e['dram__bytes_read.sum']) + num(e['dram__bytes_write.sum'])
        tj[a.traffic_key] = ent
        json.dump(tj, open(tp, 'w'), indent=1)
    with open(a.out + '_ncu_full.md', 'w') as f:
        f.write('# ncu --set full (cold caches, serialized replay)\n\n')
        for e in kern:
            f.write(f"## {e['kernel']}\n\n")
            for k, v in e.items():
                if k not in ('kernel',):
                    f.write(f"- {k}: {v}\n")
            f.write('\n')
json.dump(summary, open(a.out + '_ncu.json', 'w'), indent=1)
print(open(a.out + '_launches.md').read() if a.launches else '')
