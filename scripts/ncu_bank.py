"""Attribute shared-memory bank conflicts to SASS instructions from an
ncu --set full --import-source on report:

    python scripts/ncu_bank.py gpurun_out/prof_tlc22.ncu-rep [--out profiles/x.md]

Per kernel in the report: every SASS instruction with shared-memory wavefronts, its
ideal and excessive wavefronts (ncu's per-instruction "L1 Wavefronts Shared
Excessive"), and the kernel totals split by instruction class (LDS / STS / other, e.g.
the TMA unit's UTMA*/UBLKCP shared accesses do not appear as instructions), next to the
kernel-level l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_{ld,st} counters.
"""
import argparse, csv, io, subprocess, sys
from collections import defaultdict

ap = argparse.ArgumentParser()
ap.add_argument('rep')
ap.add_argument('--out', default='')
a = ap.parse_args()

src = subprocess.run(['ncu', '-i', a.rep, '--page', 'source', '--csv'], capture_output=True, text=True).stdout
raw = subprocess.run(['ncu', '-i', a.rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout

kernels = []          # (name, rows)
cur = None
hdr = None
for line in src.splitlines():
    if line.startswith('"Kernel Name"'):
        name = next(csv.reader(io.StringIO(line)))[1]
        cur = (name, [])
        kernels.append(cur)
        hdr = None
        continue
    if cur is None:
        continue
    row = next(csv.reader(io.StringIO(line)))
    if hdr is None:
        hdr = {h: i for i, h in enumerate(row)}
        continue
    cur[1].append((hdr, row))

# kernel-level counters (raw page: one row per launch)
rrows = list(csv.reader(io.StringIO(raw)))
rh = {h: i for i, h in enumerate(rrows[0])} if rrows else {}
klevel = []
for r in rrows[2:]:
    if len(r) < len(rh):
        continue
    def g(m):
        try:
            return float(r[rh[m]].replace(',', ''))
        except (KeyError, ValueError):
            return None
    klevel.append((r[rh['Kernel Name']],
                   g('l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum'),
                   g('l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum'),
                   g('l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum'),
                   g('l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum'),
                   g('gpu__time_duration.sum')))

lines = [f"# Shared-memory bank conflicts by SASS instruction: `{a.rep}`", ""]
seen = defaultdict(int)
for ki, (name, rows) in enumerate(kernels):
    seen[name] += 1
    short = name.replace('void perm::<unnamed>::', '').split('(perm')[0].split('(CUtensor')[0]
    tot = defaultdict(lambda: [0, 0, 0])   # class -> [wavefronts, ideal, excessive]
    hot = []
    for h, r in rows:
        def f(col):
            try:
                return float(r[h[col]].replace(',', ''))
            except (KeyError, ValueError):
                return 0.0
        wf = f('L1 Wavefronts Shared')
        if wf <= 0:
            continue
        sass = r[h['Source']].strip()
        op = sass.split()[0] if sass else '?'
        if op.startswith('@'):
            op = sass.split()[1]
        cls = 'LDS' if op.startswith('LDS') else ('STS' if op.startswith('STS') else 'other')
        ideal, exc = f('L1 Wavefronts Shared Ideal'), f('L1 Wavefronts Shared Excessive')
        t = tot[cls]
        t[0] += wf; t[1] += ideal; t[2] += exc
        hot.append((exc, wf, ideal, r[h['Address']], sass))
    lines.append(f"## {short} (launch {seen[name]})")
    lines.append("")
    lines.append("| class | wavefronts | ideal | excessive |")
    lines.append("|---|---|---|---|")
    for cls in ('LDS', 'STS', 'other'):
        t = tot.get(cls)
        if t:
            lines.append(f"| {cls} | {t[0]:.0f} | {t[1]:.0f} | {t[2]:.0f} |")
    if ki < len(klevel):
        k = klevel[ki]
        lines.append("")
        lines.append(f"kernel counters: l1tex bank conflicts ld {k[1]:.0f}, st {k[2]:.0f}; LSU shared-pipe "
                     f"wavefronts ld {k[3]:.0f}, st {k[4]:.0f}; duration {k[5]} us")
        ldi = tot.get('LDS', [0, 0, 0])[0]
        sti = tot.get('STS', [0, 0, 0])[0]
        lines.append(f"LSU wavefronts not issued by LDS / STS instructions (mbarrier SYNCS arrivals and "
                     f"try-waits, fences): ld {k[3] - ldi:.0f}, st {k[4] - sti:.0f}")
    lines.append("")
    lines.append("top instructions by excessive wavefronts:")
    lines.append("")
    lines.append("| excessive | wavefronts | ideal | address | SASS |")
    lines.append("|---|---|---|---|---|")
    for exc, wf, ideal, addr, sass in sorted(hot, reverse=True)[:8]:
        lines.append(f"| {exc:.0f} | {wf:.0f} | {ideal:.0f} | {addr[-5:]} | `{sass}` |")
    lines.append("")
text = "\n".join(lines)
print(text)
if a.out:
    open(a.out, 'w').write(text + "\n")
