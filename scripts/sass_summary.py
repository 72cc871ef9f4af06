"""Per-kernel SASS instruction-class summary of libperm.so (no GPU needed): proves the
Blackwell data-movement path (TMA bulk / tensor copies UBLKCP / UTMASTG / UTMALDG, bulk
L2 prefetch UBLKPF, mbarrier SYNCS, DSMEM) and shows each kernel's shared / global
access mix. Static instruction counts (one per SASS line), not dynamic.

    python scripts/sass_summary.py [--out profiles/r02_sass_summary.md]
"""
import argparse, os, re, subprocess, sys
from collections import Counter, OrderedDict

ap = argparse.ArgumentParser()
ap.add_argument('--lib', default=os.path.join(os.path.dirname(__file__), '..', 'paper_conf_icpp_kasagini13_b200', 'libperm.so'))
ap.add_argument('--out', default='')
a = ap.parse_args()

sass = subprocess.run(['cuobjdump', '-sass', a.lib], capture_output=True, text=True).stdout
names = subprocess.run(['cu++filt'], input='\n'.join(re.findall(r'Function : (\S+)', sass)),
                       capture_output=True, text=True).stdout.split('\n')

CLASSES = OrderedDict([
    ('TMA bulk copy (UBLKCP)', r'^UBLKCP'),
    ('TMA bulk prefetch L2 (UBLKPF)', r'^UBLKPF'),
    ('TMA tensor store (UTMASTG)', r'^UTMASTG'),
    ('TMA tensor load (UTMALDG)', r'^UTMALDG'),
    ('bulk group commit/wait (UTMACMDFLUSH, DEPBAR)', r'^(UTMACMDFLUSH|DEPBAR)'),
    ('mbarrier / sync unit (SYNCS)', r'^SYNCS'),
    ('cluster barrier (UCGABAR)', r'^UCGABAR'),
    ('CTA barrier (BAR)', r'^BAR'),
    ('shared load (LDS)', r'^LDS'),
    ('shared store (STS)', r'^STS'),
    ('DSMEM / generic-window store (ST.E / STAS)', r'^(STAS|ST\.)'),
    ('global load (LDG)', r'^LDG'),
    ('global store (STG)', r'^STG'),
    ('atomics / reductions (ATOMG, RED)', r'^(ATOMG|RED|ATOM)'),
    ('proxy / memory fences (FENCE, MEMBAR, CCTL)', r'^(FENCE|MEMBAR|CCTL)'),
    ('funnel shift / bit field (SHF, BMSK, LOP3)', r'^(SHF|BMSK|LOP3)'),
    ('tensor core (HMMA / UTC*MMA)', r'^(HMMA|UTC\w*MMA)'),
])

blocks = re.split(r'\n\s+Function : ', sass)[1:]
rows = []
for blk, dem in zip(blocks, names):
    mangled = blk.split('\n', 1)[0].strip()
    ops = Counter()
    for line in blk.split('\n'):
        m = re.match(r'\s+/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)', line)
        if m:
            ops[m.group(1)] += 1
    total = sum(ops.values())
    cls = OrderedDict()
    for nm, rx in CLASSES.items():
        cls[nm] = sum(v for k, v in ops.items() if re.match(rx, k))
    short = dem.replace('perm::(anonymous namespace)::', '').strip() or mangled
    rows.append((short, total, cls))

kernels_of_interest = ('row_pass_tlc_kernel', 'cluster_kernel', 'row_pass_tma_kernel', 'row_pass_split_stg_kernel',
                       'row_pass_split_kernel', 'transpose64_kernel', 'transpose_kernel', 'fused_kernel',
                       'fused_tlc_kernel', 'row_pass_kernel', 'scatter_kernel', 'gather_kernel',
                       'block_gather_kernel', 'copy_kernel')
lines = ["# SASS instruction classes per kernel (static counts, `cuobjdump -sass libperm.so`)", "",
         "sm_100a; one row per kernel instantiation. TMA = UBLKCP (cp.async.bulk), UTMASTG / UTMALDG",
         "(cp.async.bulk.tensor), UBLKPF (cp.async.bulk.prefetch.L2); SYNCS = mbarrier operations;",
         "no tensor-core instructions anywhere (pure data movement).", ""]
hdr = ['kernel', 'SASS'] + [k.split(' (')[0] for k in CLASSES]
lines.append('| ' + ' | '.join(hdr) + ' |')
lines.append('|' + '---|' * len(hdr))
for short, total, cls in sorted(rows):
    if not any(k in short for k in kernels_of_interest):
        continue
    nm = re.sub(r'\((int|bool)\)', '', short.replace('void ', '').replace('perm::<unnamed>::', '')).split('(')[0]
    lines.append('| `' + nm[:80] + '` | ' + str(total) + ' | ' + ' | '.join(str(v) for v in cls.values()) + ' |')
text = '\n'.join(lines)
print(text)
if a.out:
    open(a.out, 'w').write(text + '\n')
