"""Stall samples of an ncu source-page CSV (SASS) summed over address regions:
python tools/src_regions.py file.src.csv name:start:end ... (hex offsets from the kernel start)"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
ix = {k: i for i, k in enumerate(h)}
base = int(rows[2][0], 16)
regs = [(a.split(':')[0], int(a.split(':')[1], 16), int(a.split(':')[2], 16)) for a in sys.argv[2:]]
keys = [k for k in h if k.startswith('stall_') and 'Not Issued' not in k]
tot = {r[0]: {k: 0 for k in keys + ['samples', 'inst']} for r in regs}
allsum = 0
for r in rows[2:]:
    try:
        off = int(r[0], 16) - base
    except ValueError:
        continue
    s = int(r[ix['# Samples']] or 0); allsum += s
    for name, a, b in regs:
        if a <= off < b:
            t = tot[name]; t['samples'] += s; t['inst'] += int(r[ix['Instructions Executed']] or 0)
            for k in keys:
                t[k] += int(r[ix[k]] or 0)
print('total samples', allsum)
for name, t in tot.items():
    top = sorted(((v, k) for k, v in t.items() if k.startswith('stall_')), reverse=True)[:7]
    print(f"{name:10s} samples {t['samples']:7d} ({100*t['samples']/allsum:5.1f}%) warp-inst {t['inst']:9d}  " +
          "  ".join(f"{k[6:]} {v}" for v, k in top))
