"""side-by-side of ncu --page details csv files: python tools/ncu_cmp.py a.details.csv b.details.csv ..."""
import csv, sys
SECT = ('GPU Speed Of Light Throughput', 'Compute Workload Analysis', 'Occupancy', 'Warp State Statistics',
        'Memory Workload Analysis', 'Launch Statistics', 'Scheduler Statistics')
tabs = []
for fn in sys.argv[1:]:
    rows = list(csv.reader(open(fn)))
    h = rows[0]
    d = {}
    for r in rows[1:]:
        x = dict(zip(h, r))
        if x.get('Section Name') in SECT and x.get('Metric Name'):
            d[(x['Section Name'][:12], x['Metric Name'])] = x['Metric Value'] + ' ' + x.get('Metric Unit', '')
    tabs.append(d)
for k in tabs[0]:
    vals = [t.get(k, '-') for t in tabs]
    print(f"{k[0]:12s} | {k[1][:40]:40s} | " + " | ".join(f"{v:>18s}" for v in vals))
