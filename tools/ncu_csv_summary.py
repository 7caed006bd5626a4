"""Summarise `ncu --metrics ... --csv` outputs (one kernel launch each) as a markdown table:
python tools/ncu_csv_summary.py label=file.csv ..."""
import csv, sys, io
rows = []
for arg in sys.argv[1:]:
    label, _, fn = arg.partition('=')
    txt = open(fn).read()
    lines = [l for l in txt.splitlines() if l.startswith('"')]
    rdr = csv.DictReader(io.StringIO("\n".join(lines)))
    m = {}
    for r in rdr:
        m[r['Metric Name']] = (r['Metric Value'], r.get('Metric Unit', ''))
        m['_kernel'] = (r.get('Kernel Name', '')[:60], '')
    rows.append((label, m))
keys = [k for k in rows[0][1] if not k.startswith('_')]
print("| metric | " + " | ".join(l for l, _ in rows) + " |")
print("|---|" + "---|" * len(rows))
for k in keys:
    vals = []
    for _, m in rows:
        v, u = m.get(k, ('-', ''))
        vals.append(f"{v} {u}".strip())
    print(f"| {k} | " + " | ".join(vals) + " |")
print()
for l, m in rows:
    print(f"- {l}: `{m.get('_kernel', ('',''))[0]}`")
