"""instruction mix (executed warp instructions by opcode) and top stall lines from an
ncu --page source --csv --print-source sass export: python tools/sass_mix.py file.csv [N]"""
import csv, sys, collections, re
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
mix = collections.Counter(); stall = []
tot = 0
for r in rows[2:]:
    if len(r) < len(hdr): continue
    src = r[ix["Source"]]
    try: n = int(r[ix["Instructions Executed"]] or 0)
    except ValueError: continue
    op = re.sub(r'^@!?U?P\w+\s+', '', src.strip()).split(' ')[0]
    base = op.split('.')[0]
    mix[base] += n; tot += n
    s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    stall.append((s, r[ix["Address"]], src.strip()[:70], n))
print("total warp instructions", tot)
for k, v in mix.most_common(30):
    print(f"{k:10s} {v:12d} {v/tot*100:6.2f}%")
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
print("top stall-sampled instructions:")
for s, a, src, n in sorted(stall, reverse=True)[:N]:
    print(f"{s:7d} {a:>6s} {n:9d}  {src}")
