"""registers / stack per kernel of the built objects: python tools/regs.py [pattern]"""
import re, subprocess, sys, glob
pat = sys.argv[1] if len(sys.argv) > 1 else ''
for o in sorted(glob.glob('build/obj/*.o')):
    out = subprocess.run(['cuobjdump', '--dump-resource-usage', o], capture_output=True, text=True).stdout
    fn = None
    for line in out.splitlines():
        m = re.search(r'Function (\S+):', line)
        if m: fn = m.group(1); continue
        m = re.search(r'REG:(\d+) STACK:(\d+)', line)
        if m and fn and pat in fn:
            d = subprocess.run(['c++filt', fn], capture_output=True, text=True).stdout.strip()
            d = re.sub(r'\(.*', '', d).replace('st35d::', '')
            print(f"{o.split('/')[-1]:18s} REG {m.group(1):>3s} STACK {m.group(2):>5s}  {d}")
