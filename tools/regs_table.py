"""REG/STACK per st7/st13 kernel of a built library: python tools/regs_table.py [lib]"""
import re, subprocess, sys
lib = sys.argv[1] if len(sys.argv) > 1 else 'paper_conf_sc_nguyensckd10_b200/libst35d.so'
out = subprocess.run(['cuobjdump', '-res-usage', lib], capture_output=True, text=True).stdout
name = None
for line in out.splitlines():
    m = re.search(r'Function (\S+):', line)
    if m:
        name = m.group(1); continue
    m = re.search(r'REG:(\d+) STACK:(\d+)', line)
    if m and name and ('st7_35d' in name or 'st13' in name):
        t = re.search(r'kernelI(.)((?:Li\d+E|Lb\dE)+)', name)
        args = re.findall(r'L[ib](\d+)E', t.group(2)) if t else []
        print(f"{'st13' if 'st13' in name else 'st7 '} {t.group(1) if t else '?'} {' '.join(args):28s} REG {m.group(1):>3} STACK {m.group(2)}")
