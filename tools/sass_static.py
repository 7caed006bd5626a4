"""static opcode counts of one kernel in a built object:
python tools/sass_static.py build/obj/st7_f32_fast.o '<float, 3, 16, 4, false, 256, 1>'"""
import re, subprocess, sys, collections
obj, pat = sys.argv[1], sys.argv[2]
out = subprocess.run(['cuobjdump', '-sass', obj], capture_output=True, text=True).stdout
funcs = re.split(r'\n\s+Function : ', out)
for f in funcs[1:]:
    name = f.split('\n', 1)[0].strip()
    dem = subprocess.run(['c++filt', name], capture_output=True, text=True).stdout.strip()
    if pat not in dem:
        continue
    ops = collections.Counter()
    for line in f.split('\n'):
        m = re.match(r'\s+/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)', line)
        if m: ops[m.group(2)] += 1
    tot = sum(ops.values())
    print(dem[:90], 'total', tot)
    print('  '.join(f"{k}:{v}" for k, v in ops.most_common(24)))
