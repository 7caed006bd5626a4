"""A/B timing of library builds: python tools/ab.py LIB[=label] ... (ST35D_LIB per run, subprocess each)
Each case: one warm call then best of 3 timed st7_run calls (CUDA events)."""
import os, subprocess, sys, json
CASES = os.environ.get("AB_CASES", "256:f32:3,256:f32:4,512:f32:4,256:f64:3").split(",")
code = r'''
import sys, json, torch
sys.path.insert(0, '.')
import paper_conf_sc_nguyensckd10_b200 as st
out = {}
import stgen
for c in sys.argv[1].split(","):
    if c.startswith("lbm"):
        _, n, dt, D = c.split(":"); n = int(n); D = int(D)
        t = torch.float32 if dt == "f32" else torch.float64
        fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
        f = torch.from_numpy(stgen.lbm_rest(n, n, n, "float32" if dt == "f32" else "float64")).cuda(); g = torch.empty_like(f)
        p = st.Plan(n, n, n, t, D); s = torch.cuda.Stream(); p.set_stream(s.cuda_stream)
        T = 20
        p.lbm(f, g, 1.6, T, fl); p.sync()
        best = 1e9
        for _ in range(3):
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(); e0.record(s); p.lbm(f, g, 1.6, T, fl); e1.record(s); torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1))
        out[c] = round((n - 2) ** 3 * T / best / 1e6, 1)
        p.close(); del f, g
        continue
    n, dt, D = c.split(":"); n = int(n); D = int(D)
    t = torch.float32 if dt == "f32" else torch.float64
    p = st.Plan(n, n, n, t, D)
    s = torch.cuda.Stream(); p.set_stream(s.cuda_stream)
    x = torch.rand(n, n, n, dtype=t, device="cuda"); y = torch.empty_like(x)
    T = 100 if 100 % D == 0 else 99 if D == 3 else 100 - 100 % D
    p.st7(x, y, 0.4, 0.1, T); p.sync()
    best = 1e9
    for _ in range(3):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); e0.record(s); p.st7(x, y, 0.4, 0.1, T); e1.record(s); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    out[c] = round((n - 2) ** 3 * T / best / 1e6, 1)
    p.close()
print(json.dumps(out))
'''
res = {}
for a in sys.argv[1:]:
    lib, _, label = a.partition("=")
    env = dict(os.environ)
    if lib != "default":
        env["ST35D_LIB"] = lib
    r = subprocess.run([sys.executable, "-c", code, ",".join(CASES)], env=env, capture_output=True, text=True)
    res[label or lib] = json.loads(r.stdout.strip().splitlines()[-1]) if r.returncode == 0 else r.stderr[-500:]
    print(label or lib, res[label or lib], flush=True)
