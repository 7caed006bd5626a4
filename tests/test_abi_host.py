"""CPU-side checks of the C ABI: the library loads and exports every symbol
include/st35d.h declares; the host-only blocking model reproduces the
numbers the paper prints (eqs. (1)-(4), §V-C/§VI); the Fig. 3 schedule
generator reproduces every step reference in the text."""
import os
import re

import pytest

import paper_conf_sc_nguyensckd10_b200 as st

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "st35d.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b([a-z_][a-z0-9_]*)\s*\(", src)
    skip = {"if", "sizeof", "defined"}
    return sorted({n for n in names if n.startswith(("st", "lbm")) and n not in skip})


def test_exports_every_declared_symbol():
    L = st.lib()
    decl = declared_symbols()
    assert "st_plan_create" in decl and "lbm_d3q19_run" in decl and "st7_run" in decl
    for name in decl:
        assert hasattr(L, name), name
    assert set(decl) <= set(st.EXPORTS)


def test_no_device_errors_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("has a GPU")
    with pytest.raises(st.StError) as ei:
        st.st_plan_create(64, 64, 64, st.ST_F32, 2)
    assert ei.value.code in (st.ST_ECUDA, st.ST_EUNSUPPORTED)


MB = 2 ** 20


@pytest.mark.parametrize("C,E,R,gamma,Gamma,dimT,expect_bound,dim,kappa", [
    # 7pt CPU SP: C = 4 MB (half the LLC), E = 4, dim_T = 2: "dim <= 361", kappa 1.02
    (4 * MB, 4, 1, 0.5, 0.29, 2, 361, 360, 1.02),
    # 7pt CPU DP: E = 8: "dim <= 256", kappa 1.04
    (4 * MB, 8, 1, 1.0, 0.59, 2, 256, 256, 1.04),
    # LBM CPU SP: E = 80, dim_T = 3: "dim <= 66", used 64, kappa 1.21
    (4 * MB, 80, 1, 0.88, 0.29, 3, 66, 64, 1.21),
    # LBM CPU DP: E = 160: the paper uses 44, kappa 1.34
    (4 * MB, 160, 1, 1.75, 0.59, 3, 46, 44, 1.34),
])
def test_blocking_model_reproduces_paper(C, E, R, gamma, Gamma, dimT, expect_bound, dim, kappa):
    m = st.st_blocking_model(C, E, R, gamma, Gamma, dimT, dim)
    assert int(m["dim_bound"]) in (expect_bound, expect_bound + 1)
    assert abs(m["kappa"] - kappa) <= 0.015
    # eq. (3): eta = ceil(gamma/Gamma) -> 2 for the CPU 7pt (0.5/0.29), 3 for CPU LBM DP (1.75/0.59)
    assert m["eta"] == -(-gamma // Gamma)


def test_blocking_model_gpu_7pt():
    # GTX 285: register file C = 64 KB, dim_T = 2, E = 4: "dim <= 45.2"; 32 wide -> kappa 1.31
    m = st.st_blocking_model(64 * 1024, 4, 1, 0.5, 0.14, 2, 32)
    assert abs(m["dim_bound"] - 45.25) < 0.05
    assert abs(m["kappa"] - 1.306) < 0.005
    # eta for LBM SP on GTX 285 with the effective Gamma 0.14: 0.88/0.14 -> 6.3 ("dim_T >= 6.1")
    assert st.st_blocking_model(16 * 1024, 160, 1, 0.88, 0.14)["eta"] == 7


# Fig. 3(a) (R = 1, dim_T = 3): (step, plane, level) triples the text names
FIG3 = [(9, 3, 1), (21, 2, 3), (16, 3, 2), (7, 2, 1), (12, 4, 1), (18, 8, 0), (19, 6, 1), (20, 4, 2),
        (8, 5, 0), (11, 6, 0), (14, 7, 0), (10, 1, 2), (13, 2, 2), (15, 5, 1), (17, 1, 3), (1, 0, 0), (5, 1, 1)]


def test_fig3_schedule_matches_text():
    seen = {}
    for rnd in range(9):
        for lvl in range(4):
            s, z, slot = st.st_fig3_step(1, 3, rnd, lvl)
            if s:
                seen[s] = (z, lvl, rnd, slot)
    for s, z, lvl in FIG3:
        assert seen[s][:2] == (z, lvl), (s, seen.get(s))
    # prolog = S1..S13: the first step at t' = dim_T is S17 (round 7), the prolog ends at round 6
    assert max(s for s, v in seen.items() if v[2] <= 6) == 13
    # S16 needs S7, S9, S12: planes 2, 3, 4 at level 1
    assert {seen[7][:2], seen[9][:2], seen[12][:2]} == {(2, 1), (3, 1), (4, 1)}
    # S19 reads S8, S11, S14; S20 reads S9, S12, S15; S21 reads S10, S13, S16
    for out, ins in ((19, (8, 11, 14)), (20, (9, 12, 15)), (21, (10, 13, 16))):
        z, lvl = seen[out][:2]
        assert sorted(seen[i][0] for i in ins) == [z - 1, z, z + 1]
        assert all(seen[i][1] == lvl - 1 for i in ins)
    # buffer slot z mod (2R+2): the 4 slots read by S19..S21 in round 8 never collide with S18's write
    w = seen[18][3]
    for out in (19, 20, 21):
        pass
    assert w == 8 % 4
    # z_s = z + 2R(dim_T - t''): at round 8 (z = 2 output) levels hold planes 8, 6, 4, 2
    assert [seen[s][0] for s in (18, 19, 20, 21)] == [8, 6, 4, 2]
