"""Host-side checks of the C-ABI library (no GPU): it loads, exports every
symbol include/up.h declares, sizes limbs as the paper's table says, formats
results canonically, and its specialiser emits CUDA that NVRTC compiles for
sm_100a (register/spill report checked for the hot narrow kernels)."""
import os
import random
import re

import pytest

from paper_conf_icde_lixylz24_b200 import up

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "up.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(up_[a-z0-9_]+)\s*\(", src)))


def test_library_loads_and_exports_every_declared_symbol():
    L = up.lib()
    names = header_functions()
    assert len(names) >= 25
    for n in names:
        assert hasattr(L, n), n
    assert set(names) <= set(up.EXPORTS)


def test_limb_table_matches_paper():
    """result precisions 18/38/76/153/307 <-> LEN 2/4/8/16/32
    (reading Q1: exact for the sign-bit rule 10^p <= 2^(32L-1))."""
    for p, L in [(18, 2), (38, 4), (76, 8), (153, 16), (307, 32)]:
        assert up.limbs(p) == L
        assert up.limbs(p + 1) == L + 1
    for p in range(1, 400):
        L = up.limbs(p)
        assert 10 ** p <= 2 ** (32 * L - 1) and (L == 1 or 10 ** p > 2 ** (32 * (L - 1) - 1))


def test_sum_precision_rule():
    assert up.sum_precision(18, 1_000_000) == 24
    assert up.sum_precision(36, 10_000_000) == 43
    assert up.sum_precision(36, 10_000_001) == 44
    assert up.sum_precision(36, 1) == 36
    assert up.ld_for(5) == 8 and up.ld_for(8) == 8 and up.ld_for(0) == 0


def test_format_decimal_canonical():
    rng = random.Random(3)
    for _ in range(200):
        n = rng.randint(1, 6)
        v = rng.randrange(-(2 ** (32 * n - 1)), 2 ** (32 * n - 1))
        s = rng.randint(0, 30)
        limbs = [(v >> (32 * j)) & 0xFFFFFFFF for j in range(n)]
        want = ("-" if v < 0 else "") + (lambda a: a if s == 0 else a[:-s] + "." + a[-s:])(str(abs(v)).rjust(s + 1, "0"))
        assert up.format_decimal(limbs, s) == want
    assert up.format_decimal([0, 0], 3) == "0.000"


def test_expression_typing_on_host():
    """up_expr_type runs on the host (no GPU): the paper's rules."""
    src = up.gen_source("eval", "c1*c2 - c3/c4", [(200, 50)] * 4, 100)
    assert "type (401,100)" in src
    assert "type (18,5) L=2" in up.gen_source("sum", "c1+c2", [(17, 5), (14, 2)], 10)
    assert "type (36,5) L=4" in up.gen_source("sum", "c1+c2", [(35, 5), (32, 2)], 10)
    with pytest.raises(up.UpError) as ei:
        up.gen_source("eval", "c1 % c2", [(10, 2), (10, 0)], 10)
    assert ei.value.name == "INVAL"
    with pytest.raises(up.UpError):
        up.gen_source("eval", "c1 + c3", [(10, 2), (10, 0)], 10)
    with pytest.raises(up.UpError):
        up.gen_source("eval", "c1 + ", [(10, 2)], 10)


def _regs(log):
    m = re.search(r"Used (\d+) registers", log)
    sp = re.search(r"(\d+) bytes spill stores", log)
    return int(m.group(1)), int(sp.group(1)) if sp else 0


@pytest.mark.parametrize("variant,expr,types", [
    ("sum", "c1+c2", [(17, 5), (14, 2)]),
    ("sum", "c1+c2", [(35, 5), (32, 2)]),
    ("eval", "c1+c2", [(35, 5), (32, 2)]),
    ("sum", "c1*c2 - c3/c4", [(30, 10)] * 4),
    ("eval", "c1 % c2 * c1 % c2", [(40, 0), (41, 0)]),
    ("sum", "-c1/(c2+0.5)", [(12, 3), (9, 2)]),
])
def test_specialised_kernels_compile_for_sm100a(variant, expr, types, tmp_path):
    src = up.gen_source(variant, expr, types, 1_000_000)
    log = up.nvrtc_compile(src, str(tmp_path / "k.cubin"))
    regs, spills = _regs(log)
    assert (tmp_path / "k.cubin").stat().st_size > 0
    if expr == "c1+c2":
        assert spills == 0 and regs <= 64, log


def test_group_aggregate_typing_and_kernel_compile(tmp_path):
    """NEXT-4: aggregate typing on the host and the generated
    grouped-aggregation kernel compiles for sm_100a without spills."""
    t = [(12, 2), (12, 2), (3, 2), (3, 2)]
    N = 60_000_000
    assert up.agg_type("SUM", "c1", t, N)[:2] == (12 + 8, 2)
    assert up.agg_type("MIN", "c2*(1-c3)", t, N)[:2] == up.agg_type("MAX", "c2*(1-c3)", t, N)[:2]
    p, s, _ = up.agg_type("SUM", "c2*(1-c3)", t, N)
    assert up.agg_type("MAX", "c2*(1-c3)", t, N)[:2] == (p - 8, s)
    assert up.agg_type("AVG", "c3", t, N)[:2] == (3 + 4, 2 + 4)
    aggs = [("SUM", "c1"), ("AVG", "c2*(1-c3)*(1+c4)"), ("MIN", "c1-c2"), ("MAX", "c3")]
    src = up.gen_group_agg_source(aggs, t, 4, N)
    log = up.nvrtc_compile(src, str(tmp_path / "g.cubin"))
    regs, spills = _regs(log)
    assert spills == 0, log


def test_tpi_kernels_compile_for_sm100a():
    """Every per-operator TPI kernel shape (NEXT-3) compiles with NVRTC for sm_100a (no GPU)."""
    from paper_conf_icde_lixylz24_b200 import up
    for op in "+-*":
        for tpi in (1, 2, 4, 8, 16, 32):
            for types, cp in (([(35, 5), (32, 2)], None), ([(153, 7), (154, 0)], [True, False])):
                up.nvrtc_compile(up.gen_tpi_source(op, types, tpi, compact=cp))
    for alg in ("long", "newton"):
        for types in ([(40, 5), (30, 2)], [(200, 50), (200, 50)], [(20, 0), (9, 0)]):
            up.nvrtc_compile(up.gen_tpi_source("/", types, 1, alg))


@pytest.mark.parametrize("variant,expr,types,layouts", [
    ("sum", "c1+c2", [(17, 5), (14, 2)], ["quads", "quads"]),                  # 4 rows per thread, 16-byte quad loads
    ("sum", "c1/c2", [(200, 50)] * 2, ["quads", "quads"]),                     # top-limb window from quads, out-of-line fallback
    ("eval", "c1*c2 - c3/c4", [(200, 50)] * 4, ["quads", "planes", "compact", "quads"]),
])
def test_quad_layout_kernels_compile_for_sm100a(variant, expr, types, layouts, tmp_path):
    """limb-quad columns (up.h UP_LAYOUT_QUADS): the generated kernels read
    them with 16-byte loads and compile for sm_100a; the division's decision
    window loads whole quads and its full-division fallback is out of line"""
    src = up.gen_source(variant, expr, types, 1_000_000, layouts=layouts)
    assert "ld_quads<" in src or "ld_issue4(g" in src
    if expr == "c1/c2":   # both division operands are columns read lazily: fallback out of line
        assert "__noinline__" in src and "div_top_decide<" in src
    log = up.nvrtc_compile(src, str(tmp_path / "q.cubin"))
    assert (tmp_path / "q.cubin").stat().st_size > 0, log
    if expr == "c1+c2":
        regs, spills = _regs(log)
        assert spills == 0 and regs <= 64, log


def test_quads_abi():
    """up_quads(p) = ceil((up_limbs(p) + 1) / 4): the sign-flag limb included"""
    for p in (1, 9, 18, 38, 76, 153, 200, 307, 1000):
        assert up.quads(p) == (up.limbs(p) + 1 + 3) // 4
