"""C-ABI boundary checks that need no GPU (-m "not gpu"): the library loads, exports
every symbol include/smiless.h declares, validates arguments (T6), decodes indices,
and NVRTC specialises the evaluator for every BASELINE config (sm_100a, no spills).
"""
import ctypes
import re
import os

import numpy as np
import pytest

import workloads as W
from paper_conf_sc_luxl0y024_b200 import smiless as S

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "smiless.h")).read()
    return sorted(set(re.findall(r"SMILESS_API\s+[\w\s\*]+?\b(smiless_\w+)\s*\(", txt)))


def test_library_exports_every_header_symbol():
    lib = S.load_library()
    syms = header_symbols()
    assert len(syms) >= 10
    assert sorted(S.EXPORTS) == syms
    for name in syms:
        assert hasattr(lib, name), name


def test_library_has_no_cpu_fallback_dependency():
    """The product library links no oracle code and no CPU evaluator."""
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", S.LIB_PATH], capture_output=True, text=True).stdout
    assert "oracle" not in out
    src = open(os.path.join(ROOT, "paper_conf_sc_luxl0y024_b200", "smiless.py")).read()
    assert "oracle" not in src.lower().replace("no cpu fallback", "")


def planner(prob=None):
    prob = prob or W.make_config("C1")
    return S.planner_for(prob), prob


def test_create_rejects_bad_args():
    lib = S.load_library()
    ctx = ctypes.c_void_p()
    assert lib.smiless_create(None, 0, None) == S.EINVAL
    assert lib.smiless_create(ctypes.byref(ctx), -1, None) == S.EINVAL
    assert b"cuda_device" in lib.smiless_last_error(None)


def test_load_dag_validation():
    pl = S.Planner()
    with pytest.raises(S.SmilessError) as e:
        pl.load_dag([0, 0, 1], [1])          # function 1 lists itself
    assert e.value.code == S.ENOTTOPO
    with pytest.raises(S.SmilessError) as e:
        pl.load_dag([0, 1, 1], [0])          # function 0 lists 0 -> not topological
    assert e.value.code == S.ENOTTOPO
    with pytest.raises(S.SmilessError) as e:
        pl.load_dag([0, 0, 2], [0, 0])       # duplicate predecessor
    assert e.value.code == S.EINVAL
    with pytest.raises(S.SmilessError) as e:
        pl.load_dag([0, 0, 1], [5])
    assert e.value.code == S.EINVAL
    with pytest.raises(S.SmilessError) as e:
        pl.load_dag([1, 1], [])
    assert e.value.code == S.EINVAL
    with pytest.raises(S.SmilessError) as e:
        pl.load_dag([0] * 40, [])            # > SMILESS_MAX_FUNCS
    assert e.value.code == S.EINVAL
    pl.load_dag([0, 0], [])                  # single function: ok


def test_call_order_estate():
    pl = S.Planner()
    with pytest.raises(S.SmilessError) as e:
        pl.load_profiles([1], [1], [1], [1.0])
    assert e.value.code == S.ESTATE
    pl.load_dag([0, 0], [])
    with pytest.raises(S.SmilessError) as e:
        pl.plan([0, 1], 10, [0])
    assert e.value.code == S.ESTATE
    with pytest.raises(S.SmilessError) as e:
        pl.space_size(1)
    assert e.value.code == S.ESTATE


def test_profile_validation():
    pl = S.Planner()
    pl.load_dag([0, 0, 1], [0])
    for bad in [dict(n_configs=[0, 1]), dict(exec_us=[-1, 1]), dict(init_us=[1 << 29, 1]),
                dict(price_per_us=[float("nan"), 1.0]), dict(price_per_us=[-1.0, 1.0])]:
        kw = dict(n_configs=[1, 1], exec_us=[1, 1], init_us=[1, 1], price_per_us=[1.0, 1.0])
        kw.update(bad)
        with pytest.raises(S.SmilessError) as e:
            pl.load_profiles(**kw)
        assert e.value.code == S.EINVAL


def test_plan_argument_validation_before_any_gpu_work():
    pl, p = planner()
    ok = dict(arrivals=p.arrivals_us, sla_us=p.sla_us, windows_us=p.windows_us)
    cases = [
        (dict(windows_us=[0, 0, 5]), S.EINVAL),                    # not strictly increasing
        (dict(windows_us=[-1, 5]), S.EINVAL),
        (dict(windows_us=[0, 1 << 29]), S.EINVAL),
        (dict(windows_us=list(range(40))), S.EINVAL),               # W > SMILESS_MAX_WINDOWS
        (dict(sla_us=-1), S.EINVAL),
        (dict(sla_us=1 << 29), S.EINVAL),
        (dict(arrivals=[5, 3, 9]), S.EINVAL),                       # decreasing arrivals
        (dict(arrivals=[]), S.EINVAL),
        (dict(arrivals=[0, 1 << 62]), S.EINVAL),
        (dict(n_fixed=4), S.EINVAL),
        (dict(n_fixed=1, fixed_digits=[16]), S.EINVAL),             # digit >= M*W
        (dict(n_shards=2, shard=2), S.EINVAL),
        (dict(cost_cap=float("nan")), S.EINVAL),
        (dict(cost_cap=-1.0), S.EINVAL),
        (dict(cost_cap=1.0, flags=S.FLAG_NO_PRUNE), S.EINVAL),      # the cap is a prune-mode argument
        (dict(instances=[1, 0, 1]), S.EINVAL),                      # scale-out: >= 1 instance
        (dict(instances=[1, 17, 1]), S.EINVAL),                     # <= SMILESS_MAX_INSTANCES
    ]
    for over, code in cases:
        kw = dict(ok)
        kw.update(over)
        with pytest.raises(S.SmilessError) as e:
            pl.plan(**kw)
        assert e.value.code == code, over


def test_plan_digits_argument_validation_before_any_gpu_work():
    """smiless_plan_digits rejects bad digit ranges and unsupported options before touching the
    device (works without a GPU)."""
    p = W.make_config("C1", n_arrivals=20)
    pl = S.planner_for(p)
    args = (p.arrivals_us, p.sla_us, p.windows_us)
    Wn = len(p.windows_us)
    bad = [
        ((0, 0), dict(n_fixed=1, fixed_digits=[0])),                          # empty range
        ((3, 2), dict(n_fixed=1, fixed_digits=[0])),
        ((0, 4), dict(n_fixed=0)),                                             # no pinned digit
        ((0, 4 * Wn + 1), dict(n_fixed=1, fixed_digits=[0])),                  # beyond the radix
        ((-1, 2), dict(n_fixed=1, fixed_digits=[0])),
        ((0, 2), dict(n_fixed=3, fixed_digits=[0, 0, 0])),                     # nothing left to search
        ((0, 2), dict(n_fixed=1, fixed_digits=[0], cost_out=np.empty(256))),   # no per-candidate dump
    ]
    for (d0, d1), kw in bad:
        with pytest.raises(S.SmilessError) as e:
            pl.plan_digits(*args, d0, d1, **kw)
        assert e.value.code == S.EINVAL, (d0, d1, kw)


def test_negative_zero_price_rejected():
    """-0.0 would give cost bits with the sign set: rejected like a negative price."""
    pl = S.Planner(device=0)
    pl.load_dag(*W.csr_from_preds([[], [0]]))
    with pytest.raises(S.SmilessError) as e:
        pl.load_profiles([1, 1], [10, 10], [5, 5], [1.0, -0.0])
    assert e.value.code == S.EINVAL


def test_space_size_and_erange():
    pl, p = planner(W.make_config("C5", n_arrivals=10))
    with pytest.raises(S.SmilessError) as e:
        pl.space_size(16)                    # 128^10 = 2^70 > 2^63-1
    assert e.value.code == S.ERANGE
    assert pl.space_size(16, n_fixed=2) == 128 ** 8
    assert pl.space_size(16, n_fixed=1) == 2 ** 63    # indices 0 .. 2^63-1 still fit int64
    with pytest.raises(S.SmilessError) as e:
        pl.plan(p.arrivals_us, p.sla_us, p.windows_us)
    assert e.value.code == S.ERANGE


def test_decode_matches_numpy_unravel():
    pl, p = planner(W.make_config("C2", n_arrivals=10))
    Wn = len(p.windows_us)
    shape = tuple(int(m) * Wn for m in p.n_configs)
    rng = np.random.default_rng(0)
    for idx in rng.integers(0, pl.space_size(Wn), size=200):
        c, w = pl.decode(int(idx), Wn)
        d = np.unravel_index(int(idx), shape)
        assert (c == np.array(d) // Wn).all() and (w == np.array(d) % Wn).all()
    c, w = pl.decode(7, Wn, n_fixed=2, fixed_digits=[3, 9])
    assert c[:2].tolist() == [0, 1] and w[:2].tolist() == [3, 1]
    with pytest.raises(S.SmilessError) as e:
        pl.decode(pl.space_size(Wn), Wn)
    assert e.value.code == S.ERANGE


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_nvrtc_specialises_every_config_for_sm100a(name):
    """NVRTC compiles the DAG-specialised evaluator for sm_100a with no local memory."""
    p = W.make_config(name, n_arrivals=100)
    pl = S.planner_for(p)
    nf = 3 if name == "C5" else 0
    log, n = pl.jit_compile(p.arrivals_us, p.sla_us, p.windows_us, n_fixed=nf, fixed_digits=[0] * nf)
    assert n > 0
    assert "0 bytes stack frame, 0 bytes spill stores, 0 bytes spill loads" in log, log
    src = pl.kernel_source(p.arrivals_us, p.sla_us, p.windows_us, n_fixed=nf, fixed_digits=[0] * nf)
    # scale-out plans (C3 / C5) carry instance rings; a scaled-out LAST function (C5) adds the
    # virtual sink to the kernel DAG (DESIGN §5 item 13)
    scale_out = p.instances is not None and max(p.instances) > 1
    virt = False        # the default keeps a scaled-out last function's variants (ring form)
    assert "#define SM_N %d" % (p.n_funcs + virt) in src and "smiless_plan_kernel" in src
    assert ("#define SM_INST %d" % scale_out) in src and ("#define SM_VIRT %d" % virt) in src


def test_fused_memo_kernel_compiles_for_the_bench_slice(monkeypatch):
    """The bench slice (C2, throughput mode) selects the fused producer/consumer kernel
    (SMILESS_FUSED=0 the two-kernel path); it compiles for sm_100a with no local memory and
    its consumer loop reads x from shared memory, not global memory."""
    import bench
    p, kw = bench.workload("C2")
    pl = S.planner_for(p)
    args = (p.arrivals_us, p.sla_us, p.windows_us)
    assert "#define SM_FUSED 1" in pl.kernel_source(*args, flags=S.FLAG_NO_PRUNE, **kw)
    monkeypatch.setenv("SMILESS_FUSED", "0")
    assert "#define SM_FUSED 0" in pl.kernel_source(*args, flags=S.FLAG_NO_PRUNE, **kw)
    monkeypatch.delenv("SMILESS_FUSED")
    log, n = pl.jit_compile(*args, flags=S.FLAG_NO_PRUNE, **kw)
    entry = log.split("Compiling entry function 'smiless_fused_kernel'")[1].split("Compiling entry")[0]
    assert "0 bytes stack frame, 0 bytes spill stores, 0 bytes spill loads" in entry, entry
    import sys
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
    import sass_mix
    body, _ = sass_mix.loop_body("smiless_fused_kernel")
    assert any(t.startswith("LDS.128") for t in body) and not any(t.startswith("LDG") for t in body)


def test_branch_and_bound_levels_per_config():
    """B&B depths the library picks for the exact full-space plans: three levels (a middle
    level) only where a shallow survivor would have more than 2^20 deep children (C5 with
    function 0 pinned: D = 8, DA = 3 -- sub-plans keep the shallow level at <= 2^16 prefixes --
    and DM = 6), two levels on C2 and C3."""
    expect = {"C2": (4, 3, 0), "C3": (6, 3, 0), "C5": (8, 3, 6)}
    for name, (d, da, dm) in expect.items():
        p = W.make_config(name, n_arrivals=100)
        pl = S.planner_for(p)
        nf = 1 if name == "C5" else 0
        kw = dict(n_fixed=nf, fixed_digits=[96] * nf)
        if p.instances is not None:
            kw["instances"] = list(p.instances)
        src = pl.kernel_source(p.arrivals_us, p.sla_us, p.windows_us, **kw)
        got = tuple(int(re.search(r"#define %s (\d+)" % m, src).group(1)) for m in ("SM_D", "SM_DA", "SM_DM"))
        assert got == (d, da, dm), (name, got)
        assert ("smiless_bound_kernel_m" in src) and (dm == 0 or "#define SM_DM 6" in src)


def test_int64_path_selected_when_int32_range_fails():
    p = W.make_config("C1", n_arrivals=20)
    p = p.replace(windows_us=np.array([0, (1 << 29) - 1], np.int32), init_us=np.full_like(p.init_us, (1 << 29) - 1))
    pl = S.planner_for(p)
    src = pl.kernel_source(p.arrivals_us, p.sla_us, p.windows_us)
    assert "#define SM_TIME64 1" in src
    log, n = pl.jit_compile(p.arrivals_us, p.sla_us, p.windows_us)
    assert n > 0
    p2 = W.make_config("C1", n_arrivals=20)
    src2 = S.planner_for(p2).kernel_source(p2.arrivals_us, p2.sla_us, p2.windows_us)
    assert "#define SM_TIME64 0" in src2


def _sass(pl, p, **kw):
    import subprocess
    import tempfile
    log, cubin = pl.jit_compile(p.arrivals_us, p.sla_us, p.windows_us, want_cubin=True, **kw)
    with tempfile.NamedTemporaryFile(suffix=".cubin") as f:
        f.write(cubin)
        f.flush()
        return subprocess.run(["cuobjdump", "-sass", f.name], capture_output=True, text=True, check=True).stdout


def _sass_functions(sass):
    """{kernel name: [(address, instruction text)]} of a cuobjdump -sass listing."""
    import re
    out, cur = {}, None
    for line in sass.split("\n"):
        m = re.search(r"Function : (\w+)", line)
        if m:
            cur = out.setdefault(m.group(1), [])
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
        if m and cur is not None:
            cur.append((int(m.group(1), 16), m.group(2)))
    return out


def _back_branch(addr, ins):
    """Target of a backward branch at addr (a loop [target, addr]), else nothing."""
    import re
    m = re.search(r"BRA(?:\.\w+)*\s+(?:!?U?P\w+,\s*)?0x([0-9a-f]+)", ins)
    if m and int(m.group(1), 16) < addr:
        yield int(m.group(1), 16)


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_sass_has_no_vimnmx3_and_is_dpx(name):
    """ptxas 12.9 drops operand negations it folds into VIMNMX3 (tools/repro_vimnmx3.cu,
    DESIGN.md "Compiler erratum"): the evaluator must contain no VIMNMX3.  Also checks the
    hot loop really is DPX integer code with the busy mask on the FMA pipe (IMAD.HI)."""
    p = W.make_config(name, n_arrivals=100)
    pl = S.planner_for(p)
    nf = 3 if name == "C5" else 0
    sass = _sass(pl, p, n_fixed=nf, fixed_digits=[0] * nf)
    assert "VIMNMX3" not in sass
    for op in ("VIADDMNMX", "VIMNMX.RELU", "IMAD.HI", "LDS.128"):
        assert op in sass, op
    assert "HMMA" not in sass and "UTC" not in sass          # no tensor cores on this path
    # no local memory in the evaluator and B&B kernels; the memoised variants kernels may keep
    # a register spilled across the step loop (C5 / C4: 4 bytes, stored once per claimed unit
    # before the loop over 10^4 invocations and reloaded once after it) but never inside an
    # innermost loop (the step loops)
    for fn, code in _sass_functions(sass).items():
        local = [a for a, ins in code if "LDL" in ins or "STL" in ins]
        if fn not in ("smiless_variants_kernel", "smiless_variants_cost_kernel"):
            assert not local, (fn, local)
        loops = [(t, a) for a, ins in code for t in _back_branch(a, ins)]
        inner = [(lo, hi) for lo, hi in loops if not any(lo <= l2 and h2 <= hi and (l2, h2) != (lo, hi)
                                                         for l2, h2 in loops)]
        assert not [x for x in local if any(lo <= x <= hi for lo, hi in inner)], (fn, local, inner)


def test_library_kernels_have_no_vimnmx3():
    import subprocess
    out = subprocess.run(["cuobjdump", "-sass", S.LIB_PATH], capture_output=True, text=True, check=True).stdout
    assert "prep_offsets_kernel" in out and "eval_exact_kernel" in out
    assert "VIMNMX3" not in out


def test_derive_windows_is_the_papers_rule():
    p = W.make_config("C2", n_arrivals=10)
    pl = S.planner_for(p)
    for it in (0, 1_000_000, 4_000_000, 20_000_000):
        rw = pl.derive_windows(it)
        exp = [it - t - i if t + i < it else 0 for t, i in zip(p.init_us.tolist(), p.exec_us.tolist())]
        assert rw.tolist() == exp
    with pytest.raises(S.SmilessError) as e:
        pl.plan(p.arrivals_us, p.sla_us, [0, 5], row_windows=rw)       # requires n_windows == 1
    assert e.value.code == S.EINVAL


def test_autoscale_matches_brute_force_oracle():
    """NEXT-4 (Eq. (7)/(8)): bisection over B per config == brute force over
    every (config, B) (host-only, no GPU)."""
    from oracle.autoscale import autoscale
    rng = np.random.default_rng(81)
    for name in ("C1", "C2", "C3"):
        p = W.make_config(name, n_arrivals=10)
        pl = S.planner_for(p)
        for _ in range(20):
            G = rng.integers(0, 200, size=p.n_funcs)
            it = int(rng.integers(100_000, 5_000_000))
            tgt = rng.integers(50_000, 5_000_000, size=p.n_funcs)
            got = pl.autoscale(p.batch_slope_us, p.batch_intercept_us, G, it, tgt)
            ref = autoscale(p, p.batch_slope_us, p.batch_intercept_us, G, it, tgt)
            for k in range(p.n_funcs):
                c, B, inst, cost = ref[k]
                assert (int(got[k]["config"]), int(got[k]["batch"]), int(got[k]["instances"])) == (c, B, inst)
                assert float(got[k]["cost"]) == cost or (c == -1 and G[k] > 0 and np.isinf(got[k]["cost"]))


def test_autoscale_paper_properties():
    """More invocations never cost less; a looser latency target never costs more."""
    p = W.make_config("C2", n_arrivals=10)
    pl = S.planner_for(p)
    it = 1_000_000
    base = pl.autoscale(p.batch_slope_us, p.batch_intercept_us, [50] * 6, it, [2_000_000] * 6)
    more = pl.autoscale(p.batch_slope_us, p.batch_intercept_us, [100] * 6, it, [2_000_000] * 6)
    loose = pl.autoscale(p.batch_slope_us, p.batch_intercept_us, [50] * 6, it, [4_000_000] * 6)
    for k in range(6):
        assert more[k]["cost"] >= base[k]["cost"]
        assert loose[k]["cost"] <= base[k]["cost"]
