"""The C-ABI library loads and exports every symbol include/spinfer.h declares
(-m "not gpu": no compute calls), plus host-only logic (tp_rows, status strings)."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    src = open(os.path.join(ROOT, "include", "spinfer.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(spinfer_[a-z_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def sp():
    from paper_conf_eurosys_fanydlgww025_b200 import build
    build.build()
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    return sp


def test_header_symbols_exported(sp):
    names = _header_functions()
    assert set(names) == set(sp.SYMBOLS), names
    out = subprocess.run(["nm", "-D", "--defined-only", sp.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (spinfer_\w+)", out))
    assert set(names) <= exported
    # nothing else leaks from the library (hidden visibility)
    assert exported == set(names), exported - set(names)
    L = sp.lib()
    for n in names:
        assert getattr(L, n) is not None


def _kernel_sass(sp):
    """SASS of every kernel function in the library: {mangled name: text}."""
    sass = subprocess.run(["cuobjdump", "-sass", sp.LIB_PATH], capture_output=True, text=True).stdout
    out, name = {}, None
    for line in sass.splitlines():
        m = re.match(r"\s*Function : (\S+)", line)
        if m:
            name = m.group(1)
            out[name] = []
        elif name:
            out[name].append(line)
    return {k: "\n".join(v) for k, v in out.items()}


def test_built_for_sm100a(sp):
    out = subprocess.run(["cuobjdump", "--list-elf", sp.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    ks = _kernel_sass(sp)
    dw = [v for k, v in ks.items() if "k_spmm_dw" in k]
    tc = [v for k, v in ks.items() if "k_spmm_tc" in k]
    assert len(dw) == 6 and len(tc) == 2, sorted(ks)   # dw: N = 8, 16, 32 (half mode) x {plain, epilogue}
    for v in dw:   # N <= 32: mma.sync tensor cores fed by TMA, named-barrier slot release
        for mn in ("HMMA.16816.F32", "UBLKCP", "UTMALDG.2D", "LDSM.16.MT88", "SYNCS", "BAR.ARV"):
            assert mn in v, mn
    for v in tc:   # N > 16: tcgen05 MMA (UTCHMMA), TMEM stores / loads (STTM / LDTM), TMA
        for mn in ("UTCHMMA", "STTM", "LDTM", "UTMALDG.2D", "UBLKCP", "UTCBAR", "SYNCS"):
            assert mn in v, mn


def test_status_strings_and_version(sp):
    L = sp.lib()
    assert L.spinfer_status_str(0) == b"SPINFER_OK"
    assert b"EINVAL" in L.spinfer_status_str(-1)
    assert b"ENOSPC" in L.spinfer_status_str(-2)
    assert b"sm_100a" in L.spinfer_version()


def test_tp_rows_host_logic(sp):
    import oracle
    for M in (64, 100, 1000, 1152, 9216, 28672, 36864):      # 100, 1000: ragged tail (reading A8)
        for world in (1, 2, 3, 4, 8):
            spans = [sp.tp_rows(M, world, r) for r in range(world)]
            assert spans == [oracle.tp_rows(M, world, r) for r in range(world)]
            assert sum(c for _, c in spans) == M
            assert all(b % 64 == 0 or c == 0 for b, c in spans)
    with pytest.raises(sp.SpinferError):
        sp.tp_rows(0, 2, 0)
    with pytest.raises(sp.SpinferError):
        sp.tp_rows(128, 2, 2)


def test_no_cpu_fallback_without_device(sp):
    import torch
    if torch.cuda.is_available():
        pytest.skip("has a GPU")
    with pytest.raises((ValueError, RuntimeError)):
        sp.encode(torch.zeros((64, 64), dtype=torch.float16))
