"""CPU checks of the C-ABI boundary: libvs.so builds, loads, exports every symbol that
include/vs.h declares, rejects bad arguments on the host; and the oracle / CUDA path share
no code.  No compute call is made (there is no GPU here)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "vs.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_chenqldx21_b200 import _build
    path = _build.build()
    return ctypes.CDLL(path)


def declared_symbols():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(vs_[a-z_0-9]+)\s*\(", text)))


def test_header_declares_the_three_entry_points():
    syms = declared_symbols()
    for s in ("vs_encode_colvec", "vs_spmm", "vs_sddmm", "vs_status_string"):
        assert s in syms


def test_library_exports_every_declared_symbol(lib):
    for s in declared_symbols():
        assert hasattr(lib, s), f"libvs.so does not export {s}"


def test_exports_are_c_linkage():
    import subprocess
    from paper_conf_sc_chenqldx21_b200 import lib_path
    out = subprocess.run(["nm", "-D", "--defined-only", lib_path], capture_output=True, text=True).stdout
    names = {l.split()[-1] for l in out.splitlines() if l.strip()}
    for s in declared_symbols():
        assert s in names, f"{s} not exported with C linkage"


def test_status_strings(lib):
    lib.vs_status_string.restype = ctypes.c_char_p
    assert lib.vs_status_string(0) == b"VS_SUCCESS"
    assert lib.vs_status_string(1) == b"VS_ERROR_INVALID_VALUE"
    assert lib.vs_status_string(4) == b"VS_ERROR_MISALIGNED"
    assert lib.vs_version() > 0


def test_host_argument_checks_before_any_device_work(lib):
    """Invalid V / sizes / missing inputs are rejected on the host (no device needed)."""
    P = ctypes.c_void_p
    i64 = ctypes.c_int64
    lib.vs_spmm.argtypes = [i64, i64, i64, ctypes.c_int, P, P, P, P, P, P]
    lib.vs_sddmm.argtypes = [i64, i64, i64, ctypes.c_int, P, P, P, P, P, P]
    lib.vs_encode_colvec.argtypes = [i64, i64, ctypes.c_int, P, P, P, P, P, P, P]
    fake = P(4096)
    assert lib.vs_spmm(8, 8, 8, 3, fake, fake, fake, fake, fake, None) == 1
    assert lib.vs_spmm(-1, 8, 8, 4, fake, fake, fake, fake, fake, None) == 1
    assert lib.vs_spmm(0, 8, 8, 4, None, None, None, None, None, None) == 0  # M == 0: no-op
    assert lib.vs_sddmm(8, 8, 8, 5, fake, fake, fake, fake, fake, None) == 1
    assert lib.vs_encode_colvec(8, 8, 4, None, None, fake, None, None, None, None) == 1
    assert lib.vs_spmm(8, 8, 8, 4, P(4098), fake, fake, fake, fake, None) == 4  # row_ptr misaligned
    assert lib.vs_sddmm(8, 8, 8, 4, fake, fake, P(4097), fake, fake, None) == 4  # A misaligned
    lib.vs_spmm_scatter.argtypes = [i64, i64, i64, ctypes.c_int, P, P, P, P,
                                    ctypes.POINTER(P), ctypes.c_int, i64, P]
    dsts = (P * 2)(4096, 8192)
    assert lib.vs_spmm_scatter(8, 8, 8, 4, fake, fake, fake, fake, None, 1, 8, None) == 1
    assert lib.vs_spmm_scatter(8, 8, 8, 4, fake, fake, fake, fake, dsts, 0, 8, None) == 1
    assert lib.vs_spmm_scatter(8, 8, 8, 4, fake, fake, fake, fake, dsts, 9, 8, None) == 1
    assert lib.vs_spmm_scatter(8, 8, 8, 4, fake, fake, fake, fake, dsts, 2, 7, None) == 1  # ldc < N
    bad = (P * 2)(4096, 8193)
    assert lib.vs_spmm_scatter(8, 8, 8, 4, fake, fake, fake, fake, bad, 2, 8, None) == 4
    assert lib.vs_spmm_scatter(0, 8, 8, 4, fake, fake, fake, fake, dsts, 2, 8, None) == 0


def test_no_shared_code_between_oracle_and_cuda_path():
    """The oracle includes only system headers and imports nothing of the CUDA path; the
    CUDA path never includes or imports the oracle."""
    inc = re.compile(r'^\s*#\s*include\s*[<"]([^>"]+)[>"]', re.M)
    imp = re.compile(r'^\s*(?:from|import)\s+([\w.]+)', re.M)
    pkg = os.path.join(ROOT, "paper_conf_sc_chenqldx21_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            text = open(os.path.join(dirpath, f), errors="ignore").read() if f.endswith(
                (".cu", ".cuh", ".py", ".h", ".cpp")) else ""
            assert not any("oracle" in h for h in inc.findall(text)), f
            assert not any(m.split(".")[0] == "oracle" for m in imp.findall(text)), f
    otext = open(os.path.join(ROOT, "oracle", "oracle.c")).read()
    assert set(inc.findall(otext)) <= {"stdint.h", "stddef.h", "stdlib.h", "math.h", "string.h", "time.h"}
    ptext = open(os.path.join(ROOT, "oracle", "__init__.py")).read()
    assert not any(m.split(".")[0] in ("paper_conf_sc_chenqldx21_b200", "synth")
                   for m in imp.findall(ptext))


def test_package_fails_loudly_without_library(tmp_path, monkeypatch):
    import paper_conf_sc_chenqldx21_b200 as vs
    monkeypatch.setattr(vs, "lib_path", str(tmp_path / "missing.so"))
    monkeypatch.setattr(vs, "_lib", None)
    with pytest.raises(ImportError):
        vs.load()
