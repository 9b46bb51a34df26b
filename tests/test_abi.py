"""C-ABI checks that need no GPU: the library loads, exports every symbol include/gpapriori.h
declares, the header compiles standalone as C and C++, host-only entry points behave, and
compute entry points fail loudly (no CPU fallback) when no GPU is present."""
import ctypes
import os
import re
import subprocess
from fractions import Fraction

import numpy as np
import pytest

import paper_conf_cluster_zhangzb11a_b200 as gpa

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "gpapriori.h")


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    names = set()
    for m in re.finditer(r"^[A-Za-z_][\w \*]*?\b(gpa_\w+)\s*\(", text, flags=re.M):
        names.add(m.group(1))
    return names


def test_library_exports_every_declared_symbol():
    names = declared_functions()
    assert len(names) >= 25
    lib = ctypes.CDLL(gpa.LIB_PATH)
    missing = [n for n in sorted(names) if not hasattr(lib, n)]
    assert not missing, missing
    out = subprocess.run(["nm", "-D", "--defined-only", gpa.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (gpa_\w+)", out))
    assert names == exported, (names ^ exported)


@pytest.mark.parametrize("cc,flags", [("gcc", ["-std=c99", "-x", "c"]), ("g++", ["-std=c++17", "-x", "c++"])])
def test_header_compiles_standalone(tmp_path, cc, flags):
    src = tmp_path / "t.src"
    src.write_text('#include "gpapriori.h"\nint main(void){ gpa_options o; gpa_options_default(&o); return (int)o.count_kernel; }\n')
    r = subprocess.run([cc, *flags, "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"), "-c", str(src), "-o",
                        str(tmp_path / "t.o")], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr


def test_sm100a_cubin_present():
    out = subprocess.run(["cuobjdump", "--list-elf", gpa.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_min_count_host_function():
    for n, s in [(3196, "0.90"), (8124, "0.20"), (100_000, "0.01"), (340_183, "0.30"), (10_000_000, "0.005"),
                 (100, "0.07"), (7, "1"), (0, "0.5"), (1, "0")]:
        f = Fraction(s) * n
        assert gpa.min_count(n, s) == max(1, -(-f.numerator // f.denominator))
    assert gpa.lib().gpa_min_count(10, 1, 0) == 0


def test_options_default():
    o = gpa.Options()._c()
    assert o.count_kernel == 0 and o.flags == 0 and o.device == -1 and o.max_k == 0


def test_version():
    assert "sm_100a" in gpa.version()


def test_no_cpu_fallback_without_gpu():
    """Without a CUDA device every compute entry point returns an error (no silent CPU path)."""
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    offsets = np.array([0, 2, 3], dtype=np.uint64)
    items = np.array([1, 2, 1], dtype=np.uint32)
    with pytest.raises(gpa.GpaError) as e:
        gpa.mine(offsets, items, 4, min_count=1)
    assert e.value.status == 4  # GPA_ERR_CUDA
    with pytest.raises(gpa.GpaError):
        gpa.Bitset(offsets, items, 4)


def test_null_arguments_are_rejected():
    L = gpa.lib()
    h = ctypes.c_void_p()
    assert L.gpa_mine(None, 1, None, None, ctypes.byref(h)) == 1
    assert L.gpa_bitset_create(None, 1, None, None, ctypes.byref(h)) == 1
    assert b"NULL" in L.gpa_last_error()
    for fn in ("gpa_bitset_destroy", "gpa_result_destroy", "gpa_dist_destroy"):
        assert getattr(L, fn)(None) == 0


def test_c_example_builds_and_fails_loudly_without_gpu(tmp_path):
    """examples/gpa_mine_fimi.c uses only the C ABI; without a GPU it must exit non-zero with the
    library's CUDA error, not produce output."""
    exe = os.path.join(ROOT, "examples", "gpa_mine_fimi")
    subprocess.check_call(["make", "-C", ROOT, "-s", "examples/gpa_mine_fimi"])
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    dat = tmp_path / "t.dat"
    dat.write_text("1 2 3\n2 3\n")
    r = subprocess.run([exe, str(dat), "0.5"], capture_output=True, text=True)
    assert r.returncode != 0 and r.stdout == "" and "status 4" in r.stderr
