"""The C-ABI library loads on a CPU-only host and exports every entry point include/gd.h
declares; host-only entry points behave as documented.  No compute calls (no GPU here)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "gd.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:gd_status|const char\*|int|void\*)\s+(gd_\w+)\s*\(", src, flags=re.M)))


@pytest.fixture(scope="module")
def gd():
    from tools import build_native
    build_native.build()
    from paper_conf_icpp_jiangj024_b200 import _lib
    return _lib


def test_header_and_binding_agree(gd):
    assert declared_functions() == sorted(gd.EXPORTS)


def test_every_declared_symbol_is_exported(gd):
    for name in declared_functions():
        assert hasattr(gd.lib, name), name
    nm = subprocess.run(["nm", "-D", "--defined-only", gd.LIB_PATH], capture_output=True, text=True).stdout
    for name in declared_functions():
        assert re.search(rf"\bT {name}\b", nm), f"{name} not a defined text symbol"


def test_kernels_are_sm100a(gd):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", gd.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version_and_bounds_host_only(gd):
    assert gd.lib.gd_version() >= 10000
    from paper_conf_icpp_jiangj024_b200 import sample_bounds
    nm, em = sample_bounds(1000, [15, 10, 5], 111_000_000, 1_600_000_000)
    assert nm == [1000, 16000, 176000, 1056000] and em == [15000, 160000, 880000]
    nm, em = sample_bounds(4, [-1, 2], 10, 50)
    assert em == [50, 20] and nm == [4, 10, 10]


def test_bounds_reject_bad_fanout(gd):
    from paper_conf_icpp_jiangj024_b200 import GdError, sample_bounds
    with pytest.raises(GdError) as e:
        sample_bounds(10, [300], 100, 1000)
    assert e.value.status == 1 and "fanout" in str(e.value)
    with pytest.raises(GdError):
        sample_bounds(10, [1] * 9, 100, 1000)


def test_null_handles_rejected(gd):
    L = gd.lib
    assert L.gd_sample(None, None, 0, None, 1, 0, 0, None, None) == 1
    assert L.gd_extract(None, None, None, 0, None, None, None, None, None) == 1
    assert L.gd_buffer_release(None, None, None, 0, None) == 1
    assert L.gd_check_device_status(None, None) == 1
    assert b"null" in L.gd_last_error()
    assert L.gd_graph_destroy(None) == 0 and L.gd_buffer_destroy(None) == 0


def test_plain_c_client_compiles_links_and_runs(gd, tmp_path):
    """gd.h is a C header (gcc -std=c99, no nvcc, no CUDA headers): a plain C client takes the
    address of every declared entry point, links against libgd.so and runs its host-only calls."""
    names = declared_functions()
    src = tmp_path / "client.c"
    src.write_text(
        '#include <stdio.h>\n#include "gd.h"\n'
        "int main(void) {\n"
        f"    void* syms[] = {{ {', '.join('(void*)' + n for n in names)} }};\n"
        f"    for (unsigned i = 0; i < {len(names)}u; ++i) if (!syms[i]) return 10;\n"
        "    int32_t fan[3] = {15, 10, 5};\n"
        "    int64_t nm[4], em[3];\n"
        "    if (gd_sample_bounds(1000, fan, 3, 111000000, 1600000000, nm, em) != GD_OK) return 11;\n"
        "    if (nm[3] != 1056000 || em[2] != 880000) return 12;\n"
        "    int32_t bad[1] = {GD_MAX_FANOUT + 1};\n"
        "    if (gd_sample_bounds(10, bad, 1, 100, 1000, nm, em) != GD_ERR_INVALID) return 13;\n"
        "    if (gd_last_error()[0] == 0) return 14;\n"
        "    if (gd_extract(NULL, NULL, NULL, 0, NULL, NULL, NULL, NULL, NULL) != GD_ERR_INVALID) return 15;\n"
        '    printf("%d\\n", gd_version());\n'
        "    return 0;\n}\n")
    exe = tmp_path / "client"
    libdir = os.path.dirname(gd.LIB_PATH)
    r = subprocess.run(["gcc", "-std=c99", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"), str(src), "-o",
                        str(exe), "-L", libdir, "-l:libgd.so", f"-Wl,-rpath,{libdir}"], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    r = subprocess.run([str(exe)], capture_output=True, text=True)
    assert r.returncode == 0, (r.returncode, r.stderr)
    assert int(r.stdout) == gd.lib.gd_version()
