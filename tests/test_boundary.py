"""CPU checks of the boundary: the C-ABI library builds for sm_100a, loads,
and exports every symbol include/tq.h declares; the oracle and the product
share no code; the product path has no CPU fallback."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_icpp_troendletj19_b200")


def header_functions():
    src = open(os.path.join(ROOT, "include", "tq.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(\w+)\s*\(", src, flags=re.M)) - {"if"}


@pytest.fixture(scope="module")
def libtq():
    from paper_conf_icpp_troendletj19_b200 import _build
    return _build.build()


def test_header_declares_the_boundary():
    fns = header_functions()
    for f in ("tq_create", "tq_destroy", "tq_reset", "tq_device_view_get", "bfs_run", "bfs_run_ex",
              "bfs_plan_create", "bfs_plan_run", "bfs_plan_destroy", "tq_bench", "tq_strerror"):
        assert f in fns


def test_library_exports_every_declared_symbol(libtq):
    out = subprocess.check_output(["nm", "-D", "--defined-only", libtq], text=True)
    exported = {line.split()[-1] for line in out.splitlines() if " T " in line}
    missing = header_functions() - exported
    assert not missing, f"declared in tq.h but not exported: {missing}"
    from paper_conf_icpp_troendletj19_b200 import _lib
    assert set(_lib.EXPORTS) == header_functions()


def test_library_loads_and_reports(libtq):
    from paper_conf_icpp_troendletj19_b200 import _lib
    L = _lib.lib()
    assert b"sm_100a" in L.tq_version()
    assert L.tq_strerror(-4).startswith(b"queue full")


def test_struct_mirrors_match_the_header(libtq):
    """Every ctypes mirror has the C layout's size (include/tq.h)."""
    import ctypes
    from paper_conf_icpp_troendletj19_b200 import _lib
    L = _lib.lib()
    for name, cls in _lib.STRUCTS.items():
        assert L.tq_struct_size(name.encode()) == ctypes.sizeof(cls), name
    assert L.tq_struct_size(b"no_such_struct") == 0


def test_library_is_sm_100a_code(libtq):
    out = subprocess.check_output(["cuobjdump", "--list-elf", libtq], text=True)
    assert "sm_100a" in out


def test_device_header_compiles_standalone(tmp_path):
    # a user kernel built against include/tq_device.cuh alone
    cu = tmp_path / "user.cu"
    cu.write_text('#include "tq_device.cuh"\n'
                  '__global__ void k(tq_device_view q, unsigned *out) {\n'
                  '  unsigned long long t = tq_warp_dequeue_n(q, true);\n'
                  '  unsigned it; if (tq_take(q, t, &it)) out[threadIdx.x] = it;\n'
                  '  unsigned items[1] = {threadIdx.x};\n'
                  '  tq_warp_enqueue_n<1>(q, 1u, items);\n}\n')
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-c",
                           "-I", os.path.join(ROOT, "include"), "-o", str(tmp_path / "u.o"), str(cu)])


def _imports(path):
    txt = open(path).read()
    return set(re.findall(r"^\s*(?:from|import)\s+([\w.]+)", txt, flags=re.M))


def test_product_and_oracle_share_no_code():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            p = os.path.join(dirpath, f)
            if f.endswith(".py"):
                assert not any(m.split(".")[0] == "oracle" for m in _imports(p)), p
                assert not any(m.split(".")[0] == "inputs" for m in _imports(p)), p
            if f.endswith((".cu", ".cuh")):
                assert "oracle" not in re.findall(r'#include\s+"([^"]+)"', open(p).read())
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        p = os.path.join(ROOT, "oracle", f)
        if f.endswith(".py"):
            assert not any(m.startswith("paper_conf") for m in _imports(p)), p
        if f.endswith((".c", ".h")):
            txt = open(p).read()
            assert "tq.h" not in txt and "tq_device" not in txt


def test_missing_library_fails_loudly(monkeypatch, tmp_path):
    from paper_conf_icpp_troendletj19_b200 import _lib
    monkeypatch.setattr(_lib, "_lib", None)
    monkeypatch.setattr(_lib, "LIB_PATH", str(tmp_path / "nope.so"))
    with pytest.raises(ImportError):
        _lib.lib()


def test_input_generator_builds():
    import inputs.gpu
    assert os.path.exists(inputs.gpu.build())


def test_probe_ceiling_rejects_bad_sizes(libtq):
    """Argument checks run before any device work (no GPU needed)."""
    import ctypes
    from paper_conf_icpp_troendletj19_b200 import _lib
    L = _lib.lib()
    g = ctypes.c_double(-1.0)
    for table, probes in [(1 << 11, 1 << 22), (1 << 32, 1 << 22), (1 << 20, 1 << 19), (1 << 20, 1 << 32)]:
        assert L.tq_probe_ceiling(0, table, probes, None, ctypes.byref(g)) == -1
    assert L.tq_probe_ceiling(0, 1 << 20, 1 << 22, None, None) == -1
