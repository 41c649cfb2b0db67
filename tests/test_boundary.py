"""CPU-only checks of the C-ABI boundary: the library builds for sm_100a, loads,
exports every function include/moe.h declares, and the Python binding's
ctypes structs match the C layout (gcc-compiled probe).  No compute calls."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "moe.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import build
    build.build()
    return ctypes.CDLL(build.LIB)


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(moe_\w+)\s*\(", src, flags=re.M)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for f in ("moe_layer_create", "moe_layer_forward", "moe_layer_forward_deferred", "moe_layer_destroy"):
        assert f in names


def test_library_exports_every_declared_symbol(lib):
    for name in declared_functions():
        assert hasattr(lib, name), f"{name} declared in include/moe.h but not exported"


def test_library_is_sm100a(lib):
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import build
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", build.LIB], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_status_strings(lib):
    lib.moe_status_string.restype = ctypes.c_char_p
    assert lib.moe_status_string(0) == b"MOE_OK"
    assert lib.moe_status_string(-6) == b"MOE_ERR_CAPACITY"


def test_create_rejects_bad_config_without_gpu(lib):
    """Argument validation runs before any device call (status, not abort)."""
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    moe._lib = None
    L = moe.load_library()
    cfg = moe.MoEConfig(hidden=100, ffn=256, n_experts=8, top_k=2, n_group=1, topk_group=1, ep_size=1)
    w = moe.MoEWeights()
    h = ctypes.c_void_p()
    assert L.moe_layer_create(ctypes.byref(cfg), ctypes.byref(w), ctypes.byref(h)) == -2
    assert b"hidden" in L.moe_last_error()
    cfg.hidden = 128
    cfg.top_k = 9
    assert L.moe_layer_create(ctypes.byref(cfg), ctypes.byref(w), ctypes.byref(h)) == -1
    assert L.moe_layer_destroy(None) == 0


def test_struct_layout_matches_header(tmp_path):
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    probe = tmp_path / "probe.c"
    fields = {"moe_layer_config": moe.MoEConfig, "moe_layer_weights": moe.MoEWeights,
              "moe_routing_out": moe.MoERouting, "moe_layer_info": moe.MoEInfo}
    lines = ["#include <stdio.h>", "#include <stddef.h>", f'#include "{HEADER}"', "int main(void){"]
    for cname, py in fields.items():
        lines.append(f'printf("{cname} %zu\\n", sizeof({cname}));')
        for fname, _ in py._fields_:
            lines.append(f'printf("{cname}.{fname} %zu\\n", offsetof({cname}, {fname}));')
    lines.append("return 0;}")
    probe.write_text("\n".join(lines))
    exe = tmp_path / "probe"
    subprocess.run(["gcc", str(probe), "-o", str(exe)], check=True)
    got = dict(l.split() for l in subprocess.run([str(exe)], capture_output=True, text=True).stdout.splitlines())
    for cname, py in fields.items():
        assert int(got[cname]) == ctypes.sizeof(py), cname
        for fname, _ in py._fields_:
            assert int(got[f"{cname}.{fname}"]) == getattr(py, fname).offset, f"{cname}.{fname}"
