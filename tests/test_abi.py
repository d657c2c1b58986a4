"""CPU-side checks of the C-ABI library: it builds for sm_100a, exports every
symbol include/jigsaw.h declares, and validates arguments without a GPU."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_icpp_zhanglyfyllq24_b200 as jig

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    return jig.lib()


def test_header_declares_exactly_the_bound_symbols():
    hdr = open(os.path.join(ROOT, "include", "jigsaw.h")).read()
    declared = set(re.findall(r"JIGSAW_API\s+[\w\s\*]*?\b(jigsaw_\w+)\s*\(", hdr))
    assert declared == set(jig.ABI_SYMBOLS)


def test_library_exports_every_symbol(L):
    out = subprocess.run(["nm", "-D", "--defined-only", jig.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (jigsaw_\w+)", out))
    assert set(jig.ABI_SYMBOLS) <= exported
    for s in jig.ABI_SYMBOLS:
        assert hasattr(L, s)


def test_library_is_sm100a_tcgen05(L):
    """The SpMM kernel is real tcgen05 sparse MMA + TMA, compiled for sm_100a."""
    sass = subprocess.run(["cuobjdump", "-sass", jig.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in subprocess.run(["cuobjdump", "-lelf", jig.LIB_PATH], capture_output=True,
                                       text=True).stdout
    assert "UTCHMMA" in sass          # tcgen05.mma(.sp) kind::f16
    assert "UTMALDG" in sass or "UBLKCP" in sass   # TMA
    assert "LDTM" in sass             # tcgen05.ld


def test_version(L):
    assert "sm_100a" in jig.version()


def _status(L):
    return L.jigsaw_last_status(), L.jigsaw_last_error_string().decode()


def test_reorder_validates_arguments_before_touching_the_device(L):
    buf = np.zeros(64, np.uint16)
    p = buf.ctypes.data_as(ctypes.c_void_p)
    assert L.jigsaw_reorder(None, 8, 8, 1) is None
    assert _status(L)[0] == 1
    for (M, K, v) in [(0, 8, 1), (8, -1, 1), (8, 8, 3), (6, 8, 4)]:
        assert L.jigsaw_reorder(p, M, K, v) is None
        st, msg = _status(L)
        assert st == 1 and msg
    opt = jig.Options(64, 0)
    out = ctypes.c_void_p(0)
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 2
    opt = jig.Options(128, 7)
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 1
    opt = jig.Options(128, 0)
    opt.reserved[1] = 1
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 1
    opt = jig.Options(128, 0, 0, 0, 0, -1)             # cc_max_nnz must be >= 0
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 1
    opt = jig.Options(128, 0, 0, 0, 0, 1 << 24)        # ... and < 2^24
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 1
    opt = jig.Options(128, 0, 0, 0, 0, 16)             # valid: fails only for want of a device
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 2
    opt = jig.Options(128, 0, 2)                       # c_dtype must be 0 (fp16) or 1 (fp32)
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 1
    opt = jig.Options(128, 0, 0, 0, 256)               # autotune_n only with panel_rows = -1
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 1
    opt = jig.Options(-1, 0, 0, 0, 100)                # autotune_n must be a multiple of 8
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 1
    opt = jig.Options(-1, 0, 0, 0, 0)                  # valid: fails only for want of a device
    assert L.jigsaw_reorder_ex(p, 8, 8, 1, ctypes.byref(opt), None, ctypes.byref(out)) == 2


def test_binding_struct_layouts_match_header(tmp_path):
    """The ctypes structures of the binding have the sizes and field offsets the C
    compiler gives the structs of include/jigsaw.h (compiled here with gcc)."""
    structs = {"jigsaw_options_t": jig.Options, "jigsaw_info_t": jig.Info, "jigsaw_format_host_t": jig.FormatHost,
               "jigsaw_launch_desc_t": jig.LaunchDesc, "jigsaw_launch_override_t": jig.LaunchOverride}
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "jigsaw.h"', 'int main(void) {']
    for cname, py in structs.items():
        lines.append(f'  printf("{cname} size %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'  printf("{cname} {f} %zu\\n", offsetof({cname}, {f}));')
    lines.append("  return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c99", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = {}
    for line in subprocess.check_output([str(exe)], text=True).splitlines():
        c, f, v = line.split()
        got[(c, f)] = int(v)
    for cname, py in structs.items():
        assert got[(cname, "size")] == ctypes.sizeof(py), cname
        for f, _ in py._fields_:
            assert got[(cname, f)] == getattr(py, f).offset, (cname, f)


def test_launch_override_and_descriptor(L):
    """Diagnostic calls work without a device: the override is validated and
    per-thread, the launch descriptor readable."""
    for bad in [dict(tile_n=48), dict(split_k=3), dict(host_chunks=-1)]:
        with pytest.raises(jig.JigsawError) as e:
            jig.set_launch_override(**bad)
        assert e.value.status == 1
    o = jig.LaunchOverride(0, 0, 0, 0)
    o.reserved[1] = 5
    assert L.jigsaw_set_launch_override(ctypes.byref(o)) == 1
    with jig.launch_override(tile_n=64, split_k=2):
        pass
    assert L.jigsaw_set_launch_override(None) == 0
    d = jig.last_launch()
    assert set(d) >= {"launches", "tile_n", "split_k", "grid", "cta_pair", "dynamic_schedule", "split_slots"}


def test_spmm_validates_arguments(L):
    buf = np.zeros(64, np.uint16)
    p = buf.ctypes.data_as(ctypes.c_void_p)
    assert L.jigsaw_spmm(None, p, 8, p, None) == 1
    assert L.jigsaw_spmm_batched(None, None, None, None, -1, None) == 1
    assert L.jigsaw_spmm_batched(None, None, None, None, 0, None) == 0


def test_free_null_is_noop(L):
    L.jigsaw_free(None)


def test_no_gpu_is_reported_not_crashed(L):
    """Without an sm_100 device a valid call fails with UNSUPPORTED (no CPU fallback)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    buf = np.zeros(64, np.uint16)
    p = buf.ctypes.data_as(ctypes.c_void_p)
    assert L.jigsaw_reorder(p, 8, 8, 1) is None
    assert _status(L)[0] == 2


def test_product_does_not_reference_oracle():
    """The product package and library never import / link the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_zhanglyfyllq24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src
                assert "liboracle" not in src and "orc_" not in src
    out = subprocess.run(["ldd", jig.LIB_PATH], capture_output=True, text=True).stdout
    assert "oracle" not in out
