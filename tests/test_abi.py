"""C-ABI boundary checks that need no GPU (include/sf.h vs the built library / binding).

- the library builds for sm_100a and loads; every function declared in sf.h is exported
  and declared in the ctypes binding with the same name;
- SASS of the library contains tcgen05 MMAs (UTCHMMA) and TMEM loads (LDTM);
- enum values in sf.h equal the codes of sf_inputs.ir (the workload spec);
- ctypes struct sizes / field offsets equal the C compiler's (gcc, sizeof / offsetof);
- the binding fails loudly without the library (no CPU fallback).
"""
import ctypes
import os
import re
import subprocess
import tempfile

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "sf.h")


@pytest.fixture(scope="module")
def built():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_middleware_wur0hdh21_b200 import _abi
    return _abi


def header_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:sf_status|void|const char\*|int32_t|uint64_t)\s+(sf_\w+)\s*\(",
                                 src, flags=re.M)))


def test_every_header_symbol_exported_and_bound(built):
    names = header_functions()
    assert len(names) >= 30
    L = built.lib()
    for n in names:
        assert hasattr(L, n), n
        assert n in built.PROTOTYPES, f"{n} missing from the ctypes binding"
    assert sorted(built.PROTOTYPES) == names
    assert L.sf_abi_version() == 1


def test_sass_has_tcgen05(built):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", built.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "UTCHMMA" in out and "LDTM" in out
    assert "HMMA" not in out.replace("UTCHMMA", "")  # no legacy mma.sync path


def test_enum_values_match_workload_codes():
    from sf_inputs import ir
    src = open(HEADER).read()
    vals = dict(re.findall(r"(SF_[A-Z0-9_]+)\s*=\s*(\d+)", src))
    for name in ("PARAM", "SLOT", "SCALAR_STATE", "DATASET", "INPUT", "LABEL", "ACT", "GRAD", "OUTPUT"):
        assert int(vals["SF_" + name]) == getattr(ir, name)
    for name in ("GEMM", "BIAS_ACT", "BIAS_ACT_BWD", "COLSUM", "SOFTMAX_CE", "SOFTMAX", "SGD_MOM",
                 "ADAM", "FEED", "STEP_INC"):
        assert int(vals["SF_OP_" + name]) == getattr(ir, name)
    assert int(vals["SF_F32"]) == ir.F32 and int(vals["SF_I32"]) == ir.I32
    defs = dict(re.findall(r"#define\s+(SF_\w+)\s+\(?(-?\d+)\)?", src))
    assert int(defs["SF_GEMM_TA"]) == ir.TA and int(defs["SF_GEMM_TB"]) == ir.TB
    assert int(defs["SF_GEMM_ACC"]) == ir.ACC and int(defs["SF_ACT_RELU"]) == ir.RELU
    assert int(defs["SF_ACT_GELU"]) == ir.GELU


def test_struct_layouts_match_c(built):
    structs = ["sf_tensor_desc", "sf_op_desc", "sf_graph_desc", "sf_config", "sf_partition_opts",
               "sf_partition_info", "sf_job_info", "sf_cut_info", "sf_timing", "sf_trace_event",
               "sf_cut_request", "sf_copy_desc", "sf_feed_desc", "sf_u8_stage", "sf_gemm_path",
               "sf_migration_probe", "sf_slot_info"]
    lines = ['#include <stdio.h>', '#include <stddef.h>', f'#include "{HEADER}"', "int main(){"]
    for s in structs:
        lines.append(f'printf("{s} %zu\\n", sizeof({s}));')
        for f, _ in getattr(built, s)._fields_:
            cf = "in" if f == "in_" else f
            lines.append(f'printf("{s}.{f} %zu\\n", offsetof({s}, {cf}));')
    lines.append("return 0;}")
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "t.c")
        open(c, "w").write("\n".join(lines))
        exe = os.path.join(d, "t")
        subprocess.run(["gcc", "-std=c99", c, "-o", exe], check=True)
        out = subprocess.run([exe], capture_output=True, text=True, check=True).stdout
    got = dict(l.split() for l in out.strip().splitlines())
    for s in structs:
        cls = getattr(built, s)
        assert int(got[s]) == ctypes.sizeof(cls), s
        for f, _ in cls._fields_:
            assert int(got[f"{s}.{f}"]) == getattr(cls, f).offset, f"{s}.{f}"


def test_missing_library_fails_loudly(monkeypatch, built):
    monkeypatch.setattr(built, "_lib", None)
    monkeypatch.setattr(built, "LIB_PATH", "/nonexistent/libswitchflow_b200.so")
    with pytest.raises(RuntimeError, match="no CPU fallback"):
        built.lib()


def test_create_without_gpu_reports_cuda_error(built):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
    with pytest.raises(built.SFError):
        Runtime([0])


def test_builtin_host_stage_equals_oracle(built):
    """sf_stage_u8_normalize (host code, no GPU) is bit-identical to oracle/feed.py."""
    import numpy as np
    from oracle import feed as FD
    from sf_inputs import data as D
    imgs, labels = D.u8_images(96, 28 * 28, 10, seed=3)
    st = built.sf_u8_stage(imgs.ctypes.data, labels.ctypes.data, 96, 32, 784, 28, 77)
    x = np.empty((32, 784), np.float32)
    y = np.empty((32, 1), np.int32)
    dst = (ctypes.c_void_p * 2)(x.ctypes.data, y.ctypes.data)
    nb = (ctypes.c_uint64 * 2)(x.nbytes, y.nbytes)
    for it in (0, 1, 2, 5):
        assert built.lib().sf_stage_u8_normalize(ctypes.addressof(st), it, dst, nb, 2) == 0
        rx, ry = FD.u8_stage(imgs, labels, it, 32, 28, seed=77)
        assert x.tobytes() == rx.tobytes() and y.tobytes() == ry.tobytes()
    nb[0] = 4  # size mismatch is an error, not a buffer overrun
    assert built.lib().sf_stage_u8_normalize(ctypes.addressof(st), 0, dst, nb, 2) != 0
