"""CPU-side checks of the C ABI boundary: the library loads without a GPU and
exports every symbol include/scalfrag.h declares (no compute calls here)."""
import ctypes
import os
import re
import subprocess

import paper_conf_cluster_linwds24_b200 as sf

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "scalfrag.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sf_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    d = _declared()
    for name in ("sf_tensor_create", "sf_plan", "sf_mttkrp"):
        assert name in d


def test_library_exports_every_declared_symbol():
    L = sf.lib()
    out = subprocess.run(["nm", "-D", "--defined-only", sf._build.SO], capture_output=True, text=True).stdout
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    for name in _declared():
        assert name in exported, name
        assert hasattr(L, name)
    assert set(sf.EXPORTED) == set(_declared())


def test_status_strings_and_version():
    L = sf.lib()
    for code, name in sf.STATUS.items():
        assert L.sf_status_string(code).decode() == name
    assert "sm_100a" in sf.version()
    assert sf.kernel_launches() == 0  # nothing launched on a CPU box


def test_struct_layouts_match_header(tmp_path):
    """ctypes mirrors == the C compiler's layout of include/scalfrag.h (sizes and offsets)."""
    src = tmp_path / "sz.c"
    src.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "scalfrag.h"\n'
                   'int main(void) { printf("%zu %zu %zu %zu %zu %zu\\n", sizeof(sf_launch_t), '
                   'sizeof(sf_features_t), sizeof(sf_plan_info_t), offsetof(sf_launch_t, hot_kb), '
                   'offsetof(sf_plan_info_t, out_rows), offsetof(sf_plan_info_t, plan_ms)); return 0; }\n')
    exe = tmp_path / "sz"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = [int(x) for x in subprocess.check_output([str(exe)], text=True).split()]
    want = [ctypes.sizeof(sf.Launch), ctypes.sizeof(sf.Features), ctypes.sizeof(sf.PlanInfo),
            sf.Launch.hot_kb.offset, sf.PlanInfo.out_rows.offset, sf.PlanInfo.plan_ms.offset]
    assert got == want


def test_no_oracle_in_product_path():
    """The product package must not import or link anything under oracle/."""
    pkg = os.path.join(ROOT, "paper_conf_cluster_linwds24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle.c" not in txt and "liboracle" not in txt, f


def test_streamed_modes_argument_errors_without_gpu():
    """sf_mttkrp_streamed_modes rejects bad arguments before touching the device (the checks a
    C caller relies on: no output mode, a NULL factor a requested mode gathers, bad rank)."""
    import numpy as np
    import pytest
    dims = (4, 3, 2)
    inds = [np.zeros(5, np.uint32) for _ in dims]
    vals = np.ones(5, np.float32)
    facs = [np.ones((d, 16), np.float32) for d in dims]
    with pytest.raises(sf.SfError) as ei:
        sf.mttkrp_streamed_modes(dims, inds, vals, facs, [None, None, None], stream=0)
    assert ei.value.status == 1  # SF_ERR_INVALID_ARG
    out = np.zeros((4, 16), np.float32)
    with pytest.raises(sf.SfError) as ei:  # mode 0 gathers A_1: it must not be NULL
        sf.mttkrp_streamed_modes(dims, inds, vals, [facs[0], None, facs[2]], [out, None, None], stream=0)
    assert ei.value.status == 1
    L = sf.lib()
    d = (ctypes.c_uint64 * 3)(*dims)
    op = (ctypes.c_void_p * 3)(out.ctypes.data, None, None)
    fp = (ctypes.c_void_p * 3)(*[f.ctypes.data for f in facs])
    ip = (ctypes.c_void_p * 3)(*[a.ctypes.data for a in inds])
    assert L.sf_mttkrp_streamed_modes(3, d, 5, ip, vals.ctypes.data, fp, 0, op, 4, 2, None) == 1  # rank 0
    assert L.sf_mttkrp_streamed_modes(1, d, 5, ip, vals.ctypes.data, fp, 16, op, 4, 2, None) == 1  # nmodes 1
