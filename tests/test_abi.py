"""The C-ABI library loads and exports every symbol include/pepp_spmv.h declares;
the ctypes structs match the C layout; no CPU fallback (CPU only)."""
from __future__ import annotations

import ctypes
import os
import re
import subprocess
import tempfile

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "pepp_spmv.h")


def _declared_functions() -> list[str]:
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_]*\s*\**\s*(pepp_[a-z0-9_]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_header_declares_core_calls():
    names = _declared_functions()
    for n in ["pepp_spmv_plan", "pepp_spmv_exec", "pepp_spmv_select", "pepp_spmv_destroy", "pepp_status_str",
              "pepp_spmv_exec_host", "pepp_partition_rows", "pepp_halo_ghosts", "pepp_history_select"]:
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_sc_dastgeerlk12_b200 import _capi
    L = _capi.lib()
    declared = _declared_functions()
    missing = [n for n in declared if not hasattr(L, n)]
    assert not missing, missing
    # the binding covers every declared symbol too
    assert sorted(_capi.SIGNATURES) == declared
    out = subprocess.run(["nm", "-D", "--defined-only", _capi.LIB_PATH], capture_output=True, text=True).stdout
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    assert set(declared) <= exported
    # nothing else leaks out of the C-ABI namespace (hidden visibility)
    assert {e for e in exported if e.startswith("pepp_")} == set(declared)


def test_abi_version_and_status_strings():
    from paper_conf_sc_dastgeerlk12_b200 import _capi
    L = _capi.lib()
    assert L.pepp_abi_version() == _capi.ABI_VERSION == 10
    for s in [0, -1, -2, -3, -4, -5, -6]:
        assert L.pepp_status_str(s).decode().startswith("PEPP_")


def test_struct_layouts_match_c():
    """Every field of every ctypes mirror sits at the C offset (generated from
    the mirrors' _fields_, so a field added on one side only fails here)."""
    from paper_conf_sc_dastgeerlk12_b200 import _capi as C
    structs = {"pepp_csr_t": C.CSR_T, "pepp_spmv_opts_t": C.OPTS_T, "pepp_choice_t": C.CHOICE_T,
               "pepp_plan_info_t": C.INFO_T}
    lines = []
    for cname, py in structs.items():
        lines.append(f'printf("{cname} %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'printf("{cname}.{f} %zu\\n", offsetof({cname}, {f}));')
    probe = ("#include <stdio.h>\n#include <stddef.h>\n#include \"pepp_spmv.h\"\nint main(void) {\n" +
             "\n".join(lines) + '\nprintf("x_p2p %d\\n", (int)PEPP_X_P2P);\nreturn 0;\n}\n')
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "p.c")
        open(c, "w").write(probe)
        exe = os.path.join(d, "p")
        subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        vals = dict(l.rsplit(" ", 1) for l in subprocess.check_output([exe], text=True).splitlines())
    for cname, py in structs.items():
        assert int(vals[cname]) == ctypes.sizeof(py), cname
        for f, _ in py._fields_:
            assert int(vals[f"{cname}.{f}"]) == getattr(py, f).offset, f"{cname}.{f}"
    # and the C structs have no field the mirrors lack (sizes match, offsets ascend)
    assert int(vals["x_p2p"]) == C.X_P2P


def test_sm100a_cubin_present():
    """The library carries sm_100a SASS (not PTX-only, not another arch)."""
    from paper_conf_sc_dastgeerlk12_b200 import _capi
    out = subprocess.run(["cuobjdump", "--list-elf", _capi.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_no_cpu_fallback_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present: the CUDA path runs")
    import gen
    from paper_conf_sc_dastgeerlk12_b200 import Plan, PeppError, _capi
    A = gen.laplacian2d(8)
    with pytest.raises(PeppError) as e:
        Plan.from_csr(A)
    assert e.value.status == _capi.PEPP_E_CUDA


def test_product_path_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sc_dastgeerlk12_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", txt).lower() or f == "__init__.py" and \
                    "import oracle" not in txt, f


def test_invalid_arguments_rejected_on_host():
    """Argument checks that need no device."""
    from paper_conf_sc_dastgeerlk12_b200 import _capi as C
    L = C.lib()
    h = ctypes.c_void_p()
    assert L.pepp_spmv_plan(None, None, ctypes.byref(h)) == C.PEPP_E_INVALID
    assert L.pepp_spmv_exec(None, None, None, 0, None, None, None) == C.PEPP_E_INVALID
    assert L.pepp_spmv_destroy(None) == C.PEPP_OK
    rp = np.array([0, 2, 1], dtype=np.int64)
    b = np.zeros(3, dtype=np.int64)
    assert L.pepp_partition_rows(rp.ctypes.data, 2, 5, 2, b.ctypes.data) == C.PEPP_E_INVALID  # row_ptr[0] != first


def test_oversized_block_refused_before_touching_memory():
    """nnz >= 2^31 in one block is refused (PEPP_E_UNSUPPORTED, reading A3)
    by the argument checks, before any pointer is dereferenced."""
    from paper_conf_sc_dastgeerlk12_b200 import _capi as C
    L = C.lib()
    dummy = np.zeros(4, dtype=np.int64)
    A = C.CSR_T(10, 10, 1 << 31, 0, dummy.ctypes.data, dummy.ctypes.data, dummy.ctypes.data, 0, 0)
    h = ctypes.c_void_p()
    assert L.pepp_spmv_plan(ctypes.byref(A), None, ctypes.byref(h)) == C.PEPP_E_UNSUPPORTED
    A.nnz, A.value_type = 4, 7                      # unknown value type
    assert L.pepp_spmv_plan(ctypes.byref(A), None, ctypes.byref(h)) == C.PEPP_E_INVALID
