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
    assert L.pepp_abi_version() == _capi.ABI_VERSION == 5
    for s in [0, -1, -2, -3, -4, -5, -6]:
        assert L.pepp_status_str(s).decode().startswith("PEPP_")


def test_struct_layouts_match_c():
    from paper_conf_sc_dastgeerlk12_b200 import _capi as C
    probe = r"""
#include <stdio.h>
#include <stddef.h>
#include "pepp_spmv.h"
#define P(T, f) printf(#T "." #f " %zu\n", offsetof(T, f));
int main(void) {
  printf("csr %zu\nopts %zu\nchoice %zu\ninfo %zu\n", sizeof(pepp_csr_t), sizeof(pepp_spmv_opts_t),
         sizeof(pepp_choice_t), sizeof(pepp_plan_info_t));
  P(pepp_csr_t, on_device) P(pepp_spmv_opts_t, row_bounds) P(pepp_spmv_opts_t, exchange)
  P(pepp_spmv_opts_t, history_path) P(pepp_spmv_opts_t, prune) P(pepp_choice_t, predicted_us) P(pepp_choice_t, launches) P(pepp_plan_info_t, key)
  P(pepp_plan_info_t, sell_fill) P(pepp_plan_info_t, halo_send) P(pepp_plan_info_t, sell_col16_frac) P(pepp_plan_info_t, prior_key) P(pepp_plan_info_t, sell_stencil_frac)
  P(pepp_spmv_opts_t, overlap) P(pepp_plan_info_t, overlap) P(pepp_plan_info_t, overlap_head) P(pepp_plan_info_t, overlap_tail)
  P(pepp_spmv_opts_t, predict) P(pepp_spmv_opts_t, predict_user) P(pepp_plan_info_t, predicted)
  P(pepp_spmv_opts_t, compress_values) P(pepp_plan_info_t, sell_constval_frac) P(pepp_plan_info_t, p2p_buffers) P(pepp_plan_info_t, sell_long_rows) P(pepp_plan_info_t, sell_cap)
  printf("x_p2p %d\n", (int)PEPP_X_P2P);
  return 0;
}
"""
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "p.c")
        open(c, "w").write(probe)
        exe = os.path.join(d, "p")
        subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        vals = dict(l.rsplit(" ", 1) for l in subprocess.check_output([exe], text=True).splitlines())
    assert int(vals["csr"]) == ctypes.sizeof(C.CSR_T)
    assert int(vals["opts"]) == ctypes.sizeof(C.OPTS_T)
    assert int(vals["choice"]) == ctypes.sizeof(C.CHOICE_T)
    assert int(vals["info"]) == ctypes.sizeof(C.INFO_T)
    assert int(vals["pepp_csr_t.on_device"]) == C.CSR_T.on_device.offset
    assert int(vals["pepp_spmv_opts_t.row_bounds"]) == C.OPTS_T.row_bounds.offset
    assert int(vals["pepp_spmv_opts_t.exchange"]) == C.OPTS_T.exchange.offset
    assert int(vals["pepp_spmv_opts_t.history_path"]) == C.OPTS_T.history_path.offset
    assert int(vals["pepp_spmv_opts_t.prune"]) == C.OPTS_T.prune.offset
    assert int(vals["pepp_choice_t.predicted_us"]) == C.CHOICE_T.predicted_us.offset
    assert int(vals["pepp_choice_t.launches"]) == C.CHOICE_T.launches.offset
    assert int(vals["pepp_plan_info_t.key"]) == C.INFO_T.key.offset
    assert int(vals["pepp_plan_info_t.sell_fill"]) == C.INFO_T.sell_fill.offset
    assert int(vals["pepp_plan_info_t.halo_send"]) == C.INFO_T.halo_send.offset
    assert int(vals["pepp_plan_info_t.sell_col16_frac"]) == C.INFO_T.sell_col16_frac.offset
    assert int(vals["pepp_plan_info_t.prior_key"]) == C.INFO_T.prior_key.offset
    assert int(vals["pepp_plan_info_t.sell_stencil_frac"]) == C.INFO_T.sell_stencil_frac.offset
    for f in ("overlap", "overlap_head", "overlap_tail"):
        assert int(vals["pepp_plan_info_t." + f]) == getattr(C.INFO_T, f).offset
    assert int(vals["pepp_spmv_opts_t.overlap"]) == C.OPTS_T.overlap.offset
    assert int(vals["pepp_spmv_opts_t.predict"]) == C.OPTS_T.predict.offset
    assert int(vals["pepp_spmv_opts_t.predict_user"]) == C.OPTS_T.predict_user.offset
    assert int(vals["pepp_plan_info_t.predicted"]) == C.INFO_T.predicted.offset
    assert int(vals["pepp_spmv_opts_t.compress_values"]) == C.OPTS_T.compress_values.offset
    assert int(vals["pepp_plan_info_t.sell_constval_frac"]) == C.INFO_T.sell_constval_frac.offset
    assert int(vals["pepp_plan_info_t.p2p_buffers"]) == C.INFO_T.p2p_buffers.offset
    assert int(vals["pepp_plan_info_t.sell_long_rows"]) == C.INFO_T.sell_long_rows.offset
    assert int(vals["pepp_plan_info_t.sell_cap"]) == C.INFO_T.sell_cap.offset
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
