"""CPU-only checks of the C-ABI library: it loads, exports every symbol include/astra.h declares,
reports parameter layouts that agree with the oracle's definitions, and rejects bad arguments
synchronously with the documented status codes (no compute calls: there is no GPU here)."""
import ctypes
import os
import re

import pytest

import paper_conf_asplos_sivathanucsz19_b200 as A
from oracle import cells as C

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    src = open(os.path.join(ROOT, "include", "astra.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(astra_[a-z0-9_]+)\s*\(", src)))


def test_library_loads_and_exports_every_declared_symbol():
    L = A.lib()
    syms = _declared_symbols()
    assert len(syms) >= 30
    missing = [s for s in syms if not hasattr(L, s)]
    assert not missing, missing
    # and the binding wraps all of them
    assert set(syms) <= set(A._SIGS), set(syms) - set(A._SIGS)


def test_library_is_sm100a():
    """The .so carries sm_100a SASS with tcgen05 MMAs and TMA loads (cuobjdump, no GPU needed)."""
    import shutil
    import subprocess
    cu = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(cu):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([cu, "-sass", A.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert "UTCHMMA" in out and "UTMALDG" in out and "LDTM" in out


@pytest.mark.parametrize("cell,shapes,kw", [
    ("milstm", C.milstm_param_shapes(32, 64), {}),
    ("lstm", C.lstm_param_shapes(32, 64), {}),
    ("sublstm", C.lstm_param_shapes(32, 64), {}),
    ("scrn", C.scrn_param_shapes(32, 64, 40), {"context": 40}),
    ("rhn", C.rhn_param_shapes(32, 64, 3), {"depth": 3}),
])
def test_param_layout_matches_oracle(cell, shapes, kw):
    import numpy as np
    c = A.Cell(cell, 64, 32, 4, 8, dtype="fp32", allocate=False, **kw)
    assert set(c.param_info) == set(shapes)
    prev_end = 0
    for name, (off, r, cc) in sorted(c.param_info.items(), key=lambda kv: kv[1][0]):
        shp = shapes[name]
        assert r * cc == int(np.prod(shp))
        if len(shp) == 3:   # RHN R[ℓ] stacked: [L·H][2H]
            assert (r, cc) == (shp[0] * shp[1], shp[2])
        else:
            assert (r, cc) == ((shp[0], shp[1]) if len(shp) == 2 else (1, shp[0]))
        assert off % 64 == 0 and off >= prev_end
        prev_end = off + r * cc
    assert c.n_params >= prev_end


def test_workspace_scales_with_shape():
    a = A.Cell("milstm", 64, 32, 4, 8, dtype="bf16", allocate=False)
    b = A.Cell("milstm", 64, 32, 4, 16, dtype="bf16", allocate=False)
    assert b.saved_bytes > a.saved_bytes and b.scratch_bytes >= a.scratch_bytes


def test_bad_arguments_are_rejected():
    L = A.lib()
    h = ctypes.c_void_p()
    assert L.astra_cell_create(ctypes.byref(h), 1, 0, 32, 4, 8) == 1          # E_ARG: hidden = 0
    assert L.astra_cell_create(ctypes.byref(h), 99, 64, 32, 4, 8) == 1         # E_ARG: unknown cell
    assert "unknown" in L.astra_last_error().decode()
    assert L.astra_cell_create(None, 1, 64, 32, 4, 8) == 1
    with pytest.raises(A.AstraError):
        A.Cell("milstm", 64, 32, 4, 8, dtype="fp32", allocate=False).forward(None)   # E_STATE: not bound
    c = A.Cell("milstm", 64, 32, 4, 8, dtype="fp32", allocate=False)
    assert L.astra_tune_mode(c.h, 7, None) == 1
    assert L.astra_tune_mode(c.h, 2, b"a1=100") == 1
    assert L.astra_tune_mode(c.h, 2, b"a1=256.8.2") == 1
    assert L.astra_tune_mode(c.h, 2, b"nonsense=1") == 1
    assert L.astra_status_string(4) == b"ASTRA_E_CUDA"
    # peer-memory backend (K11p): handle before bind, init before handle, short buffer, null handles
    buf = ctypes.create_string_buffer(256)
    assert L.astra_comm_peer_handle(c.h, buf, 256) == 3                        # E_STATE: not bound
    assert L.astra_comm_peer_init(c.h, buf, 0, 2) == 3                          # E_STATE: no handle yet
    assert L.astra_comm_peer_handle(c.h, buf, 16) in (1, 3)
    assert L.astra_comm_peer_handle(c.h, None, 256) == 1                        # E_ARG: null buffer
    assert L.astra_debug_set_trace(7, None) == 1                                # E_ARG: unknown trace kind
    assert L.astra_debug_set_trace(0, None) == 0                                # tracing off


def test_tune_report_is_json():
    c = A.Cell("milstm", 64, 32, 4, 8, dtype="bf16", allocate=False)
    c.tune_mode(A.TUNE_FROZEN, "a1=128.2.2,rec=256.4.1,wg_side=1")
    r = c.tune_report()
    assert "a1=128.2.2" in r["variant"] and "rec=256.4.1" in r["variant"] and "wg_side=1" in r["variant"]


def test_strided_tensor_refused():
    """The C ABI takes dense row-major buffers: a strided view (numpy fancy indexing yields one) must
    be refused by the binding, never silently read in the wrong order."""
    import numpy as np
    import torch
    a = np.arange(18, dtype=np.int32).reshape(9, 2)[:, np.array([0, 1, 0, 1])]
    t = torch.as_tensor(a)
    assert not t.is_contiguous()
    with pytest.raises(ValueError):
        A._ptr(t)
    assert A._ptr(t.contiguous()) is not None
