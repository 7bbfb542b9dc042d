"""The C-ABI library loads and exports every symbol include/temco.h declares
(host only; no compute calls)."""
import ctypes
import os
import re

from paper_conf_icpp_songljkj0024_b200 import library_path


def test_every_declared_symbol_is_exported(root):
    hdr = open(os.path.join(root, "include", "temco.h")).read()
    declared = set(re.findall(r"^\s*(?:temco_status|const char\*)\s+(temco_\w+)\s*\(", hdr, re.M))
    assert {"temco_plan_create", "temco_run", "temco_peak_internal_bytes"} <= declared
    lib = ctypes.CDLL(library_path())
    for name in sorted(declared):
        assert hasattr(lib, name), name


def test_status_strings():
    lib = ctypes.CDLL(library_path())
    lib.temco_status_string.restype = ctypes.c_char_p
    assert lib.temco_status_string(0) == b"ok"
    assert lib.temco_status_string(7) == b"no device"


def test_library_is_sm100a(root):
    """The shipped kernels are sm_100a cubins (no PTX JIT, no other arch)."""
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", library_path()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_compute_calls_need_a_device():
    """No CPU fallback: a host-only plan (TEMCO_FLAG_NO_DEVICE) answers the planner queries but every
    compute entry point -- including the per-step verification hooks -- returns TEMCO_ERR_NO_DEVICE."""
    import workloads as W
    from paper_conf_icpp_songljkj0024_b200 import FLAG_NO_DEVICE, Plan
    from paper_conf_icpp_songljkj0024_b200.temco import _lib
    p = Plan(W.c1_basic_block(), flags=FLAG_NO_DEVICE)
    assert p.peak_internal_bytes(0) > 0
    nb = ctypes.c_int64(0)
    for st in (_lib.temco_run(p._h, ctypes.c_void_p(1), ctypes.c_void_p(1), None),
               _lib.temco_debug_step_output(p._h, ctypes.c_void_p(1), ctypes.c_void_p(1), None, 1, None, 0,
                                            ctypes.byref(nb)),
               _lib.temco_debug_step_tensor(p._h, ctypes.c_void_p(1), ctypes.c_void_p(1), None, 1, 0, None, 0,
                                            ctypes.byref(nb))):
        assert st == 7, st   # TEMCO_ERR_NO_DEVICE
