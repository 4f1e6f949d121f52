"""ctypes loader for libtfhe_b200.so (the C ABI in include/tfhe_b200.h) and its nvcc build.

The product path has no CPU fallback: if the shared library is missing or no sm_100 device is present,
every entry point raises.  Argument marshalling only -- all gate arithmetic runs in the CUDA kernels.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

_PKG = os.path.dirname(os.path.abspath(__file__))
_CSRC = os.path.join(_PKG, "csrc")
_ROOT = os.path.dirname(_PKG)
SO_PATH = os.path.join(_PKG, "libtfhe_b200.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17", "-Xcompiler", "-fPIC",
              "-shared", "-cudart", "static"]

TB_OK, TB_EINVAL, TB_EUNSUPPORTED, TB_ENOKEYS, TB_ECUDA, TB_ENOMEM = 0, -1, -2, -3, -4, -5
ERRORS = {TB_EINVAL: "EINVAL", TB_EUNSUPPORTED: "EUNSUPPORTED", TB_ENOKEYS: "ENOKEYS", TB_ECUDA: "ECUDA",
          TB_ENOMEM: "ENOMEM"}


def _sources():
    out = [os.path.join(_ROOT, "include", "tfhe_b200.h")]
    for f in sorted(os.listdir(_CSRC)):
        if f.endswith((".cu", ".cuh")):
            out.append(os.path.join(_CSRC, f))
    return out


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile csrc/tb_lib.cu into libtfhe_b200.so for sm_100a (in-tree, so it travels with the repo)."""
    if not force and os.path.exists(SO_PATH) and os.path.getmtime(SO_PATH) >= max(
            os.path.getmtime(p) for p in _sources()):
        return SO_PATH
    tmp = SO_PATH + ".tmp%d" % os.getpid()
    cmd = [NVCC] + NVCC_FLAGS + ["-o", tmp, os.path.join(_CSRC, "tb_lib.cu")]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd)
    os.replace(tmp, SO_PATH)
    return SO_PATH


class TBError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__("tfhe_b200 %s (%d): %s" % (ERRORS.get(code, "?"), code, msg))
        self.code = code


class Params(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int32) for k in ("n", "N", "k", "l", "Bgbit", "ks_t", "ks_basebit")]


class Netlist(ctypes.Structure):
    _fields_ = [("n_inputs", ctypes.c_int64), ("n_gates", ctypes.c_int64), ("type", ctypes.c_void_p),
                ("in0", ctypes.c_void_p), ("in1", ctypes.c_void_p), ("in2", ctypes.c_void_p)]


# every symbol the header declares: (restype, argtypes)
_vp, _i32, _i64, _sz = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_size_t
_pi64 = ctypes.POINTER(ctypes.c_int64)
SIGNATURES = {
    "tb_default_params": (Params, []),
    "tb_ctx_create": (ctypes.c_int, [ctypes.POINTER(Params), ctypes.c_int, ctypes.POINTER(_vp)]),
    "tb_ctx_destroy": (ctypes.c_int, [_vp]),
    "tb_load_bk": (ctypes.c_int, [_vp, _vp, _sz]),
    "tb_load_ksk": (ctypes.c_int, [_vp, _vp, _sz]),
    "tb_gates": (ctypes.c_int, [_vp, ctypes.c_int, _vp, _vp, _vp, _vp, _i64, _i64, _vp]),
    "tb_gates_host": (ctypes.c_int, [_vp, ctypes.c_int, _vp, _vp, _vp, _vp, _i64, _i64]),
    "tb_levelise": (ctypes.c_int, [ctypes.POINTER(Netlist), _vp, _pi64]),
    "tb_netlist_plan": (ctypes.c_int, [ctypes.POINTER(Netlist), _pi64, _vp, _vp]),
    "tb_netlist_plan_capacity": (ctypes.c_int, [ctypes.POINTER(Netlist), _i64, _pi64, _vp, _vp]),
    "tb_netlist_upload":(ctypes.c_int, [_vp, ctypes.POINTER(Netlist), ctypes.POINTER(_vp)]),
    "tb_netlist_free": (ctypes.c_int, [_vp, _vp]),
    "tb_netlist_info": (ctypes.c_int, [_vp, _pi64, _pi64]),
    "tb_netlist_wire_rows": (ctypes.c_int, [_vp, _vp]),
    "tb_netlist_level": (ctypes.c_int, [_vp, _i64, _pi64, _pi64, _pi64, _pi64]),
    "tb_run_level": (ctypes.c_int, [_vp, _vp, _i64, _i64, _i64, _vp, _i64, _vp]),
    "tb_run_netlist": (ctypes.c_int, [_vp, _vp, _vp, _i64, _vp]),
    "tb_set_peer_wires": (ctypes.c_int, [_vp, _vp, _vp, ctypes.c_int]),
    "tb_ipc_export": (ctypes.c_int, [_vp, _vp, _pi64]),
    "tb_ipc_import": (ctypes.c_int, [_vp, _vp, _i64, ctypes.POINTER(_vp), ctypes.POINTER(_vp)]),
    "tb_ipc_close": (ctypes.c_int, [_vp, _vp]),
    "tb_run_netlist_host": (ctypes.c_int, [_vp, _vp, _vp, _i64, _vp, _i64, _vp, _i64]),
    "tb_profile_enable": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tb_profile_read": (ctypes.c_int, [_vp, ctypes.POINTER(ctypes.c_double), _pi64, ctypes.POINTER(ctypes.c_double),
                                       _pi64]),
    "tb_bootstrap_wo_ks": (ctypes.c_int, [_vp, _vp, _i64, _vp, _i64, _i64, _vp]),
    "tb_keyswitch": (ctypes.c_int, [_vp, _vp, _i64, _vp, _i64, _i64, _vp]),
    "tb_ntt_muladd6": (ctypes.c_int, [_vp, _vp, _vp, _vp]),
    "tb_fft_muladd6": (ctypes.c_int, [_vp, _vp, _vp, _vp]),
    "tb_set_lanes_per_cta": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tb_br6_lanes_per_cta": (ctypes.c_int, [_vp, ctypes.c_int64]),
    "tb_set_br_variant": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tb_set_ks_tile": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tb_set_narrow_lanes": (ctypes.c_int, [_vp, _i64]),
    "tb_set_narrow_kernel": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tb_set_level_capacity": (ctypes.c_int, [_vp, _i64]),
    "tb_key_bytes": (ctypes.c_int, [_vp, ctypes.POINTER(_sz)]),
    "tb_microbench_fields": (ctypes.c_int, [_vp, ctypes.c_int, ctypes.POINTER(ctypes.c_double)]),
    "tb_tc_mma_test": (ctypes.c_int, [_vp, _vp, _vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                      ctypes.c_int, _vp]),
    "tb_tc_muladd": (ctypes.c_int, [_vp, _vp, _vp, _vp]),
    "tb_set_plan_world": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tb_netlist_world": (ctypes.c_int, [_vp, ctypes.POINTER(ctypes.c_int)]),
    "tb_netlist_early": (ctypes.c_int, [_vp, _i64, ctypes.c_int, ctypes.POINTER(_i64)]),
    "tb_netlist_plan_world": (ctypes.c_int, [_vp, _i64, ctypes.c_int, ctypes.POINTER(_i64), _vp, _vp, _vp]),
    "tb_set_host_overlap": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tb_microbench": (ctypes.c_int, [_vp, ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                                     ctypes.POINTER(ctypes.c_double)]),
    "tb_last_error": (ctypes.c_char_p, []),
    "tb_version": (ctypes.c_char_p, []),
}

_lib = None


def lib():
    """Load the in-tree shared library (raises if it has not been built)."""
    global _lib
    if _lib is None:
        path = os.environ.get("TB_LIB", SO_PATH)     # A/B timing of alternative builds (tools/ab.sh)
        if not os.path.exists(path):
            raise RuntimeError("%s is not built (run __graft_entry__.build()); there is no CPU fallback" % path)
        L = ctypes.CDLL(path)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(rc: int) -> None:
    if rc != TB_OK:
        raise TBError(rc, lib().tb_last_error().decode(errors="replace"))
