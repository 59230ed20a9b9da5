"""CPU oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package.  The product path
(``paper_conf_ipps_gavierrprs23_b200``) never imports it and shares no code with
it; the only common dependency is the seeded input generator ``workloads``.

``oracle.c`` is the plain gate-by-gate, lane-by-lane simulator (see its header for
the paper passages each rule follows); ``mobius.py`` is Algorithm 1 read literally.
Parity status of every function is listed in DESIGN.md §"Oracle pins".
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

from . import mobius  # noqa: F401  (re-export)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (-O2, OpenMP).  Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-std=c11", "-fopenmp", "-fPIC", "-shared",
                               "-Wall", "-Wextra", "-Wno-unused-parameter",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _Netlist(C.Structure):
    _fields_ = [("n_pi", C.c_uint32), ("n_reg", C.c_uint32), ("n_gates", C.c_uint32),
                ("n_po", C.c_uint32),
                ("reg_init", C.c_void_p), ("reg_d", C.c_void_p), ("gate_k", C.c_void_p),
                ("gate_in_off", C.c_void_p), ("gate_in", C.c_void_p), ("gate_tt", C.c_void_p),
                ("po", C.c_void_p), ("gate_tt_hi", C.c_void_p)]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = C.CDLL(build())
            u64, u32, i64 = C.c_uint64, C.c_uint32, C.c_int64
            for name, res, args in [
                ("orc_mix64", u64, [u64]),
                ("orc_stim_word", u64, [u64, u64, u64, u64]),
                ("orc_misr_step", u64, [u64, u64]),
                ("orc_lane_sig_term", u64, [u64, u64]),
                ("orc_mobius_def", None, [u64, C.c_int, C.c_void_p]),
                ("orc_mobius_def_wide", None, [C.c_void_p, C.c_int, C.c_void_p]),
                ("orc_poly_eval", i64, [C.c_void_p, C.c_int, u32]),
                ("orc_topo_order", C.c_int, [C.c_void_p, C.c_void_p]),
                ("orc_asap_levels", C.c_int, [C.c_void_p, C.c_void_p]),
                ("orc_simulate", i64, [C.c_void_p, C.c_int, u64, C.c_void_p, u64, u32,
                                       C.c_void_p, u32, C.c_int, C.c_void_p, C.c_void_p,
                                       C.c_void_p, C.c_void_p]),
                ("orc_max_threads", C.c_int, []),
            ]:
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _ptr(a):
    return a.ctypes.data_as(C.c_void_p) if a is not None else None


class _NL:
    """Keeps the contiguous arrays alive while the C struct points at them."""

    def __init__(self, nl):
        self.arrs = [np.ascontiguousarray(nl.reg_init, dtype=np.uint8),
                     np.ascontiguousarray(nl.reg_d, dtype=np.uint32),
                     np.ascontiguousarray(nl.gate_k, dtype=np.uint8),
                     np.ascontiguousarray(nl.gate_in_off, dtype=np.uint32),
                     np.ascontiguousarray(nl.gate_in, dtype=np.uint32),
                     np.ascontiguousarray(nl.gate_tt, dtype=np.uint64),
                     np.ascontiguousarray(nl.po, dtype=np.uint32)]
        hi = getattr(nl, "gate_tt_hi", None)
        self.arrs.append(None if hi is None else np.ascontiguousarray(hi, dtype=np.uint64))
        self.s = _Netlist(nl.n_pi, nl.n_reg, nl.n_gates, nl.n_po, *[_ptr(a) for a in self.arrs])

    @property
    def ref(self):
        return C.byref(self.s)


# ---------------------------------------------------------------- helpers

def mix64(z: int) -> int:
    return lib().orc_mix64(z & (2**64 - 1))


def stim_word(seed: int, p: int, c: int, w: int) -> int:
    return lib().orc_stim_word(seed, p, c, w)


def misr_step(sig: int, v: int) -> int:
    return lib().orc_misr_step(sig, v)


def lane_sig_sum(sigs, lanes) -> int:
    L = lib()
    tot = 0
    for sg, s in zip(np.asarray(sigs, dtype=np.uint64).tolist(), np.asarray(lanes).tolist()):
        tot = (tot + L.orc_lane_sig_term(int(sg), int(s))) & (2**64 - 1)
    return tot


def mobius_def(tt: int, k: int) -> list[int]:
    w = np.zeros(1 << k, dtype=np.int64)
    lib().orc_mobius_def(tt, k, _ptr(w))
    return w.tolist()


def mobius_def_wide(words, k: int) -> list[int]:
    """Definition of the coefficients for a table of up to 256 entries (4 uint64 words)."""
    t = np.zeros(4, dtype=np.uint64)
    t[:len(words)] = np.asarray(words, dtype=np.uint64)
    w = np.zeros(1 << k, dtype=np.int64)
    lib().orc_mobius_def_wide(_ptr(t), k, _ptr(w))
    return w.tolist()


def poly_eval(w, k: int, x: int) -> int:
    wa = np.ascontiguousarray(w, dtype=np.int64)
    return lib().orc_poly_eval(_ptr(wa), k, x)


def topo_order(nl) -> np.ndarray | None:
    n = _NL(nl)
    order = np.zeros(max(nl.n_gates, 1), dtype=np.uint32)
    rc = lib().orc_topo_order(n.ref, _ptr(order))
    return None if rc != 0 else order[:nl.n_gates]


def asap_levels(nl) -> np.ndarray | None:
    n = _NL(nl)
    lv = np.zeros(max(nl.n_gates, 1), dtype=np.uint32)
    rc = lib().orc_asap_levels(n.ref, _ptr(lv))
    return None if rc != 0 else lv[:nl.n_gates]


def max_threads() -> int:
    return lib().orc_max_threads()


def simulate(nl, lanes, cycles: int, seed: int = 0, host_stim=None, mode: str = "tt",
             threads: int = 0, want=("trace", "last", "regs", "sig")) -> dict:
    """Simulate the given global lanes for `cycles` cycles (see oracle.c orc_simulate).

    host_stim: optional uint64 array [cycles][n_pi][stim_words] (global word index).
    Returns a dict with 'trace' [nl][cycles][n_po] u8, 'last' [nl][n_po] u8,
    'regs' [nl][n_reg] u8, 'sig' [nl] u64 and 'violations' (mode 'poly').
    """
    n = _NL(nl)
    lanes = np.ascontiguousarray(lanes, dtype=np.uint64)
    nlanes = int(lanes.shape[0])
    out = {}
    trace = np.zeros((nlanes, cycles, nl.n_po), dtype=np.uint8) if "trace" in want else None
    last = np.zeros((nlanes, nl.n_po), dtype=np.uint8) if "last" in want else None
    regs = np.zeros((nlanes, nl.n_reg), dtype=np.uint8) if "regs" in want else None
    sig = np.zeros(nlanes, dtype=np.uint64) if "sig" in want else None
    stim, sw = None, 0
    if host_stim is not None:
        stim = np.ascontiguousarray(host_stim, dtype=np.uint64)
        assert stim.shape[0] >= cycles and stim.shape[1] == nl.n_pi
        sw = stim.shape[2]
        assert int(lanes.max(initial=0)) >> 6 < sw
    v = lib().orc_simulate(n.ref, 1 if mode == "poly" else 0, seed, _ptr(stim), sw, cycles,
                           _ptr(lanes), nlanes, threads, _ptr(trace), _ptr(last), _ptr(regs),
                           _ptr(sig))
    if v < 0:
        raise ValueError("oracle: invalid netlist (combinational loop or bad net id)")
    out.update(trace=trace, last=last, regs=regs, sig=sig, violations=int(v))
    return out
