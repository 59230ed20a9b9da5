"""Python binding of the gsim C-ABI (include/gsim.h) — argument marshalling only.

Every step of the simulation runs inside ``libgsim.so`` (host compiler in C++, the
hot path in sm_100a CUDA kernels).  This module loads the library with ctypes and
exposes the C functions under their C names (``gs_*``), plus thin handle wrappers
(:class:`Netlist`, :class:`Program`, :class:`Sim`) whose methods are one C call each.
PyTorch is used only to own the device workspace and to supply the CUDA stream.

There is NO fallback: if ``libgsim.so`` is missing or a call fails, an exception is
raised.  Build with ``python -m paper_conf_ipps_gavierrprs23_b200._build`` or
``__graft_entry__.build()``.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libgsim.so")

GS_OK = 0
GS_ERR_ARG, GS_ERR_ARITY, GS_ERR_UNDRIVEN, GS_ERR_COMB_LOOP = -1, -2, -3, -4
GS_ERR_BUFFER_TOO_SMALL, GS_ERR_CUDA, GS_ERR_STATE, GS_ERR_NOMEM = -5, -6, -7, -8
GS_MAX_K = 6
GS_MAX_K_POLY = 8
GS_SIM_NO_PDL = 1
GS_SIM_NO_GRID_STRIDE = 8     # kernel A: one CTA per work chunk (A/B measurement only)
GS_SIM_TILE_DESC_GLOBAL = 16  # kernel T: descriptors read from global memory
GS_SIM_TILE_DESC_TMA = 32     # kernel T: descriptors TMA-streamed level by level
GS_SIM_TILE_DESC_RESIDENT = 512  # kernel T: descriptor table resident in shared memory
GS_KERNEL_AUTO, GS_KERNEL_LUT, GS_KERNEL_POLY, GS_KERNEL_AB, GS_KERNEL_TILE, GS_KERNEL_CLUSTER = 0, 1, 2, 3, 5, 6
KERNELS = {"auto": 0, "lut": 1, "A": 1, "poly": 2, "B": 2, "ab": 3, "AB": 3, "tile": 5, "T": 5,
           "cluster": 6, "C": 6}


class GsError(RuntimeError):
    def __init__(self, code: int, fn: str, msg: str):
        super().__init__(f"{fn} -> {code}: {msg}")
        self.code = code


# ------------------------------------------------------------------ C structs
class gs_netlist_arrays(C.Structure):
    _fields_ = [("n_pi", C.c_uint32), ("n_reg", C.c_uint32), ("n_gates", C.c_uint32),
                ("n_po", C.c_uint32), ("reg_init", C.c_void_p), ("reg_d", C.c_void_p),
                ("gate_k", C.c_void_p), ("gate_in_off", C.c_void_p), ("gate_in", C.c_void_p),
                ("gate_tt", C.c_void_p), ("po", C.c_void_p), ("gate_tt_hi", C.c_void_p)]


class gs_netlist_counts(C.Structure):
    _fields_ = [("n_nets", C.c_uint32), ("n_pi", C.c_uint32), ("n_reg", C.c_uint32),
                ("n_gates", C.c_uint32), ("n_po", C.c_uint32), ("n_edges", C.c_uint64)]


class gs_compile_opts(C.Structure):
    _fields_ = [("balance", C.c_int), ("max_k", C.c_uint32), ("lut_k", C.c_uint32), ("level_seed", C.c_uint64)]


class gs_program_info(C.Structure):
    _fields_ = [("n_pi", C.c_uint32), ("n_reg", C.c_uint32), ("n_po", C.c_uint32),
                ("n_gates", C.c_uint32), ("n_eval_gates", C.c_uint32), ("n_levels", C.c_uint32),
                ("max_width", C.c_uint32), ("min_width", C.c_uint32),
                ("k_hist", C.c_uint32 * (GS_MAX_K_POLY + 1)), ("n_edges", C.c_uint64),
                ("nnz_coeffs", C.c_uint64), ("hidden_neurons", C.c_uint64), ("n_rows", C.c_uint64),
                ("program_hash", C.c_uint64)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["k_hist"] = list(self.k_hist)
        return d


class gs_sim_opts(C.Structure):
    _fields_ = [("device", C.c_int), ("stream", C.c_void_p), ("lanes", C.c_uint64),
                ("lane_offset", C.c_uint64), ("kernel", C.c_int), ("n_trace_words", C.c_uint32),
                ("trace_words", C.c_void_p), ("trace_cycles", C.c_uint32), ("use_graphs", C.c_int),
                ("lut_unroll", C.c_uint32), ("flags", C.c_uint32), ("tile_words", C.c_uint32),
                ("tile_groups", C.c_uint32), ("lane_groups", C.c_uint32), ("cluster_size", C.c_uint32),
                ("slab_lanes", C.c_uint32), ("slab_min_gates", C.c_uint32)]


class gs_signature(C.Structure):
    _fields_ = [("lane_sig_sum", C.c_uint64), ("out_popcount", C.c_uint64),
                ("ab_mismatch", C.c_uint64), ("invariant_violations", C.c_uint64),
                ("cycles", C.c_uint64)]

    def as_dict(self):
        return {f: int(getattr(self, f)) for f, _ in self._fields_}


class gs_launch_info(C.Structure):
    _fields_ = [("kernel", C.c_int), ("lane_groups", C.c_uint32), ("tile_words", C.c_uint32),
                ("tile_groups", C.c_uint32), ("tile_desc", C.c_uint32), ("grid", C.c_uint32),
                ("cluster_size", C.c_uint32), ("slab_lanes", C.c_uint32), ("live_slots", C.c_uint32)]


class gs_profile(C.Structure):
    _fields_ = [("level_ms", C.c_double), ("total_ms", C.c_double), ("level_launches", C.c_uint64),
                ("total_launches", C.c_uint64), ("level_bytes", C.c_double),
                ("grid_stride_launches", C.c_uint64), ("multi_gate_launches", C.c_uint64)]


# ------------------------------------------------------------------ loading
_P = C.c_void_p
_SIGS = {
    "gs_last_error": (C.c_char_p, []),
    "gs_version": (C.c_char_p, []),
    "gs_build_id": (C.c_char_p, []),
    "gs_netlist_create": (C.c_int32, [_P]),
    "gs_netlist_destroy": (C.c_int32, [_P]),
    "gs_add_input": (C.c_int32, [_P, _P]),
    "gs_add_const": (C.c_int32, [_P, C.c_int, _P]),
    "gs_add_gate": (C.c_int32, [_P, C.c_uint32, _P, C.c_uint64, _P]),
    "gs_add_gate_wide": (C.c_int32, [_P, C.c_uint32, _P, _P, _P]),
    "gs_add_register": (C.c_int32, [_P, C.c_int, _P]),
    "gs_set_register_d": (C.c_int32, [_P, C.c_uint32, C.c_uint32]),
    "gs_mark_output": (C.c_int32, [_P, C.c_uint32, _P]),
    "gs_netlist_load_arrays": (C.c_int32, [_P, _P]),
    "gs_netlist_get_counts": (C.c_int32, [_P, _P]),
    "gs_compile": (C.c_int32, [_P, _P, _P]),
    "gs_program_destroy": (C.c_int32, [_P]),
    "gs_program_get_info": (C.c_int32, [_P, _P]),
    "gs_program_level_widths": (C.c_int32, [_P, _P, C.c_uint32]),
    "gs_program_gate_levels": (C.c_int32, [_P, _P, C.c_uint32]),
    "gs_program_coeffs": (C.c_int32, [_P, C.c_uint32, _P, C.c_uint32]),
    "gs_program_tile_slots": (C.c_int32, [_P, _P]),
    "gs_program_save": (C.c_int32, [_P, C.c_char_p]),
    "gs_program_load": (C.c_int32, [C.c_char_p, _P]),
    "gs_program_gate_lut": (C.c_int32, [_P, C.c_uint32, _P, _P, _P]),
    "gs_sim_workspace_bytes": (C.c_int32, [_P, _P, _P]),
    "gs_sim_create": (C.c_int32, [_P, _P, _P, C.c_size_t, _P]),
    "gs_sim_destroy": (C.c_int32, [_P]),
    "gs_sim_bind_stimulus_generated": (C.c_int32, [_P, C.c_uint64]),
    "gs_sim_bind_stimulus_host": (C.c_int32, [_P, _P, C.c_uint32]),
    "gs_sim_bind_stimulus_device": (C.c_int32, [_P, _P, C.c_uint32]),
    "gs_sim_reset": (C.c_int32, [_P]),
    "gs_sim_set_lane_offset": (C.c_int32, [_P, C.c_uint64]),
    "gs_sim_step": (C.c_int32, [_P, C.c_uint32]),
    "gs_sim_sync": (C.c_int32, [_P]),
    "gs_sim_run_streamed": (C.c_int32, [_P, _P, _P, C.c_uint32, C.c_uint32]),
    "gs_sim_get_cycle": (C.c_int32, [_P, _P]),
    "gs_sim_get_config": (C.c_int32, [_P, _P, _P]),
    "gs_sim_get_launch": (C.c_int32, [_P, _P]),
    "gs_sim_read_outputs": (C.c_int32, [_P, _P, C.c_size_t]),
    "gs_sim_read_registers": (C.c_int32, [_P, _P, C.c_size_t]),
    "gs_sim_write_registers": (C.c_int32, [_P, _P, C.c_size_t]),
    "gs_sim_read_trace": (C.c_int32, [_P, _P, C.c_size_t, _P]),
    "gs_sim_read_lane_signatures": (C.c_int32, [_P, _P, C.c_size_t]),
    "gs_sim_read_signature": (C.c_int32, [_P, _P]),
    "gs_sim_profile_step": (C.c_int32, [_P, C.c_uint32, _P]),
    "gs_sim_launches_per_cycle": (C.c_int32, [_P, _P]),
}
EXPORTED = tuple(_SIGS)
_lib = None


def lib():
    """The loaded libgsim.so (raises if it has not been built — there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with "
                              "`python -m paper_conf_ipps_gavierrprs23_b200._build`")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _call(name, *args):
    rc = getattr(lib(), name)(*args)
    if rc != GS_OK:
        raise GsError(rc, name, lib().gs_last_error().decode())
    return rc


def __getattr__(name):            # gs_* names resolve to the raw C functions
    if name in _SIGS:
        return getattr(lib(), name)
    raise AttributeError(name)


def _p(a):
    return a.ctypes.data_as(C.c_void_p) if a is not None else None


# ------------------------------------------------------------------ handles
class Netlist:
    """gs_netlist handle.  ``Netlist.from_arrays(nl)`` bulk-loads a workloads.Netlist."""

    def __init__(self):
        h = C.c_void_p()
        _call("gs_netlist_create", C.byref(h))
        self.h = h

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.gs_netlist_destroy(self.h)
            self.h = None

    @classmethod
    def from_arrays(cls, nl) -> "Netlist":
        self = cls()
        keep = [np.ascontiguousarray(nl.reg_init, dtype=np.uint8),
                np.ascontiguousarray(nl.reg_d, dtype=np.uint32),
                np.ascontiguousarray(nl.gate_k, dtype=np.uint8),
                np.ascontiguousarray(nl.gate_in_off, dtype=np.uint32),
                np.ascontiguousarray(nl.gate_in, dtype=np.uint32),
                np.ascontiguousarray(nl.gate_tt, dtype=np.uint64),
                np.ascontiguousarray(nl.po, dtype=np.uint32)]
        hi = getattr(nl, "gate_tt_hi", None)
        keep.append(None if hi is None else np.ascontiguousarray(hi, dtype=np.uint64))
        a = gs_netlist_arrays(nl.n_pi, nl.n_reg, nl.n_gates, nl.n_po, *[_p(x) for x in keep])
        _call("gs_netlist_load_arrays", self.h, C.byref(a))
        return self

    def add_input(self) -> int:
        n = C.c_uint32()
        _call("gs_add_input", self.h, C.byref(n))
        return n.value

    def add_const(self, v: int) -> int:
        n = C.c_uint32()
        _call("gs_add_const", self.h, int(v), C.byref(n))
        return n.value

    def add_gate(self, ins, tt: int) -> int:
        """k-input LUT; tt is the LSB-first table as a Python int (up to 2^8 bits)."""
        arr = np.ascontiguousarray(list(ins), dtype=np.uint32)
        n = C.c_uint32()
        if len(arr) <= GS_MAX_K:
            _call("gs_add_gate", self.h, len(arr), _p(arr) if len(arr) else None, int(tt), C.byref(n))
        else:
            words = np.array([(int(tt) >> (64 * i)) & (2**64 - 1) for i in range(4)], dtype=np.uint64)
            _call("gs_add_gate_wide", self.h, len(arr), _p(arr), _p(words), C.byref(n))
        return n.value

    def add_register(self, init: int = 0) -> int:
        n = C.c_uint32()
        _call("gs_add_register", self.h, int(init), C.byref(n))
        return n.value

    def set_register_d(self, q: int, d: int) -> None:
        _call("gs_set_register_d", self.h, q, d)

    def mark_output(self, net: int) -> int:
        i = C.c_uint32()
        _call("gs_mark_output", self.h, net, C.byref(i))
        return i.value

    def counts(self) -> dict:
        c = gs_netlist_counts()
        _call("gs_netlist_get_counts", self.h, C.byref(c))
        return {f: int(getattr(c, f)) for f, _ in c._fields_}

    def compile(self, balance=True, max_k: int = 0, lut_k: int = 0, level_seed: int = 0) -> "Program":
        return Program(self, balance, max_k, lut_k, level_seed=level_seed)


class Program:
    def __init__(self, netlist: Netlist | None, balance=True, max_k: int = 0, lut_k: int = 0,
                 _handle=None, level_seed: int = 0):
        if _handle is None:
            h = C.c_void_p()
            # balance: True/1 slack-balanced, False/0 ASAP, 2 or "alap" ALAP levels
            b = 2 if balance in (2, "alap") else (1 if balance else 0)
            o = gs_compile_opts(b, max_k, lut_k, int(level_seed))
            _call("gs_compile", netlist.h, C.byref(o), C.byref(h))
        else:
            h = _handle
        self.h = h
        inf = gs_program_info()
        _call("gs_program_get_info", self.h, C.byref(inf))
        self.info = inf.as_dict()

    def save(self, path: str) -> None:
        _call("gs_program_save", self.h, os.fsencode(path))

    @classmethod
    def load(cls, path: str) -> "Program":
        h = C.c_void_p()
        _call("gs_program_load", os.fsencode(path), C.byref(h))
        return cls(None, _handle=h)

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.gs_program_destroy(self.h)
            self.h = None

    def level_widths(self) -> np.ndarray:
        w = np.zeros(max(self.info["n_levels"], 1), dtype=np.uint32)
        _call("gs_program_level_widths", self.h, _p(w), len(w))
        return w[:self.info["n_levels"]]

    def gate_levels(self) -> np.ndarray:
        lv = np.zeros(max(self.info["n_gates"], 1), dtype=np.uint32)
        _call("gs_program_gate_levels", self.h, _p(lv), len(lv))
        return lv[:self.info["n_gates"]]

    def gate_lut(self, gate: int) -> tuple[list[int], int]:
        """(input nets, truth table as a Python int) of the LUT evaluated for netlist gate `gate`."""
        k = C.c_uint32()
        ins = np.zeros(GS_MAX_K_POLY, dtype=np.uint32)
        tt = np.zeros(4, dtype=np.uint64)
        _call("gs_program_gate_lut", self.h, int(gate), C.byref(k), _p(ins), _p(tt))
        return ins[:k.value].tolist(), sum(int(w) << (64 * i) for i, w in enumerate(tt))

    def tile_slots(self) -> int:
        v = C.c_uint32()
        _call("gs_program_tile_slots", self.h, C.byref(v))
        return v.value

    def coeffs(self, gate: int, k: int) -> list[int]:
        w = np.zeros(1 << k, dtype=np.int32)
        _call("gs_program_coeffs", self.h, gate, _p(w), len(w))
        return w.tolist()


class Sim:
    """gs_sim in a torch-owned device workspace, queued on a torch CUDA stream."""

    def __init__(self, program: Program, lanes: int, lane_offset: int = 0, kernel="lut",
                 device: int = 0, stream=None, trace_words=(), trace_cycles: int = 0,
                 use_graphs: bool = True, lut_unroll: int = 0, pdl: bool = True,
                 tile_words: int = 0, tile_groups: int = 0, flags: int = 0, lane_groups: int = 0,
                 cluster_size: int = 0, slab_lanes: int = 0, slab_min_gates: int = 0):
        import torch
        self.program = program
        self.lanes, self.words = int(lanes), int(lanes) // 64
        self.device = torch.device("cuda", device)
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        self._tw = np.ascontiguousarray(list(trace_words), dtype=np.uint32)
        o = gs_sim_opts(device, C.c_void_p(self.stream.cuda_stream), self.lanes, int(lane_offset),
                        KERNELS[kernel] if isinstance(kernel, str) else int(kernel), len(self._tw),
                        _p(self._tw) if len(self._tw) else None, int(trace_cycles),
                        1 if use_graphs else 0, int(lut_unroll),
                        (0 if pdl else GS_SIM_NO_PDL) | int(flags), int(tile_words), int(tile_groups),
                        int(lane_groups), int(cluster_size), int(slab_lanes), int(slab_min_gates))
        nbytes = C.c_size_t()
        _call("gs_sim_workspace_bytes", program.h, C.byref(o), C.byref(nbytes))
        self.workspace = torch.empty(int(nbytes.value) + 256, dtype=torch.uint8, device=self.device)
        base = self.workspace.data_ptr()
        aligned = (base + 255) & ~255
        h = C.c_void_p()
        _call("gs_sim_create", program.h, C.byref(o), C.c_void_p(aligned), int(nbytes.value),
              C.byref(h))
        self.h = h
        self.n_po, self.n_reg = program.info["n_po"], program.info["n_reg"]
        self.n_trace_words = len(self._tw)
        self.trace_cycles = int(trace_cycles)
        self._stim_keep = None

    def close(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.gs_sim_destroy(self.h)
            self.h = None

    def __del__(self):
        self.close()

    # each method = one C call (plus numpy buffer allocation)
    def bind_generated(self, seed: int):
        _call("gs_sim_bind_stimulus_generated", self.h, int(seed))

    def bind_host(self, words: np.ndarray):
        w = np.ascontiguousarray(words, dtype=np.uint64)
        assert w.ndim == 3 and w.shape[2] == self.words
        self._stim_keep = w
        _call("gs_sim_bind_stimulus_host", self.h, _p(w), int(w.shape[0]))

    def bind_device(self, tensor, cycles: int):
        self._stim_keep = tensor
        _call("gs_sim_bind_stimulus_device", self.h, C.c_void_p(tensor.data_ptr()), int(cycles))

    def reset(self):
        _call("gs_sim_reset", self.h)

    def set_lane_offset(self, lane_offset: int):
        """Move to another lane range of the same job (sub-batching), then reset."""
        _call("gs_sim_set_lane_offset", self.h, int(lane_offset))

    def step(self, n: int = 1):
        _call("gs_sim_step", self.h, int(n))

    def sync(self):
        _call("gs_sim_sync", self.h)

    def run_streamed(self, stim: np.ndarray, out: np.ndarray | None = None, chunk: int = 0):
        """Stream stim [cycles][n_pi][W] in and every output [cycles][n_po][W] out (async;
        pinned arrays for overlap; call sync() before reading `out`)."""
        assert stim.dtype == np.uint64 and stim.flags.c_contiguous and stim.shape[2] == self.words
        if out is not None:
            assert out.dtype == np.uint64 and out.flags.c_contiguous and out.shape == (stim.shape[0], self.n_po, self.words)
        self._stim_keep = (stim, out)
        _call("gs_sim_run_streamed", self.h, _p(stim), _p(out), int(stim.shape[0]), int(chunk))

    @property
    def config(self) -> dict:
        """Resolved launch configuration: {'kernel': GS_KERNEL_*, 'lane_groups': G}."""
        k, g = C.c_int32(), C.c_uint32()
        _call("gs_sim_get_config", self.h, C.byref(k), C.byref(g))
        return {"kernel": k.value, "lane_groups": g.value}

    @property
    def launch(self) -> dict:
        """Resolved launch plan (gs_sim_get_launch)."""
        li = gs_launch_info()
        _call("gs_sim_get_launch", self.h, C.byref(li))
        return {f: int(getattr(li, f)) for f, _ in li._fields_}

    @property
    def cycle(self) -> int:
        c = C.c_uint64()
        _call("gs_sim_get_cycle", self.h, C.byref(c))
        return c.value

    def read_outputs(self, out: np.ndarray | None = None) -> np.ndarray:
        out = np.empty((self.n_po, self.words), dtype=np.uint64) if out is None else out
        _call("gs_sim_read_outputs", self.h, _p(out), out.size)
        return out

    def read_registers(self) -> np.ndarray:
        out = np.empty((self.n_reg, self.words), dtype=np.uint64)
        _call("gs_sim_read_registers", self.h, _p(out), out.size)
        return out

    def write_registers(self, regs: np.ndarray):
        r = np.ascontiguousarray(regs, dtype=np.uint64)
        _call("gs_sim_write_registers", self.h, _p(r), r.size)

    def read_trace(self) -> np.ndarray:
        rec = min(self.cycle, self.trace_cycles)
        out = np.empty((rec, self.n_po, self.n_trace_words), dtype=np.uint64)
        n = C.c_uint32()
        _call("gs_sim_read_trace", self.h, _p(out), out.size, C.byref(n))
        return out[:n.value]

    def read_lane_signatures(self) -> np.ndarray:
        out = np.empty(self.lanes, dtype=np.uint64)
        _call("gs_sim_read_lane_signatures", self.h, _p(out), out.size)
        return out

    def signature(self) -> dict:
        s = gs_signature()
        _call("gs_sim_read_signature", self.h, C.byref(s))
        return s.as_dict()

    def profile_step(self, n: int) -> dict:
        p = gs_profile()
        _call("gs_sim_profile_step", self.h, int(n), C.byref(p))
        return {f: getattr(p, f) for f, _ in p._fields_}

    def launches_per_cycle(self) -> int:
        v = C.c_uint64()
        _call("gs_sim_launches_per_cycle", self.h, C.byref(v))
        return v.value


def version() -> str:
    return lib().gs_version().decode()


def build_id() -> str:
    """Hash of the sources and flags libgsim.so was built from (gs_build_id)."""
    return lib().gs_build_id().decode()


def unpack_lanes(words: np.ndarray) -> np.ndarray:
    """[..., W] uint64 words -> [..., W*64] bits (lane s = bit s%64 of word s//64)."""
    w = np.ascontiguousarray(words, dtype=np.uint64)
    b = np.unpackbits(w.view(np.uint8).reshape(*w.shape, 8), axis=-1, bitorder="little")
    return b.reshape(*w.shape[:-1], w.shape[-1] * 64)
