"""Gate netlists: the in-memory program DAG, Algorithm-1 levelisation (native) and the PyTFHE binary format.

P:N = /root/reference/PAPER.md line N.
  - A TFHE program is "a DAG of gates" traversed by Algorithm 1.
  - The PyTFHE binary (Fig. 5): 128-bit instructions -- header (field [65:4] = total
    number of gates), input (all fields all ones), gate (in0 index [127:66], in1 index [65:4], 4-bit type
    [3:0]), output (in0 field all ones, producing gate index in [65:4], type field 0x3).  Indices are the
    instruction positions (header = 0), so inputs are 1..n_in and gates follow (Fig. 6 half adder: A=1, B=2,
    XOR=3, AND=4).  Reading C15: little-endian, low 64 bits first; kinds decoded by field pattern.
Wire ids used in this package: [0, n_inputs) = inputs, n_inputs + g = output of gate g.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass, field

import numpy as np

from . import _native

NOR, ANDNY, NOT, ANDYN, XOR, NAND, AND, XNOR, ORNY, ORYN, OR, MUX = 1, 2, 3, 4, 6, 7, 8, 9, 11, 13, 14, 16
GATE_CODES = {"NOR": NOR, "ANDNY": ANDNY, "NOT": NOT, "ANDYN": ANDYN, "XOR": XOR, "NAND": NAND, "AND": AND,
              "XNOR": XNOR, "ORNY": ORNY, "ORYN": ORYN, "OR": OR, "MUX": MUX}
BINARY_GATES = (NOR, ANDNY, NOT, ANDYN, XOR, NAND, AND, XNOR, ORNY, ORYN, OR)   # the 11 gates of P:176

_ONES62 = (1 << 62) - 1


@dataclass
class Netlist:
    n_inputs: int
    type: np.ndarray                     # int32 [n_gates]
    in0: np.ndarray                      # int64 [n_gates]
    in1: np.ndarray                      # int64 [n_gates] (-1 for NOT)
    in2: np.ndarray = None               # int64 [n_gates] (-1 unless MUX)
    outputs: np.ndarray = field(default_factory=lambda: np.zeros(0, np.int64))   # wire ids

    def __post_init__(self):
        self.type = np.ascontiguousarray(self.type, np.int32)
        self.in0 = np.ascontiguousarray(self.in0, np.int64)
        self.in1 = np.ascontiguousarray(self.in1, np.int64)
        self.in2 = (np.full(self.type.size, -1, np.int64) if self.in2 is None
                    else np.ascontiguousarray(self.in2, np.int64))
        self.outputs = np.ascontiguousarray(self.outputs, np.int64)

    @property
    def n_gates(self) -> int:
        return int(self.type.size)

    @property
    def n_wires(self) -> int:
        return self.n_inputs + self.n_gates

    def c_struct(self) -> _native.Netlist:
        return _native.Netlist(self.n_inputs, self.n_gates, self.type.ctypes.data, self.in0.ctypes.data,
                               self.in1.ctypes.data, self.in2.ctypes.data)

    def levels(self):
        """Algorithm 1, native: (level_of_gate int64 [n_gates], n_levels)."""
        lv = np.zeros(self.n_gates, np.int64)
        nl = ctypes.c_int64(0)
        s = self.c_struct()
        _native.check(_native.lib().tb_levelise(ctypes.byref(s), lv.ctypes.data, ctypes.byref(nl)))
        return lv, int(nl.value)

    def plan(self):
        """Host-only execution plan (tb_netlist_plan): (levels [(row0, n_gates)], row_of_wire int64).  Level L's
        outputs are rows row0 .. row0 + n_gates - 1 of the wire array (contiguous, as the all-gather needs)."""
        s = self.c_struct()
        nl = ctypes.c_int64(0)
        _native.check(_native.lib().tb_netlist_plan(ctypes.byref(s), ctypes.byref(nl), None, None))
        off = np.zeros(int(nl.value) + 1, np.int64)
        rows = np.zeros(self.n_wires, np.int64)
        _native.check(_native.lib().tb_netlist_plan(ctypes.byref(s), ctypes.byref(nl), off.ctypes.data,
                                                    rows.ctypes.data))
        levels = [(self.n_inputs + int(off[L]), int(off[L + 1] - off[L])) for L in range(int(nl.value))]
        return levels, rows


# ------------------------------------------------------------------------------------- binary format
def _inst(hi62: int, mid62: int, t4: int) -> bytes:
    v = ((hi62 & _ONES62) << 66) | ((mid62 & _ONES62) << 4) | (t4 & 0xF)
    return v.to_bytes(16, "little")


def write_pytfhe_binary(net: Netlist) -> bytes:
    """Fig. 5 writer.  MUX has no 4-bit code in the paper's format (C10) and is rejected."""
    if (net.type == MUX).any():
        raise ValueError("MUX is an in-memory extension; the PyTFHE binary has only the 11 two-input/NOT gates")
    out = [_inst(0, net.n_gates, 0)]
    out += [_inst(_ONES62, _ONES62, 0xF)] * net.n_inputs
    idx = lambda w: int(w) + 1                                  # wire id -> instruction index
    for t, a, b in zip(net.type.tolist(), net.in0.tolist(), net.in1.tolist()):
        out.append(_inst(idx(a), idx(b) if b >= 0 else 0, t))
    for w in net.outputs.tolist():
        out.append(_inst(_ONES62, idx(w), 0x3))
    return b"".join(out)


def read_pytfhe_binary(data: bytes) -> Netlist:
    """Fig. 5 reader -> Netlist (wire id = instruction index - 1).  Gate instructions may reference later
    indices (no topological order assumed)."""
    if len(data) % 16:
        raise ValueError("PyTFHE binary length must be a multiple of 16 bytes")
    insts = [int.from_bytes(data[i:i + 16], "little") for i in range(0, len(data), 16)]
    if not insts:
        raise ValueError("empty binary")
    f = lambda v: (v >> 66, (v >> 4) & _ONES62, v & 0xF)
    h0, n_gates, ht = f(insts[0])
    if h0 != 0 or ht != 0:
        raise ValueError("first instruction is not a header")
    n_in, types, a, b, outs = 0, [], [], [], []
    for v in insts[1:]:
        x0, x1, t = f(v)
        if x0 == _ONES62:
            if x1 == _ONES62 and t == 0xF:
                if types:
                    raise ValueError("input instruction after a gate instruction")
                n_in += 1
            elif t == 0x3:
                outs.append(x1 - 1)
            else:
                raise ValueError("unknown instruction pattern")
        else:
            if t not in BINARY_GATES:
                raise ValueError("unknown gate type %d" % t)
            types.append(t)
            a.append(x0 - 1)
            b.append(-1 if t == NOT else x1 - 1)
    if len(types) != n_gates:
        raise ValueError("header says %d gates, found %d" % (n_gates, len(types)))
    return Netlist(n_in, np.array(types, np.int32), np.array(a, np.int64), np.array(b, np.int64),
                   outputs=np.array(outs, np.int64))
