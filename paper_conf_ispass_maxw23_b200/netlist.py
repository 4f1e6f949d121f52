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

    def plan(self, capacity: int = 0):
        """Host-only execution plan (tb_netlist_plan_capacity): (levels [(row0, n_gates)], row_of_wire int64).
        Level L's outputs are rows row0 .. row0 + n_gates - 1 of the wire array (contiguous, as the all-gather
        needs).  capacity > 0: the capacity-aware level schedule (f1) that tb_netlist_upload uses."""
        s = self.c_struct()
        nl = ctypes.c_int64(0)
        f = _native.lib().tb_netlist_plan_capacity
        _native.check(f(ctypes.byref(s), capacity, ctypes.byref(nl), None, None))
        off = np.zeros(int(nl.value) + 1, np.int64)
        rows = np.zeros(self.n_wires, np.int64)
        _native.check(f(ctypes.byref(s), capacity, ctypes.byref(nl), off.ctypes.data, rows.ctypes.data))
        levels = [(self.n_inputs + int(off[L]), int(off[L + 1] - off[L])) for L in range(int(nl.value))]
        return levels, rows

    def plan_world(self, world: int, capacity: int = 0):
        """Host-only plan for a level loop over `world` ranks (tb_netlist_plan_world): (levels, row_of_wire, early)
        with early[L - 1][r] = the gates at the start of rank r's chunk of level L that r can run before the
        exchange of level L - 1."""
        s = self.c_struct()
        nl = ctypes.c_int64(0)
        f = _native.lib().tb_netlist_plan_world
        _native.check(f(ctypes.byref(s), capacity, world, ctypes.byref(nl), None, None, None))
        L = int(nl.value)
        off = np.zeros(L + 1, np.int64)
        rows = np.zeros(self.n_wires, np.int64)
        early = np.zeros((L, world), np.int64)
        _native.check(f(ctypes.byref(s), capacity, world, ctypes.byref(nl), off.ctypes.data, rows.ctypes.data,
                        early.ctypes.data))
        levels = [(self.n_inputs + int(off[k]), int(off[k + 1] - off[k])) for k in range(L)]
        return levels, rows, early


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


# ------------------------------------------------------------------ synthesised-netlist import
# PyTFHE's flow is Verilog -> (augmented) Yosys -> gate netlist -> assembler -> Fig. 5 binary.
# These readers take the gate-level netlist a synthesis tool writes and build the in-memory Netlist, which
# write_pytfhe_binary() then assembles.  Two input forms:
#   * Yosys JSON (`write_json` after `abc -g AND,NAND,OR,NOR,XOR,XNOR,ANDNOT,ORNOT,MUX`): internal cell types
#     $_AND_ $_NAND_ $_OR_ $_NOR_ $_XOR_ $_XNOR_ $_ANDNOT_ (A & ~B) $_ORNOT_ (A | ~B) $_NOT_ $_BUF_ $_MUX_
#     (Y = S ? B : A);
#   * BLIF (`write_blif`): `.names` covers of <= 2 inputs (any 2-input function maps to one gate code, since the
#     code IS the truth table at bit 2a+b, reading C15) and 3-input multiplexer covers.
# Constant drivers are folded away (AND(x, 0) = 0, XOR(x, 1) = NOT x, ...); an output that folds to a constant
# cannot be carried by a ciphertext wire and is rejected.
_YOSYS_CELLS = {"$_AND_": AND, "$_NAND_": NAND, "$_OR_": OR, "$_NOR_": NOR, "$_XOR_": XOR, "$_XNOR_": XNOR,
                "$_ANDNOT_": ANDYN, "$_ORNOT_": ORYN}


class _Assembler:
    """Topological emission of (code, fanins) nodes keyed by net name, with constant folding.
    A resolved net is ('c', 0|1), ('w', wire id)."""

    def __init__(self, inputs):
        self.inputs = list(inputs)
        self.val = {n: ("w", i) for i, n in enumerate(self.inputs)}
        self.val[("c", 0)], self.val[("c", 1)] = ("c", 0), ("c", 1)
        self.t, self.a, self.b, self.c = [], [], [], []
        self.nodes = {}

    def add(self, out, code, fanins):
        if out in self.nodes or out in self.val:
            raise ValueError("net %r driven twice" % (out,))
        self.nodes[out] = (code, list(fanins))

    def _gate(self, code, a, b=-1, c=-1):
        self.t.append(code)
        self.a.append(a)
        self.b.append(b)
        self.c.append(c)
        return ("w", len(self.inputs) + len(self.t) - 1)

    def _fold2(self, code, x, y):
        """2-input truth-table code on resolved operands."""
        f = lambda a, b: (code >> (2 * a + b)) & 1
        if x[0] == "c" and y[0] == "c":
            return ("c", f(x[1], y[1]))
        if x[0] == "c" or y[0] == "c":        # one constant: the gate is const, identity or NOT of the other
            if x[0] == "c":
                r0, r1, w = f(x[1], 0), f(x[1], 1), y
            else:
                r0, r1, w = f(0, y[1]), f(1, y[1]), x
            if r0 == r1:
                return ("c", r0)
            return w if (r0, r1) == (0, 1) else self._gate(NOT, w[1])
        if x == y:                             # same wire twice: const, identity or NOT
            r0, r1 = f(0, 0), f(1, 1)
            if r0 == r1:
                return ("c", r0)
            return x if (r0, r1) == (0, 1) else self._gate(NOT, x[1])
        if code in (0, 15):
            return ("c", code & 1)
        if code == 12:                         # f = a
            return x
        if code == 10:                         # f = b
            return y
        if code == 3:                          # f = !a
            return self._gate(NOT, x[1])
        if code == 5:                          # f = !b
            return self._gate(NOT, y[1])
        return self._gate(code, x[1], y[1])

    def resolve(self, net):
        stack = [net]
        while stack:
            n = stack[-1]
            if n in self.val:
                stack.pop()
                continue
            if n not in self.nodes:
                raise ValueError("net %r has no driver" % (n,))
            code, fins = self.nodes[n]
            pend = [f for f in fins if f not in self.val]
            if pend:
                if any(p in stack for p in pend):
                    raise ValueError("combinational loop through %r" % (n,))
                stack.extend(pend)
                continue
            ops = [self.val[f] for f in fins]
            if code == "BUF":
                r = ops[0]
            elif code == NOT:
                r = ("c", 1 - ops[0][1]) if ops[0][0] == "c" else self._gate(NOT, ops[0][1])
            elif code == MUX:                  # s ? x : y
                s, x, y = ops
                if s[0] == "c":
                    r = x if s[1] else y
                elif x == y:
                    r = x
                elif x[0] == "c" or y[0] == "c":   # s ? 1 : y = OR(s, y); s ? 0 : y = ANDNY(s, y); ...
                    if x[0] == "c" and y[0] == "c":
                        r = s if (x[1], y[1]) == (1, 0) else self._gate(NOT, s[1])
                    elif x[0] == "c":
                        r = self._fold2(OR if x[1] else ANDNY, s, y)
                    else:
                        r = self._fold2(AND if y[1] == 0 else ORNY, s, x)
                else:
                    r = self._gate(MUX, s[1], x[1], y[1])
            else:
                r = self._fold2(code, ops[0], ops[1])
            self.val[n] = r
            stack.pop()
        return self.val[net]

    def netlist(self, outputs) -> Netlist:
        outs = []
        for o in outputs:
            r = self.resolve(o)
            if r[0] == "c":
                raise ValueError("output %r is the constant %d: no ciphertext wire carries it" % (o, r[1]))
            outs.append(r[1])
        return Netlist(len(self.inputs), np.array(self.t, np.int32), np.array(self.a, np.int64),
                       np.array(self.b, np.int64), np.array(self.c, np.int64), outputs=np.array(outs, np.int64))


def read_yosys_json(doc, module: str | None = None) -> Netlist:
    """Yosys `write_json` gate-level module -> Netlist.  Inputs are the module's input port bits in port
    order (then bit order), outputs its output port bits likewise.  `doc` is the parsed JSON or its text."""
    import json
    if isinstance(doc, (str, bytes)):
        doc = json.loads(doc)
    mods = doc["modules"]
    if module is None:
        if len(mods) != 1:
            raise ValueError("several modules: name one of %s" % sorted(mods))
        module = next(iter(mods))
    m = mods[module]
    def key(bit):
        if isinstance(bit, str):
            if bit not in ("0", "1"):
                raise ValueError("undefined constant bit %r" % bit)
            return ("c", int(bit))
        return bit
    ins, outs = [], []
    for name, p in m["ports"].items():
        (ins if p["direction"] == "input" else outs if p["direction"] == "output" else []).extend(p["bits"])
        if p["direction"] not in ("input", "output"):
            raise ValueError("inout port %r" % name)
    A = _Assembler(ins)
    for cname, cell in m["cells"].items():
        t, cn = cell["type"], cell["connections"]
        one = lambda pin: key(cn[pin][0])
        if t in _YOSYS_CELLS:
            A.add(one("Y"), _YOSYS_CELLS[t], [one("A"), one("B")])
        elif t == "$_NOT_":
            A.add(one("Y"), NOT, [one("A")])
        elif t == "$_BUF_":
            A.add(one("Y"), "BUF", [one("A")])
        elif t == "$_MUX_":
            A.add(one("Y"), MUX, [one("S"), one("B"), one("A")])
        else:
            raise ValueError("cell %r has unsupported type %r (map to simple gates first)" % (cname, t))
    # nets named in "netnames" may alias output bits to input bits directly: handled by resolve()
    return A.netlist([key(b) for b in outs])


def read_blif(text: str) -> Netlist:
    """BLIF (one combinational .model) -> Netlist.  `.names` with 0-2 inputs become one gate (the 4-bit code is
    the truth table of the cover); 3-input covers must be a multiplexer (s ? x : y in some input order)."""
    lines, cur = [], ""
    for raw in text.splitlines():
        raw = raw.split("#", 1)[0].rstrip()
        if raw.endswith("\\"):
            cur += raw[:-1] + " "
            continue
        cur += raw
        if cur.strip():
            lines.append(cur.split())
        cur = ""
    ins, outs, A, i = [], [], None, 0
    while i < len(lines):
        tok = lines[i]
        if tok[0] == ".model":
            i += 1
        elif tok[0] == ".inputs":
            ins += tok[1:]
            i += 1
        elif tok[0] == ".outputs":
            outs += tok[1:]
            i += 1
        elif tok[0] == ".names":
            if A is None:
                A = _Assembler(ins)
            nets, i = tok[1:], i + 1
            cover = []
            while i < len(lines) and not lines[i][0].startswith("."):
                cover.append(lines[i])
                i += 1
            _blif_names(A, nets[:-1], nets[-1], cover)
        elif tok[0] == ".end":
            break
        else:
            raise ValueError("unsupported BLIF construct %r" % tok[0])
    if A is None:
        A = _Assembler(ins)
    return A.netlist(outs)


def _blif_names(A: _Assembler, fins, out, cover):
    k = len(fins)
    onset = None
    table = np.zeros(1 << k, np.uint8)
    for row in cover:
        if k == 0:
            pat, val = "", row[0]
        else:
            pat, val = row
        bit = int(val)
        if onset is None:
            onset = bit
            table[:] = 1 - bit
        elif onset != bit:
            raise ValueError("mixed on-set / off-set cover for %r" % out)
        for m in range(1 << k):                    # minterm m: input j = bit (k-1-j) of m
            if all(c == "-" or int(c) == (m >> (k - 1 - j)) & 1 for j, c in enumerate(pat)):
                table[m] = bit
    if k == 0:
        const = int(table[0]) if cover else 0
        A.val[out] = ("c", const)
        return
    if k == 1:
        if (table == [0, 1]).all():
            A.add(out, "BUF", fins)
        elif (table == [1, 0]).all():
            A.add(out, NOT, fins)
        else:
            A.add(out, "BUF", [("c", int(table[0]))])
        return
    if k == 2:
        code = sum(int(table[(a << 1) | b]) << (2 * a + b) for a in (0, 1) for b in (0, 1))
        A.add(out, code, fins)
        return
    if k == 3:
        for s in range(3):                          # find the select input: f = s ? x : y
            x, y = [j for j in range(3) if j != s]
            for sw in (False, True):
                xi, yi = (y, x) if sw else (x, y)
                ok = all(table[m] == ((m >> (2 - xi)) & 1 if (m >> (2 - s)) & 1 else (m >> (2 - yi)) & 1)
                         for m in range(8))
                if ok:
                    A.add(out, MUX, [fins[s], fins[xi], fins[yi]])
                    return
    raise ValueError(".names %r: only <= 2-input functions and multiplexers are supported" % out)
