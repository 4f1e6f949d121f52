"""Synthesised-netlist import: Yosys JSON and BLIF gate-level netlists -> Netlist -> Fig. 5 binary.

The fixtures in tests/golden/ are hand-written full adders in the shapes those tools write (they are not from the
paper, which prints no netlist); what pins the importers is the plaintext semantics of every output on all 8 input
assignments, checked against the arithmetic definition, plus the Fig. 5 assembler round trip.
"""
import itertools
import os

import numpy as np
import pytest

from oracle.plain import simulate
from paper_conf_ispass_maxw23_b200 import netlist as NL

GOLD = os.path.join(os.path.dirname(__file__), "golden")
ALL = np.array(list(itertools.product((0, 1), repeat=3)), np.uint8)      # a, b, cin


def run(net, bits):
    w = simulate(net.n_inputs, net.type, net.in0, net.in1, net.in2, bits)
    return w[:, net.outputs]


def test_yosys_json_full_adder():
    net = NL.read_yosys_json(open(os.path.join(GOLD, "full_adder_yosys.json")).read())
    assert net.n_inputs == 3 and net.outputs.size == 3
    out = run(net, ALL)
    a, b, c = ALL.T.astype(int)
    assert (out[:, 0] == (a ^ b ^ c)).all()
    assert (out[:, 1] == ((a & b) | (c & (a ^ b)))).all()
    assert (out[:, 2] == ((a & (1 - b)) | (b & c))).all()
    # the constant input of k0 is folded away, the dead NOR is never emitted, $_MUX_ becomes a MUX gate
    assert (net.type == NL.MUX).sum() == 1 and net.n_gates == 7


def test_blif_full_adder():
    net = NL.read_blif(open(os.path.join(GOLD, "full_adder.blif")).read())
    out = run(net, ALL)
    a, b, c = ALL.T.astype(int)
    assert (out[:, 0] == (a ^ b ^ c)).all()
    assert (out[:, 1] == ((a & b) | (c & (a ^ b)))).all()
    assert (out[:, 2] == (a & (1 - b))).all()
    assert set(net.type.tolist()) <= {NL.XOR, NL.OR, NL.AND, NL.MUX, NL.ANDYN}


def test_every_two_input_cover_maps_to_its_truth_table():
    """all 16 two-input functions as BLIF covers: gates, folded constants, identities and inverters"""
    for code in range(16):
        rows = ["%d%d 1" % (a, b) for a in (0, 1) for b in (0, 1) if (code >> (2 * a + b)) & 1]
        text = ".model f\n.inputs a b\n.outputs y z\n.names a b y\n%s\n.names a b z\n01 1\n10 1\n.end\n" % "\n".join(rows)
        if code in (0, 15):
            with pytest.raises(ValueError, match="constant"):
                NL.read_blif(text)
            continue
        net = NL.read_blif(text)
        ab = np.array(list(itertools.product((0, 1), repeat=2)), np.uint8)
        got = run(net, ab)[:, 0]
        want = np.array([(code >> (2 * a + b)) & 1 for a, b in ab], np.uint8)
        assert (got == want).all(), code


def test_import_then_assemble_round_trip():
    """BLIF without MUX -> Fig. 5 binary -> reader: same plaintext function"""
    text = open(os.path.join(GOLD, "full_adder.blif")).read()
    text = text.replace(".names cin o n cout\n11- 1\n0-1 1\n", ".names o n cout\n00 0\n")     # cout = o | n
    net = NL.read_blif(text)
    back = NL.read_pytfhe_binary(NL.write_pytfhe_binary(net))
    assert (run(back, ALL) == run(net, ALL)).all()


def test_import_errors():
    with pytest.raises(ValueError, match="no driver"):
        NL.read_blif(".model f\n.inputs a\n.outputs y\n.end\n")
    with pytest.raises(ValueError, match="loop"):
        NL.read_blif(".model f\n.inputs a\n.outputs y\n.names a z y\n11 1\n.names y z\n1 1\n.end\n")
    with pytest.raises(ValueError, match="unsupported type"):
        NL.read_yosys_json({"modules": {"m": {"ports": {"a": {"direction": "input", "bits": [2]},
                                                        "y": {"direction": "output", "bits": [3]}},
                                              "cells": {"c": {"type": "$_DFF_P_", "connections": {}}}}}})
