"""Plaintext semantics of a gate netlist -- the f of "Decrypt(Evaluate_f(c...)) = f(m...)" (Sec. II-A).
TEST INFRASTRUCTURE ONLY (oracle/).  Gate codes: truth table f(a,b) at bit (2a+b) (reading C15); NOT = !a;
MUX(s, x, y) = s ? x : y (the 3-input extension).
"""
from __future__ import annotations

import numpy as np

from .algorithm1 import algorithm1

NOT, MUX = 3, 16


def gate_bits(t: int, a, b=None, c=None):
    a = np.asarray(a, np.uint8)
    if t == NOT:
        return (1 - a).astype(np.uint8)
    if t == MUX:
        return np.where(a == 1, np.asarray(b, np.uint8), np.asarray(c, np.uint8)).astype(np.uint8)
    b = np.asarray(b, np.uint8)
    return ((t >> (2 * a.astype(np.int64) + b)) & 1).astype(np.uint8)


def simulate(n_inputs, types, in0, in1, in2, input_bits: np.ndarray) -> np.ndarray:
    """Evaluate every wire for a batch of input assignments.  input_bits: [n_inputs] or [batch, n_inputs].
    Returns wires [batch, n_inputs + n_gates].  Gates are visited level by level (Algorithm 1), so any gate
    order is accepted."""
    x = np.atleast_2d(np.asarray(input_bits, np.uint8))
    ng = len(types)
    w = np.zeros((x.shape[0], n_inputs + ng), np.uint8)
    w[:, :n_inputs] = x
    for level in algorithm1(n_inputs, types, in0, in1, in2):
        for g in level:
            t = int(types[g])
            b = w[:, in1[g]] if t != NOT else None
            c = w[:, in2[g]] if t == MUX else None
            w[:, n_inputs + g] = gate_bits(t, w[:, in0[g]], b, c)
    return w
