"""Parsers for the text fixtures under tests/golden/ (no method arithmetic here)."""
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
SYMBOLS = {"A": 0x3FC00000, "B": 0x40200000, "C": 0xC0400000, "0": 0}


def read_pairs(name):
    out = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":", 1)
            out[k.strip()] = v.strip()
    return out


def words(s):
    return np.array([SYMBOLS[t] if t in SYMBOLS else int(t, 0) for t in s.split()], dtype=np.uint32)


def ints(s):
    return [int(t, 0) for t in s.split()]


def lz4_cases():
    cases = {}
    for k, v in read_pairs("lz4_examples.txt").items():
        src, dst = v.split("->")
        cases[k] = (bytes.fromhex(src.replace(" ", "")), bytes.fromhex(dst.replace(" ", "")))
    return cases
