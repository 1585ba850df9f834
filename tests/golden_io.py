"""Readers for tests/golden/*.txt fixtures (each file carries its PAPER.md citation)."""
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _lines(name):
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if line:
                yield line


def binarize_cases():
    for line in _lines("binarize.txt"):
        lhs, rhs = line.split("|")
        x = np.array([float(v) for v in lhs.split(",")], np.float32)
        words = np.array([int(v, 16) for v in rhs.split(",")], np.uint32)
        yield x, words


def dpr_cases():
    """Yields (bits, inputs float32[], expected word/code uint32, packed: bool)."""
    for line in _lines("dpr.txt"):
        bits, xs, code = line.split()
        x = np.array([float(v) for v in xs.split(",")], np.float32)
        yield int(bits), x, int(code, 16), "," in xs
