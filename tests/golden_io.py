"""Loader for the small text fixtures under tests/golden/ (sections '[name ...]', rows of numbers)."""
import os
from fractions import Fraction

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_sections(fname):
    out, cur = {}, None
    with open(os.path.join(GOLDEN, fname)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            if line.startswith("["):
                cur = line[1:line.index("]")]
                out[cur] = []
            else:
                out[cur].append([Fraction(t) for t in line.split()])
    return out
