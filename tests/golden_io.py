"""Parser for the hand-worked fixtures in tests/golden/ (values are fractions, 'ln3', '-inf')."""
import math
import os
from fractions import Fraction

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def val(tok: str) -> float:
    if tok == "ln3":
        return math.log(3.0)
    if tok in ("-inf", "inf"):
        return float(tok)
    return float(Fraction(tok))


def load(name: str) -> dict:
    out = {}
    lines = [l.strip() for l in open(os.path.join(GOLDEN, name)) if l.strip() and not l.startswith("#")]
    i = 0
    while i < len(lines):
        parts = lines[i].split()
        key = parts[0]
        if key == "O":
            S = int(out["S"])
            out["O"] = [[val(t) for t in lines[i + 1 + r].split()] for r in range(S)]
            i += 1 + S
            continue
        vals = [val(t) for t in parts[1:]]
        out[key] = vals[0] if len(vals) == 1 else vals
        i += 1
    return out
