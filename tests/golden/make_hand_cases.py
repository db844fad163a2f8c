"""Writes tests/golden/hand_cases.json.

Every expected value is the closed form of Eq.1-2 (SS I)
for a hand-picked input, evaluated with math.exp in FP64.  The paper prints no
worked numeric example.  This script calls neither oracle/ nor the CUDA path.
"""
import json
import math
import os

e = math.exp
cases = {
    "_citation": ("Hand cases for Eq.1 (PAPER.md P:L24-28, SS I) and Eq.2 (P:L30-38). The paper prints "
                  "no worked numeric example, so every expected value is the closed form of Eq.1-2 for "
                  "the given inputs (expected_expr), evaluated in FP64 by tests/golden/make_hand_cases.py. "
                  "Reading Q1 (DESIGN.md SS3): the exponent is -||a-b||^2/(2h^2)."),
    "cases": [
        {"name": "pythagorean", "why": "d^2 = 3^2+4^2 = 25, d^2/(2h^2) = 25/50 = 1/2",
         "K": 2, "h": 5.0, "alpha": [[0.0, 0.0]], "W": [[1.0]], "beta": [[3.0, 4.0]],
         "expected": [[e(-0.5)]], "expected_expr": "exp(-1/2)"},
        {"name": "unit_1d", "why": "K=1, |0-1|^2/(2*1) = 1/2",
         "K": 1, "h": 1.0, "alpha": [[0.0]], "W": [[1.0]], "beta": [[1.0]],
         "expected": [[e(-0.5)]], "expected_expr": "exp(-1/2)"},
        {"name": "unit_axes_sum", "why": "sources e1,e2,e3, target 0, h=1: each d^2=1 -> (1+2+3) e^{-1/2}",
         "K": 3, "h": 1.0, "alpha": [[1, 0, 0], [0, 1, 0], [0, 0, 1]], "W": [[1.0], [2.0], [3.0]],
         "beta": [[0, 0, 0]], "expected": [[6 * e(-0.5)]], "expected_expr": "6 exp(-1/2)"},
        {"name": "cancellation", "why": "sources at +-1, target 0, W=(1,-1): equal kernels cancel exactly",
         "K": 1, "h": 1.0, "alpha": [[1.0], [-1.0]], "W": [[1.0], [-1.0]], "beta": [[0.0]],
         "expected": [[0.0]], "expected_expr": "0", "exact": True},
        {"name": "two_targets_two_cols",
         "why": "K=2, h=1; target (0,0): d^2 = 0 and 2; target (1,1): d^2 = 2 and 0; R=2 columns",
         "K": 2, "h": 1.0, "alpha": [[0, 0], [1, 1]], "W": [[1.0, 0.5], [2.0, -1.0]],
         "beta": [[0, 0], [1, 1]],
         "expected": [[1.0 + 2.0 * e(-1.0), 0.5 - e(-1.0)], [e(-1.0) + 2.0, 0.5 * e(-1.0) - 1.0]],
         "expected_expr": "[[1+2e^-1, 1/2-e^-1], [e^-1+2, e^-1/2-1]]"},
        {"name": "bandwidth_is_2h2",
         "why": "Q1: d^2=1, h=0.5 -> exponent 1/(2*0.25) = 2 (not 1/h^2 = 4, not 1/(2h)^2 = 1)",
         "K": 1, "h": 0.5, "alpha": [[0.0]], "W": [[1.0]], "beta": [[1.0]],
         "expected": [[e(-2.0)]], "expected_expr": "exp(-2)"},
    ],
}

if __name__ == "__main__":
    out = os.path.join(os.path.dirname(os.path.abspath(__file__)), "hand_cases.json")
    with open(out, "w") as f:
        json.dump(cases, f, indent=1)
        f.write("\n")
