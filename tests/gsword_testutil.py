"""Helpers shared by the test modules (golden-file reader, tolerances)."""
import math
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")


def read_golden(name):
    """Non-comment, non-empty lines of tests/golden/<name>, split on whitespace."""
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            rows.append(line.replace("->", " ").split())
    return rows


def variance_tolerance(agg, rel=1e-12):
    """Absolute tolerance for comparing variances: the subtraction sumsq - sum^2/n can
    cancel, so the error bound scales with sumsq / (n (n-1))."""
    n = agg["n"]
    return rel * abs(agg["sumsq"]) / (n * (n - 1)) + 1e-300 if n >= 2 else math.inf
