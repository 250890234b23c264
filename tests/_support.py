"""Small helpers shared by the tests (no method arithmetic)."""
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def read_golden(name):
    vals = {}
    with open(os.path.join(ROOT, "tests", "golden", name)) as fh:
        for line in fh:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            if "=" in line:
                k, v = line.split("=", 1)
                vals[k.strip()] = float(v)
            else:
                vals.setdefault("_rows", []).append(line.split())
    return vals
