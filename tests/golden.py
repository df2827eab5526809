"""Loader of tests/golden/*.txt: the paper's printed values for its worked
examples (`key = value  # citation`).  Test infrastructure only."""
import os

_DIR = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def paper_values(name: str = "paper_worked_examples.txt") -> dict:
    out = {}
    with open(os.path.join(_DIR, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            k, v = (x.strip() for x in line.split("=", 1))
            out[k] = int(v) if v.lstrip("-").isdigit() else float(v)
    return out


PAPER = paper_values()
