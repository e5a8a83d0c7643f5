"""Reader for the tests/golden/*.txt fixtures (values printed in or forced by the paper)."""
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def read(name):
    out = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            key, val = line.split(":", 1)
            out[key.strip()] = val.strip()
    return out


def pairs(val):
    return [tuple(int(x) for x in tok.split("-")) for tok in val.split()]


def ints(val):
    return [int(x) for x in val.split()]


def tuples(val):
    return [tuple(int(x) for x in part.split()) for part in val.split("|")]
