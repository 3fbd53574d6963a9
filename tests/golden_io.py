"""Reader for the text fixtures under tests/golden/ (values from cited textbooks).

Format: '#' comments; an "arcs:" section of "u v w" lines (vertex numbers as
printed in the fixture, `base` subtracted); optional "source: s"; a "dist:"
section (the full matrix, or the one row of the source).
"""
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(name, base=0):
    arcs, dist, source = [], [], None
    section = None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#")[0].strip()
            if not line:
                continue
            if line in ("arcs:", "dist:"):
                section = line
                continue
            if line.startswith("source:"):
                source = int(line.split(":")[1]) - base
                continue
            vals = [int(x) for x in line.split()]
            if section == "arcs:":
                u, v, w = vals
                arcs.append((u - base, v - base, w))
            else:
                dist.append(vals)
    return arcs, source, dist
