"""Readers for the tests/golden fixtures (plain text, cited inside each file)."""
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def read_triples(name):
    """Sections 'A', 'B', 'C' of 'row col val' lines plus 'key v v v' scalars."""
    sections, scalars, cur = {}, {}, None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            parts = line.split()
            if parts[0] in ("A", "B", "C") and len(parts) == 1:
                cur = parts[0]
                sections[cur] = []
            elif len(parts) == 3 and cur is not None and parts[0].lstrip("-").isdigit():
                sections[cur].append((int(parts[0]), int(parts[1]), float(parts[2])))
            else:
                scalars[parts[0]] = [int(x) for x in parts[1:]]
    out = {k: tuple(np.array(col) for col in zip(*v)) for k, v in sections.items()}
    return out, scalars


def read_kv(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if line:
                rows.append(line.split())
    return rows
