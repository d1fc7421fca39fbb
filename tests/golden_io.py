"""Reader for the hand-worked fixtures under tests/golden/ (see README)."""
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(name):
    mats, scalars = {}, {}
    cur = None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            tok = line.split()
            if tok[0] == "matrix":
                cur = (tok[1], int(tok[2]), int(tok[3]), [])
            elif tok[0] == "end":
                nm, nr, nc, pairs = cur
                p = np.array(pairs, dtype=np.uint32).reshape(-1, 2)
                mats[nm] = (nr, nc, p[:, 0].copy(), p[:, 1].copy())
                cur = None
            elif tok[0] == "scalar":
                scalars[tok[1]] = int(tok[2])
            else:
                cur[3].append((int(tok[0]), int(tok[1])))
    return mats, scalars
