"""Reader for the text fixtures under tests/golden/ (format in each file's header)."""
import os

import numpy as np

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    """Return (Graph with 0-based ids, expected bc f64[n])."""
    n, us, vs, bc = 0, [], [], {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            t = line.split("#", 1)[0].split()
            if not t:
                continue
            if t[0] == "n":
                n = int(t[1])
            elif t[0] == "e":
                us.append(int(t[1]) - 1)
                vs.append(int(t[2]) - 1)
            elif t[0] == "bc":
                bc[int(t[1]) - 1] = float(t[2])
    g = gg.csr_from_edges(n, np.array(us, dtype=np.int64), np.array(vs, dtype=np.int64),
                          directed=False, name=name)
    return g, np.array([bc[i] for i in range(n)], dtype=np.float64)
