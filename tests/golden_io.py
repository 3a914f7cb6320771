"""Parser for the tests/golden/*.txt worked-example fixtures."""
import os

import graphgen

HERE = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(name):
    meta, rows, expect = {}, {}, {}
    with open(os.path.join(HERE, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip() if not line.startswith("expect") else line.strip()
            if not line:
                continue
            tok = line.split()
            if tok[0] == "row":
                rows[int(tok[1])] = [int(x) for x in tok[2:]]
            elif tok[0] == "expect":
                expect[tok[1]] = tok[2:]
            else:
                meta[tok[0]] = tok[1]
    n = int(meta["n"])
    edges = [(u, v, 1) for u in range(n) for v in rows.get(u, [])]
    return graphgen.from_edge_list(n, edges, name), meta, expect
