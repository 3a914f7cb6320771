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


def load_sec3(name):
    """§3 fixtures (tests/golden/sec3_*.txt): ``arc u v w`` (one direction),
    ``edge u v w`` (both directions), scalar meta lines, and
    ``expect added a:b:w ...`` (insertion order) / ``expect tiles c:t:m,m,...``.
    Returns (raw graph, meta, added [(a, b, w)], tiles [(c, [members], t)])."""
    meta, edges, added, tiles = {}, [], [], []
    with open(os.path.join(HERE, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            tok = line.split()
            if tok[0] == "arc":
                edges.append((int(tok[1]), int(tok[2]), int(tok[3])))
            elif tok[0] == "edge":
                u, v, w = int(tok[1]), int(tok[2]), int(tok[3])
                edges += [(u, v, w), (v, u, w)]
            elif tok[0] == "expect" and tok[1] == "added":
                added = [] if tok[2:] == ["none"] else [tuple(int(x) for x in t.split(":")) for t in tok[2:]]
            elif tok[0] == "expect" and tok[1] == "tiles":
                for t in ([] if tok[2:] == ["none"] else tok[2:]):
                    c, it, mem = t.split(":")
                    tiles.append((int(c), [int(x) for x in mem.split(",")], int(it)))
            else:
                meta[tok[0]] = tok[1]
    n = int(meta["n"])
    edges.sort(key=lambda e: e[0])          # rows in the order written within each source
    return graphgen.from_edge_list(n, edges, name), meta, added, tiles
