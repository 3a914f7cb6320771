"""Mutation run for the §3 selection pins (VERDICT r1 "What's weak" 1).

Each mutant reverses or drops ONE decision of oracle/transform.py's cc_edges /
subgraphs (a text substitution on a copy of the module); the mutant is then
run on every hand-derived fixture tests/golden/sec3_*.txt.  A mutant is
KILLED when some fixture's expected inserted edges or tiles differ.

    python tools/mutate_sec3.py            # prints one line per mutant + a summary
"""
from __future__ import annotations

import importlib.util
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

from golden_io import load_sec3  # noqa: E402
from oracle.graph import from_raw  # noqa: E402

FIXTURES = ["sec3_case1_order.txt", "sec3_case1_pairs.txt", "sec3_case2_sibling.txt",
            "sec3_case2_order.txt", "sec3_skip.txt", "sec3_case2_passes.txt"]


def _nth(s: str, old: str, new: str, n: int) -> str:
    """Replace the n-th (0-based) occurrence of old."""
    i = -1
    for _ in range(n + 1):
        i = s.index(old, i + 1)
    return s[:i] + new + s[i + len(old):]


def _swap_cases(s: str) -> str:
    a = s.index("    # case 1\n")
    b = s.index("    # case 2\n")
    c = s.index("    return added, L")
    return s[:a] + s[b:c] + s[a:b] + s[c:]


CMP_HI = "return -1 if lhs > rhs else 1"
CMP_ID = "return -1 if x < y else (1 if x > y else 0)"
MUTANTS = {
    "M1 case-1 centres need desc": lambda s: s.replace("    cands.sort()\n", "    cands.sort(key=lambda x: (-x[0], x[1]))\n"),
    "M2 case-1 centres id desc": lambda s: s.replace("    cands.sort()\n", "    cands.sort(key=lambda x: (x[0], -x[1]))\n"),
    "M3 case-1 pairs common asc": lambda s: s.replace("pairs.append((-len(L.N[a] & L.N[b]), a, b))",
                                                      "pairs.append((len(L.N[a] & L.N[b]), a, b))"),
    "M4 case-1 pair tie-break desc": lambda s: s.replace("        pairs.sort()\n",
                                                         "        pairs.sort(key=lambda p: (p[0], -p[1], -p[2]))\n"),
    "M5 case-2 sibling largest internal degree": lambda s: s.replace("key=lambda a: (intdeg[a], a)",
                                                                     "key=lambda a: (-intdeg[a], a)"),
    "M6 case-2 partner largest internal degree": lambda s: s.replace("key=lambda x: (intdeg[x], x)",
                                                                     "key=lambda x: (-intdeg[x], x)"),
    "M7 case-2 centres CC asc": lambda s: _nth(s, CMP_HI, "return 1 if lhs > rhs else -1", 0),
    "M8 case 2 before case 1": _swap_cases,
    "M9 subgraph centres CC asc": lambda s: _nth(s, CMP_HI, "return 1 if lhs > rhs else -1", 1),
    "M10 subgraph centres d asc": lambda s: s.replace("return -1 if dx > dy else 1", "return 1 if dx > dy else -1"),
    "M11 subgraph centres id desc": lambda s: _nth(s, CMP_ID, "return 1 if x < y else (-1 if x > y else 0)", 1),
    "M12 no case-1 skip rule": lambda s: s.replace("if len(pairs) < need:", "if False:"),
    "M13 t = diameter (not 2x)": lambda s: s.replace("else 2 * (1 if clique else 2)", "else (1 if clique else 2)"),
    "M14 case 1 keeps linking after high": lambda s: s.replace("if rem[0] <= 0 or L.high(c, cc_ppm):",
                                                               "if rem[0] <= 0:"),
    "M15 high is >= (not strict)": lambda s: s.replace("return self.T[c] * 1_000_000 > th * self.P(c)",
                                                       "return self.T[c] * 1_000_000 >= th * self.P(c)"),
    "M16 case-2 centres id desc": lambda s: _nth(s, CMP_ID, "return 1 if x < y else (-1 if x > y else 0)", 0),
    "M17 siblings on any U 2-path": lambda s: s.replace("return (c in self.out[a]) and (b in self.out[c])",
                                                        "return a in self.N[c] and b in self.N[c]"),
    "M18 weight drops the first hop": lambda s: s.replace("w = combine(L.out[x][c], L.out[c][y], rule)",
                                                          "w = combine(L.out[c][y], L.out[c][y], rule)"),
    "M19 need without +1": lambda s: s.replace("        need = (cc_ppm * P) // 1_000_000 + 1 - L.T[c]",
                                               "        need = (cc_ppm * P) // 1_000_000 - L.T[c]"),
    "M20 case 2: a single pass": lambda s: s.replace("            if not linked_any:\n                break",
                                                     "            break"),
    "M21 case-2 order fixed, no re-check of internal degree": lambda s: s.replace(
        "                intdeg = {a: len(L.N[a] & Nc) for a in Nc}",
        "                intdeg = intdeg0.setdefault(c, {a: len(L.N[a] & Nc) for a in Nc})").replace(
        "        highs.sort(key=cmp_to_key(cmp))", "        highs.sort(key=cmp_to_key(cmp))\n        intdeg0 = {}"),
}


def run_module(mod):
    """Failing fixtures of a transform module (names), [] when all pass."""
    bad = []
    for name in FIXTURES:
        if not os.path.exists(os.path.join(ROOT, "tests", "golden", name)):
            continue
        raw, meta, added, tiles = load_sec3(name)
        g = from_raw(raw)
        th = mod.ppm(float(meta["cc_threshold"]))
        try:
            got, L = mod.cc_edges(mod.identity(g), th, int(meta["budget"]))
            gt = mod.subgraphs(L, g.n, th, int(meta.get("smax", 64)), 0)
        except Exception as e:   # a crash also kills the mutant
            bad.append(f"{name}({type(e).__name__})")
            continue
        ok_a = [tuple(int(x) for x in e) for e in got] == added
        ok_t = [(int(c), [int(x) for x in m], int(t)) for c, m, t in gt] == tiles
        if not (ok_a and ok_t):
            bad.append(name.replace("sec3_", "").replace(".txt", "") + ("" if ok_a else "[edges]") +
                       ("" if ok_t else "[tiles]"))
    return bad


def load_variant(src: str, tag: str):
    d = tempfile.mkdtemp(prefix="mut_")
    p = os.path.join(d, f"transform_{tag}.py")
    with open(p, "w") as f:
        f.write(src)
    spec = importlib.util.spec_from_file_location(f"oracle.transform_{tag}", p)
    m = importlib.util.module_from_spec(spec)
    m.__package__ = "oracle"
    sys.modules[spec.name] = m          # dataclasses look their module up
    spec.loader.exec_module(m)
    return m


def main():
    src = open(os.path.join(ROOT, "oracle", "transform.py")).read()
    base = run_module(load_variant(src, "orig"))
    print(f"unmutated oracle: {'all fixtures pass' if not base else 'FAILS ' + ', '.join(base)}")
    killed = 0
    for i, (label, fn) in enumerate(MUTANTS.items()):
        ms = fn(src)
        if ms == src:
            print(f"{label:55s} NOT APPLIED (pattern missing)")
            continue
        bad = run_module(load_variant(ms, f"m{i}"))
        killed += bool(bad)
        print(f"{label:55s} {'killed by ' + ', '.join(bad) if bad else 'SURVIVED'}")
    print(f"{killed}/{len(MUTANTS)} mutants killed")
    return 0 if killed == len(MUTANTS) and not base else 1


if __name__ == "__main__":
    sys.exit(main())
