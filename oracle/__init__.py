"""Graffix ORACLE -- test infrastructure only.

Plain, slow, obviously-correct CPU implementation of what the hot path
computes, written from the paper (Singh & Nasre, "Graffix", ICPP 2020;
/root/reference/PAPER.md, cited as P@<char offset> -- the paper is one
physical line) and the readings R1..R44 of SURVEY.md §8(c) (restated in
DESIGN.md "Readings").  Floating point is fp64.

ONLY tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(paper_conf_icpp_0001n20_b200/) never imports it and shares no code with it:
the only shared module is graphgen/ (seeded inputs, none of the method).

Modules
  graph      -- canonical CSR (A0), logical graph G_L, SSSP source rule.
  transform  -- §2 renumber + replicate, §3 CC edges + subgraphs,
                §4 degree buckets + padding (Alg 2, P@16373-18419; P@29857-
                32416; P@33145-35029).
  algos      -- definitions on G_L: Dijkstra SSSP, PageRank power iteration,
                Tarjan SCC, Kruskal MST, Brandes BC (Alg 1, Eq 1-2).
  slotsim    -- the paper's loop on slots (sweep + confluence/merge every
                iteration, §2.4 P@27655-28981), used to pin Theorems E1/E3.
  metrics    -- inaccuracy (P@40990-41294) and O(m) certificates.

Parity status per function is stated in each docstring;
every function is pinned to something other than itself (printed examples,
hand-derived fixtures, closed forms, brute force or library routines).
"""
