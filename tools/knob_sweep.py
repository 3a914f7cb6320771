"""Graffix knob sweeps (paper Figs 7-9, Tables 5-8).

For each (graph, knob) point: host transform time and extra space (Table 5
analogue), SSSP and PageRank device time with the paper's thread-per-vertex
mapping and with the LB mapping, speedup against exact mode with the SAME
mapping and against the best exact kernel, and inaccuracy against the exact
run (P@40990: 100 * sum|a - e| / sum|e|).  Results: one JSON line per point.

    python tools/knob_sweep.py --config c1 [--scale-down] > profiles/r1/knobs_c1.jsonl
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402


def inacc(a, e, inf=None):
    a = np.asarray(a, dtype=np.float64)
    e = np.asarray(e, dtype=np.float64)
    if inf is not None:
        ok = (a != inf) & (e != inf)
        a, e = a[ok], e[ok]
    s = np.abs(e).sum()
    return float(100.0 * np.abs(a - e).sum() / s) if s > 0 else 0.0


def timed(G, algo, mapping, reps=3, **kw):
    best = None
    for _ in range(reps):
        r = G.run(algo, mapping=mapping, **kw)
        best = r if best is None or r["loop_ms"] < best["loop_ms"] else best
    return best


def graph_for(cfg, small):
    if cfg == "c1":
        return graphgen.rmat(14), "rmat14"
    if cfg == "c2":
        s = 20 if small else 22
        return graphgen.rmat(s), f"rmat{s}"
    if cfg in ("c3", "c3cc", "c3conn"):
        side = 1024 if small else 4900
        return graphgen.road(side), f"road{side}"
    if cfg == "c4":
        n, m = ((1 << 22, 1 << 26) if small else (1 << 24, 1 << 28))
        return graphgen.uniform(n, m), f"uniform{n}x{m}"
    if cfg == "c5":
        s = 24 if small else 26
        return graphgen.rmat(s), f"rmat{s}"
    raise ValueError(cfg)


def points(cfg):
    K = gx.Knobs
    if cfg == "c1":
        return [("coalesce k16 t0.6", K(coalesce=True)), ("coalesce k16 t0.6 aware-merge", K(coalesce=True, merge_op=1)),
                ("smem t0.5 b1%", K(smem=True)),
                ("degnorm t0.3", K(degree_norm=True)), ("degnorm t0.5", K(degree_norm=True, degsim_threshold=0.5)),
                ("all three", K(coalesce=True, smem=True, degree_norm=True))]
    if cfg == "c2":
        return [(f"coalesce t{t}", K(coalesce=True, replicate_threshold=t)) for t in (2.0, 0.9, 0.6, 0.3)] + \
               [(f"coalesce t{t} aware-merge", K(coalesce=True, replicate_threshold=t, merge_op=1)) for t in (0.9, 0.6, 0.3)]
    if cfg == "c3":
        return [(f"smem t0.5 budget {b}%", K(smem=True, cc_threshold=0.5, added_edge_budget=-2 if b < 0 else 0))
                for b in (0,)] + [(f"coalesce road t{t}", K(coalesce=True, replicate_threshold=t)) for t in (0.4, 0.6)]
    if cfg == "c3cc":   # Fig 8 (P@52695-53380): the CC threshold at a 1% budget
        return [(f"smem tcc{t} budget 1%", K(smem=True, cc_threshold=t)) for t in (0.3, 0.4, 0.5, 0.6, 0.7, 0.8, 0.9)]
    if cfg == "c3conn":   # Fig 7's connectedness sweep on the road grid (replication only bites here)
        return [(f"coalesce road t{t}", K(coalesce=True, replicate_threshold=t)) for t in (2.0, 0.9, 0.6, 0.4, 0.2)] + \
               [(f"coalesce road t{t} aware-merge", K(coalesce=True, replicate_threshold=t, merge_op=1)) for t in (0.4,)]
    if cfg == "c4":
        return [(f"degnorm t{t}", K(degree_norm=True, degsim_threshold=t)) for t in (0.0, 0.1, 0.2, 0.3, 0.4, 0.5)]
    if cfg == "c5":
        return [("all three", K(coalesce=True, smem=True, degree_norm=True)),
                ("all three aware-merge", K(coalesce=True, smem=True, degree_norm=True, merge_op=1))]
    raise ValueError(cfg)


def c5_partitioned(G, tag, base):
    """C5: the 1-D partitioned path at P = 1, 2, 4, 8 -- simulated ranks on one
    GPU (each rank's sweep + the exchange as a device reduction), so these
    times are the partitioned algorithm's cost on one device, not scaling."""
    for P in (1, 2, 4, 8):
        row = dict(base, knob=tag, P=P, note="simulated ranks on 1 GPU")
        for algo in ("sssp", "pagerank"):
            kw = {"tol": 1e-9} if algo == "pagerank" else {}
            r = G.run(algo, mapping="lb", sim_ranks=P if P > 1 else 0, **kw)
            row[f"{algo}_ms"] = r["loop_ms"]
            row[f"{algo}_iters"] = r["iterations"]
        print(json.dumps(row), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c1", choices=["c1", "c2", "c3", "c3cc", "c3conn", "c4", "c5"])
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--scale-down", action="store_true")
    ap.add_argument("--budgets", default="0,0.1,0.5,1,2,5")
    a = ap.parse_args()
    raw, gname = graph_for(a.config, a.scale_down)
    ctx = gx.Context(0)
    G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
    m = G.m
    # exact baselines: LB (best exact kernel) and TPV (same mapping as the knob runs)
    ex = {}
    for mp in ("lb", "tpv"):
        ex[("sssp", mp)] = timed(G, "sssp", mp)
        ex[("pagerank", mp)] = timed(G, "pagerank", mp, tol=1e-9)
    ex[("pagerank", "pb")] = timed(G, "pagerank", "pb", tol=1e-9)   # blocked pull (PR only)
    best = {a_: min(v["loop_ms"] for (al, _), v in ex.items() if al == a_) for a_ in ("sssp", "pagerank")}
    d0 = G.download("dist")
    G.run("pagerank", mapping="lb", tol=1e-9)
    x0 = G.download("rank")
    if a.config == "c5":
        c5_partitioned(G, "exact", {"graph": gname, "n": G.n, "m": m, "config": "c5"})
    pts = points(a.config)
    if a.config == "c3":
        pts = [(f"smem t0.5 budget {b}%", gx.Knobs(smem=True, cc_threshold=0.5, added_edge_budget=int(float(b) / 100 * m)))
               for b in a.budgets.split(",")] + pts[1:]
    base = {"graph": gname, "n": G.n, "m": m, "config": a.config}
    print(json.dumps(dict(base, knob="exact", sssp_lb_ms=ex[("sssp", "lb")]["loop_ms"],
                          sssp_tpv_ms=ex[("sssp", "tpv")]["loop_ms"], pr_lb_ms=ex[("pagerank", "lb")]["loop_ms"],
                          pr_tpv_ms=ex[("pagerank", "tpv")]["loop_ms"], pr_pb_ms=ex[("pagerank", "pb")]["loop_ms"],
                          pr_iters=ex[("pagerank", "lb")]["iterations"])),
          flush=True)
    for name, kn in pts:
        t0 = time.perf_counter()
        info = G.transform(kn)
        t_tr = time.perf_counter() - t0
        row = dict(base, knob=name, transform_s=t_tr, extra_space_pct=info["extra_space_pct"],
                   n_slots=info["n_slots"], m_slots=info["m_slots"], replicas=info["n_replicas"],
                   holes=info["n_holes"], added_coalesce=info["edges_added_coalesce"],
                   added_smem=info["edges_added_smem"], added_degnorm=info["edges_added_degnorm"],
                   subgraphs=info["n_subgraphs"])
        for algo in ("sssp", "pagerank"):
            for mp in (("tpv", "lb", "pb") if algo == "pagerank" else ("tpv", "lb")):
                r = timed(G, algo, mp, reps=a.reps, **({"tol": 1e-9} if algo == "pagerank" else {}))
                row[f"{algo}_{mp}_ms"] = r["loop_ms"]
                row[f"{algo}_{mp}_speedup_same_mapping"] = ex[(algo, mp)]["loop_ms"] / r["loop_ms"]
                row[f"{algo}_{mp}_speedup_vs_best_exact"] = best[algo] / r["loop_ms"]
                if algo == "pagerank":
                    row[f"pr_{mp}_iters"] = r["iterations"]
            if algo == "sssp":
                row["sssp_inacc_pct"] = inacc(G.download("dist"), d0, inf=0xFFFFFFFF)
                row["sssp_exact_match"] = bool(np.array_equal(G.download("dist"), d0))
            else:
                row["pr_inacc_pct"] = inacc(G.download("rank"), x0)
        print(json.dumps(row), flush=True)
        if a.config == "c5":
            c5_partitioned(G, name, base)
        G.transform(None)


if __name__ == "__main__":
    main()
