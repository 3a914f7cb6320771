#!/usr/bin/env python
"""bench.py -- Graffix B200 hot path throughput (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--workload t24|c1|c2]

A step = one pass of the whole hot path over the resident graph: an SSSP run
(source = max out-degree vertex, reading R36) plus a PageRank run (tol 1e-9)
to their fixed points on BASELINE.json's target configuration (RMAT-24,
exact mode; workload "t24").  value = edges scanned per second (GTEPS) over
all ranks; roofline = the dominant sweep kernel's algorithmic bytes per launch
/ its CUDA-event duration, against MEASURED_PEAKS.json hbm_gbs.

--impl reference times the ORACLE (the reference arm of this tier) on the
box's host cores on a bounded sample of the workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "GTEPS (edges scanned per second) of SSSP + PageRank to their fixed points"
UNIT = "GTEPS"
WORKLOADS = {
    "t24": dict(scale=24, desc="T24: RMAT-24 (GTgraph a,b,c=.45,.15,.15, EF 16), exact mode, "
                              "SSSP (R36 source, int weights 1..100) + PageRank (d=0.85, tol 1e-9)"),
    "c2": dict(scale=22, desc="C2: RMAT-22, exact mode, SSSP + PageRank"),
    "c1": dict(scale=14, desc="C1: RMAT-14, exact mode, SSSP + PageRank"),
    "c5": dict(scale=26, desc="C5 on one GPU: RMAT-26 (the paper's rmat26, P@35940), exact mode, SSSP + PageRank"),
}
CPU_SAMPLE_SCALE = 17
PR_KERNELS = {1: "k_pr_sell2", 2: "k_pr_tpv", 3: "k_pr_pb"}   # gx_mapping -> PR sweep kernel
MAPPING_NAMES = {0: "auto", 1: "lb", 2: "tpv", 3: "pb"}   # bounded oracle sample: same generator at 1/128 of T24


def _free_port() -> int:
    import socket
    so = socket.socket()
    so.bind(("127.0.0.1", 0))
    port = so.getsockname()[1]
    so.close()
    return port


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class Clocks:
    """nvidia-smi sampler running during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(device), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self) -> dict:
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        for line in open(self.f.name):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 7:
                rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"], "samples": 0}
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def oracle_sample(scale=CPU_SAMPLE_SCALE):
    """The oracle, as it stands, on the bounded sample (rank 0 only)."""
    import graphgen
    from oracle import algos as A
    from oracle.graph import from_raw, graph_to_edgelist, sssp_source
    g = from_raw(graphgen.rmat(scale))
    el = graph_to_edgelist(g)
    s = sssp_source(g)
    t0 = time.perf_counter()
    A.sssp_dijkstra(el, s)
    t1 = time.perf_counter()
    _, iters = A.pagerank(el, tol=1e-9)
    t2 = time.perf_counter()
    edges = g.m + iters * g.m     # Dijkstra relaxes each edge once; PR gathers m per iteration
    return {"edges": edges, "sec": t2 - t0, "sssp_s": t1 - t0, "pr_s": t2 - t1, "pr_iters": iters,
            "n": g.n, "m": g.m}


def inaccuracy_pct(approx, exact, inf=None):
    """PAPER.md P@40990-41294 (reading R40): 100 * sum|a - e| / sum|e| over the
    vertices finite in both runs (a metric on two GPU results, no oracle)."""
    a = np.asarray(approx, dtype=np.float64)
    e = np.asarray(exact, dtype=np.float64)
    ok = np.ones(a.shape, bool) if inf is None else (np.asarray(approx) != inf) & (np.asarray(exact) != inf)
    den = np.abs(e[ok]).sum()
    return float(100.0 * np.abs(a[ok] - e[ok]).sum() / den) if den > 0 else 0.0


GATHER_PEAK_G = 286.0   # random 4-byte gathers from a 64 MB vector (= RMAT-24 dist), 1xB200 (profiles/r1/microbench3_gather_ceiling.txt)


def knob_points(ctx, reps=2):
    """BASELINE metric's "speedup vs exact at inaccuracy%" (Tables 6 and 8,
    P@42046-42906, P@43835-44682) at three paper-style settings: C2 (RMAT-22) §2
    coalescing k=16, theta_conn=0.6 with the algorithm-aware merge; C3 (road
    grid 4900^2) §2 renumbering alone (theta_conn=2.0: no vertex can reach it, so
    no replicas -- the BFS-level isomorph of Alg 2 l.10-20 only); C4 (uniform
    16M/256M) §4 degree normalisation theta_d=0.3, f=0.85.  Per algorithm: the
    knob's best mapping vs the best exact mapping, and per mapping vs the same
    mapping exact; inaccuracy (R40) of the knob run vs the exact run; transform
    time and extra space (Table 5 analogue)."""
    import graphgen
    import paper_conf_icpp_0001n20_b200 as gx
    U32_INF = 0xFFFFFFFF
    cases = [
        ("C2 rmat22 coalesce k16 theta0.6 aware-merge", lambda: graphgen.rmat(22),
         gx.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.6, merge_op=1)),
        ("C3 road4900 coalesce k16 renumber-only (theta_conn 2.0)", lambda: graphgen.road(4900),
         gx.Knobs(coalesce=True, chunk_k=16, replicate_threshold=2.0)),
        ("C4 uniform16M/256M degnorm theta0.3 f0.85", lambda: graphgen.uniform(1 << 24, 1 << 28),
         gx.Knobs(degree_norm=True, degsim_threshold=0.3, degree_target=0.85)),
    ]
    maps = {"sssp": ("lb", "tpv"), "pagerank": ("pb", "lb", "tpv")}
    out = []
    for name, mk, kn in cases:
        # start every case from an empty caching allocator (the library allocates through
        # it): blocks cached by the earlier sections made the first SSSP runs of a later
        # graph wait on cudaMalloc retries (C4 exact SSSP 15.9 vs 3.9 ms)
        import torch
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        t0 = time.perf_counter()
        raw = mk()
        G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)

        def timed(algo, mp):
            kw = {"tol": 1e-9} if algo == "pagerank" else {}
            return min(G.run(algo, mapping=mp, **kw)["loop_ms"] for _ in range(reps))
        ex = {a: {mp: timed(a, mp) for mp in maps[a]} for a in maps}
        G.run("sssp", mapping="lb")
        de = G.download("dist").copy()
        G.run("pagerank", mapping="pb", tol=1e-9)
        xe = G.download("rank").copy()
        info = G.transform(kn)
        ap = {a: {mp: timed(a, mp) for mp in maps[a]} for a in maps}
        G.run("sssp", mapping="auto")
        da = G.download("dist")
        G.run("pagerank", mapping="auto", tol=1e-9)
        xa = G.download("rank")
        inacc = {"sssp": inaccuracy_pct(da, de, U32_INF), "pagerank": inaccuracy_pct(xa, xe)}
        pt = {}
        for a in maps:
            best_e = min(ex[a].values())
            best_k = min(ap[a].values())
            pt[a] = {"exact_ms": ex[a], "knob_ms": ap[a],
                     "speedup_vs_best_exact": best_e / best_k,
                     "speedup_same_mapping": {mp: ex[a][mp] / ap[a][mp] for mp in maps[a]},
                     "inaccuracy_pct": inacc[a]}
        out.append({"config": name, "n": G.n, "m": G.m, "transform_s": info["transform_ms"] / 1e3,
                    "extra_space_pct": info["extra_space_pct"], "algos": pt,
                    "wall_s": time.perf_counter() - t0})
        G.close()
    return out


def cpu_cores_used() -> int:
    return 1   # the oracle is single-threaded Python/numpy (numpy bincount is serial)


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


class pinned_core:
    """Run the oracle on one host core (os.sched_setaffinity, the taskset of
    SURVEY §8(d)); the previous affinity is restored afterwards."""
    def __enter__(self):
        self.old = os.sched_getaffinity(0)
        self.core = min(self.old)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.old)


def oracle_knob_points():
    """The oracle on C1 (RMAT-14) per knob setting (the oracle per
    (graph, knob) point in the same job): transform, Dijkstra and fp64 PageRank
    on the transformed graph's G_L, seconds each (bounded: a few seconds)."""
    import graphgen
    from oracle import algos as A
    from oracle import transform as T
    from oracle.graph import from_raw, graph_to_edgelist, sssp_source
    g = from_raw(graphgen.rmat(14))
    pts = []
    for name, kn in (("exact", None), ("coalesce k16 theta0.6", T.Knobs(coalesce=True)),
                     ("degnorm theta0.3", T.Knobs(degree_norm=True, degsim_threshold=0.3))):
        t0 = time.perf_counter()
        el = T.transform(g, kn).logical() if kn else graph_to_edgelist(g)
        t1 = time.perf_counter()
        A.sssp_dijkstra(el, sssp_source(g))
        t2 = time.perf_counter()
        _, it = A.pagerank(el, tol=1e-9)
        t3 = time.perf_counter()
        pts.append({"config": f"C1 rmat14 {name}", "transform_s": t1 - t0, "sssp_s": t2 - t1, "pagerank_s": t3 - t2,
                    "pagerank_iterations": it})
    return pts


def run_reference(args, rank, world):
    if rank != 0:
        return 0
    with pinned_core() as pc:
        for _ in range(args.warmup):
            oracle_sample()
        res = [oracle_sample() for _ in range(args.steps)]
    edges = sum(r["edges"] for r in res)
    sec = sum(r["sec"] for r in res)
    v = edges / sec / 1e9
    sample = (f"oracle (oracle/algos.py Dijkstra + fp64 power-iteration PR to tol 1e-9) on RMAT-{CPU_SAMPLE_SCALE} "
              f"(same generator, n={res[0]['n']}, m={res[0]['m']}), 1/{1 << (24 - CPU_SAMPLE_SCALE)} of T24")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sec / len(res),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32/f64",
            "data": "synthetic", "config": {"workload": WORKLOADS[args.workload]["desc"], "graph": f"rmat{WORKLOADS[args.workload]['scale']}",
                                            "sample": f"rmat{CPU_SAMPLE_SCALE}"},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": cpu_cores_used(), "kind": "oracle",
                             "sample": sample, "cpu_model": cpu_model(),
                             "pinned": f"host core {pc.core} (os.sched_setaffinity)"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="t24", choices=list(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-knobs", action="store_true", help="skip the knob speedup / inaccuracy points (~90 s)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--e2e-sync", action="store_true", help="upload without GX_ASYNC_UPLOAD")
    ap.add_argument("--e2e-w32", action="store_true", help="upload 32-bit weights (not GX_W_U8)")
    ap.add_argument("--pr-mapping", default="auto", choices=["auto", "lb", "tpv", "pb"],
                    help="PageRank sweep mapping (auto = the blocked pull on one GPU at these sizes)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world == 0 and args.gpus > 1 and args.impl == "ours":
        # not under torchrun: start the N ranks ourselves (one process per GPU)
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
        return subprocess.call(cmd)
    world = world or 1
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if world != args.gpus:
        raise SystemExit(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}")

    import torch
    import torch.distributed as dist
    import graphgen
    import paper_conf_icpp_0001n20_b200 as gx

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    wl = WORKLOADS[args.workload]
    raw = graphgen.rmat(wl["scale"])
    # N > 1: one process per GPU, 1-D partitioned sweeps with NCCL exchange
    ctx = gx.Context.distributed(local, rank, world) if world > 1 else gx.Context(local)
    stream = torch.cuda.ExternalStream(ctx.stream_ptr)
    G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
    n, m = G.n, G.m
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    def step(profile):
        a = G.run("sssp", source=-1, mapping="lb", profile=profile)
        b = G.run("pagerank", tol=1e-9, mapping=args.pr_mapping, profile=profile)
        return a, b

    for _ in range(args.warmup):
        step(False)
    # ---------------- timed region (inputs resident in HBM) ----------------
    clk = Clocks(local) if rank == 0 else None
    runs = []
    t_ms = []
    for _ in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(1)                      # L2 flush between steps (not timed)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        a, b = step(True)
        e1.record(stream)
        torch.cuda.synchronize()
        runs.append((a, b))
        t_ms.append(e0.elapsed_time(e1))
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks = clk.stop() if clk else None
    tot_ms = float(sum(t_ms))
    if world > 1:
        tt = torch.tensor([tot_ms], device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        tot_ms = float(tt.item())
    # edges scanned are counted per rank (SSSP relaxations of its rows, PR
    # in-edges of its rows per sweep): the job's total is the sum over ranks
    edges = sum(a["edges_scanned"] + b["edges_scanned"] for a, b in runs)
    if world > 1:
        te = torch.tensor([float(edges)], device="cuda", dtype=torch.float64)
        dist.all_reduce(te)
        edges = int(te.item())
    value = edges / (tot_ms * 1e-3) / 1e9
    launches = sum(a["kernel_launches"] + b["kernel_launches"] for a, b in runs)

    # dominant kernel roofline (live CUDA events around each sweep launch on the
    # library's stream).  One GPU: SSSP is ONE cooperative launch per run
    # (k_sssp_persist, the whole fixed-point loop); PageRank one launch per
    # sweep.  N > 1: the partitioned loops (sweeps + NCCL exchange) per rank.
    peak, peak_src = peaks()
    kern = {}
    pr_kernel = PR_KERNELS.get(runs[-1][1].get("mapping_used", 1), "k_pr_sell2")
    sssp_kernel = "k_sssp_persist" if world == 1 else "sssp partitioned loop (k_sssp_lb + exchange)"
    if world > 1:
        pr_kernel = "pagerank partitioned loop (k_pr_sell2 + exchange)"
    for name, idx in ((sssp_kernel, 0), (pr_kernel, 1)):
        if world == 1:
            ms = sum(r[idx]["sweep_ms"] for r in runs)
            # SSSP: the one cooperative launch per run; PR: the sweeps that did work
            # (a CUDA-graph batch may end with launches that return at once after
            # convergence; their ~3 us stay in ms, so this slightly under-claims)
            nl = sum(r[idx]["sweep_launches"] if idx == 0 else r[idx]["iterations"] for r in runs)
        else:
            ms = sum(r[idx]["loop_ms"] for r in runs)
            nl = len(runs)
        it = sum(r[idx]["iterations"] for r in runs)
        by = sum(r[idx]["bytes_model"] for r in runs)        # algorithmic (SURVEY §8(d) model)
        enc = sum(r[idx].get("sweep_bytes", 0) or r[idx]["bytes_model"] for r in runs)   # the kernel's encoding
        kern[name] = {"ms_total": ms, "launches": nl, "iterations": it, "bytes": by, "encoding_bytes": enc,
                      "gbs": by / (ms * 1e-3) / 1e9 if ms > 0 else None,
                      "encoding_gbs": enc / (ms * 1e-3) / 1e9 if ms > 0 else None,
                      "share_of_step": ms / tot_ms if tot_ms else None}
    dom = max(kern, key=lambda k: kern[k]["ms_total"])
    dk = kern[dom]
    achieved = dk["gbs"]
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "latest", "traffic.json")
    if os.path.exists(tpath):
        tj = json.load(open(tpath))
        if dom in tj and tj[dom].get("graph", "rmat24") == f"rmat{wl['scale']}":
            traffic = tj[dom]["traffic_bytes_per_launch"]
    # PR: a launch is one sweep (8 B/in-edge + 32 B/slot); SSSP: one launch is the whole loop
    roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak if achieved else None, "traffic": traffic,
                "traffic_unit": "bytes/launch (ncu dram read+write, profiles/latest)", "peak_source": peak_src,
                "bytes_per_launch": dk["bytes"] / max(dk["launches"], 1),
                "us_per_launch": 1e3 * dk["ms_total"] / max(dk["launches"], 1),
                "bytes_model": "SURVEY §8(d): PR 8 B/in-edge + 32 B/slot per sweep; SSSP 12 B/relaxed edge + 12 B/frontier slot"}
    if dk["encoding_bytes"] != dk["bytes"]:
        # k_pr_pb streams 12 B per edge where the §8(d) pull model counts 8 B
        # (it trades the random contrib gathers for streamed terms): frac above
        # is on the §8(d) bytes; this is the same time on the bytes it moves
        roofline["encoding"] = {"bytes_per_launch": dk["encoding_bytes"] / max(dk["launches"], 1),
                                "achieved": dk["encoding_gbs"], "frac": dk["encoding_gbs"] / peak,
                                "model": "12 B/edge + 28 B/slot (blocked pull: terms streamed along edges)"}

    a0, b0 = runs[-1]
    per_algo = {
        "sssp": {"gteps": a0["edges_scanned"] / (a0["loop_ms"] * 1e-3) / 1e9, "gteps_solution": m / (a0["loop_ms"] * 1e-3) / 1e9,
                 "iterations": a0["iterations"], "loop_ms": a0["loop_ms"], "edges_scanned": a0["edges_scanned"],
                 "roofline_frac": (a0["bytes_model"] / (a0["loop_ms"] * 1e-3) / 1e9) / peak,
                 # every relaxed edge costs one random 4-byte gather of dist (one L1TEX wavefront per
                 # distinct sector), which caps the sweep below HBM: the measured ceiling of random
                 # gathers from an L2-resident vector on this B200 (tools/microbench.cu) is the
                 # secondary roofline the SSSP loop is judged against
                 "gather_roofline": {"bound": "l1tex (random 4-B gathers, L2-resident)",
                                     "achieved": a0["edges_scanned"] / (a0["loop_ms"] * 1e-3) / 1e9,
                                     "peak": GATHER_PEAK_G, "unit": "G gathers/s",
                                     "frac": a0["edges_scanned"] / (a0["loop_ms"] * 1e-3) / 1e9 / GATHER_PEAK_G,
                                     "peak_source": "measured, profiles/r1/microbench3_gather_ceiling.txt "
                                                    "(285-287 G/s at 4-64 MB)"}},
        "pagerank": {"gteps": b0["edges_scanned"] / (b0["loop_ms"] * 1e-3) / 1e9, "iterations": b0["iterations"],
                     "loop_ms": b0["loop_ms"], "last_delta": b0["last_delta"],
                     "roofline_frac": (b0["bytes_model"] / (b0["loop_ms"] * 1e-3) / 1e9) / peak},
    }

    # ---------------- e2e through the public API with host buffers ----------------
    e2e = None
    if not args.no_e2e:
        ex = G.export()      # canonical graph (exact mode), rows sorted: caller-side canonical input
        hrp = torch.from_numpy(ex["row_ptr"]).pin_memory()
        hcol = torch.from_numpy(ex["col"]).pin_memory()
        # weights 1..100 travel as bytes (GX_W_U8, widened on the device)
        assert int(ex["w"].max()) <= 255
        hw = torch.from_numpy(ex["w"].view(np.int32) if args.e2e_w32 else ex["w"].astype(np.uint8)).pin_memory()
        hdist = torch.empty(n, dtype=torch.int32).pin_memory()
        hrank = torch.empty(n, dtype=torch.float64).pin_memory()
        h2d = hrp.numel() * 8 + hcol.numel() * 4 + hw.numel() * hw.element_size()
        d2h = n * 4 + n * 8
        e2e_ms, e2e_edges = [], 0
        # two untimed passes: the torch caching allocator (hooked into the library) takes
        # two passes to hold every block size the upload and the layout builds ask for
        # (profiles/r2/e2e_variance.txt: 125-142 ms PageRank calls in passes 0-1, 18.7 ms after)
        E2E_WARM = 2
        for i in range(args.e2e_steps + E2E_WARM):
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            # GX_ASYNC_UPLOAD: the weights' H2D overlaps the blocked PageRank
            # (structure only); SSSP joins the copy
            G2 = gx.Graph.upload(ctx, hrp.numpy(), hcol.numpy(),
                                 hw.numpy().view(np.uint32) if args.e2e_w32 else hw.numpy(), canonical=True,
                                 async_upload=not args.e2e_sync)
            b = G2.run("pagerank", tol=1e-9, mapping=args.pr_mapping)
            G2.download("rank", out=hrank.numpy(), async_copy=not args.e2e_sync)   # D2H overlaps SSSP
            a = G2.run("sssp", source=-1, mapping="lb")
            G2.download("dist", out=hdist.numpy().view(np.uint32))
            ctx.sync()
            e1.record(stream)
            torch.cuda.synchronize()
            G2.close()
            if i >= E2E_WARM:
                e2e_ms.append(e0.elapsed_time(e1))
                e2e_edges += a["edges_scanned"] + b["edges_scanned"]
        t = sum(e2e_ms)
        if world > 1:
            tt = torch.tensor([t], device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            t = float(tt.item())
            te = torch.tensor([float(e2e_edges)], device="cuda", dtype=torch.float64)
            dist.all_reduce(te)
            e2e_edges = int(te.item())
        e2e = {"value": e2e_edges / (t * 1e-3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h, "ms_per_step": t / len(e2e_ms),
               "note": "upload of canonical pinned CSR with 8-bit weights (GX_CANONICAL | GX_W_U8" + ("" if args.e2e_sync else " | GX_ASYNC_UPLOAD: weights H2D overlapping the blocked PR; rank D2H (GX_DL_ASYNC) overlapping SSSP") + ") + device layouts (blocked-PR segments, SSSP heavy chunks) + PR + download rank + SSSP + download dist"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        with pinned_core() as pc:
            r = oracle_sample()
            knob_pts = oracle_knob_points()
        cpu = {"value": r["edges"] / r["sec"] / 1e9, "unit": UNIT, "cores": cpu_cores_used(), "kind": "oracle",
               "sample": f"oracle Dijkstra + fp64 PR (tol 1e-9, {r['pr_iters']} iters) on RMAT-{CPU_SAMPLE_SCALE} "
                         f"(n={r['n']}, m={r['m']}; same generator, 1/{1 << (24 - CPU_SAMPLE_SCALE)} of T24), "
                         f"{r['sec']:.1f} s", "host_cores": os.cpu_count(), "cpu_model": cpu_model(),
               "pinned": f"host core {pc.core} (os.sched_setaffinity)", "knob_points": knob_pts}

    knobs = None
    if rank == 0 and world == 1 and not args.no_knobs:
        knobs = knob_points(ctx)

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": tot_ms / args.steps, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "u32/f64", "data": "synthetic",
                "config": {"workload": wl["desc"], "graph": f"rmat{wl['scale']}", "n": n, "m": m,
                           "knobs": "exact",
                           "mapping": {"sssp": MAPPING_NAMES.get(runs[-1][0].get("mapping_used", 1), "lb"),
                                       "pagerank": MAPPING_NAMES.get(runs[-1][1].get("mapping_used", 1), "?")}, "l2": "flushed between steps (256 MiB write)",
                           "parallelism": f"1-D partitioned x{world} (NCCL)" if world > 1 else "single"},
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
                "clocks": clocks, "per_algo": per_algo, "kernels": kern, "knobs": knobs}
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
