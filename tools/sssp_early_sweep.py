import os, sys
sys.path.insert(0, os.getcwd())
import graphgen, paper_conf_icpp_0001n20_b200 as gx
for gname, mk in (("rmat24", lambda: graphgen.rmat(24)), ("uniform24", lambda: graphgen.uniform(1 << 24, 1 << 28)), ("road4900", lambda: graphgen.road(4900))):
    raw = mk(); ctx = gx.Context(0); G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
    base = None
    for early in [0, 64, 256, 1024, 4096, 16384, 65536]:
        os.environ["GX_SSSP_EARLY"] = str(early)
        rs = [G.run("sssp", mapping="lb") for _ in range(4)]
        r = min(rs, key=lambda q: q["loop_ms"])
        d = G.download("dist")
        if base is None: base = d.copy()
        import numpy as np
        print(f"{gname} early={early} loop_ms={r['loop_ms']:.3f} iters={r['iterations']} edges={r['edges_scanned']} same={np.array_equal(d, base)}", flush=True)
    G.close()
