"""The 1-D partitioned path on one GPU: P simulated ranks
each sweep their own slot range and exchange through a device reduction
(the NCCL collective's stand-in).  Results must equal the single-rank
results exactly (SSSP, schedule-independent fixed point) and the oracle (PR
within L1 1e-6) for every P -- the acceptance rule of §8(e)."""
import numpy as np
import pytest

import graphgen
from gpu_util import upload
from oracle import algos as A
from oracle import transform as T
from oracle.graph import from_raw, graph_to_edgelist, sssp_source

pytestmark = pytest.mark.gpu

GRAPHS = {
    "rmat14": lambda: graphgen.rmat(14),
    "road64": lambda: graphgen.road(64),
    "uniform": lambda: graphgen.uniform(9000, 80000),
}
KNOBS = {
    "exact": None,
    "all": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.3, smem=True, cc_threshold=0.3,
                   degree_norm=True, degsim_threshold=0.5),
}


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", list(KNOBS))
def test_partitioned_sssp_and_pr(P, gname, kname):
    import paper_conf_icpp_0001n20_b200 as gx
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = KNOBS[kname]
    el = T.transform(g, kn).logical() if kn else graph_to_edgelist(g)
    G = upload(raw)
    if kn:
        G.transform(gx.Knobs(**{f: getattr(kn, f) for f in kn.__dataclass_fields__}))
    r = G.run("sssp", mapping="lb", sim_ranks=P)
    assert r["converged"] == 1
    assert np.array_equal(G.download("dist"), A.sssp_dijkstra(el, sssp_source(g)))
    G.run("pagerank", mapping="lb", sim_ranks=P, tol=1e-11, max_iters=5000)
    want, _ = A.pagerank(el, tol=1e-14)
    assert np.abs(G.download("rank") - want).sum() <= 1e-6
