"""Render tools/knob_sweep.py JSON lines as a table."""
import glob
import json
import sys

for f in sorted(glob.glob(sys.argv[1] + "/*.jsonl")):
    print("==", f.split("/")[-1])
    for line in open(f):
        d = json.loads(line)
        if "P" in d:
            print(f"  [{d['knob']}] P={d['P']} ({d['note']}): SSSP {d['sssp_ms']:.2f} ms ({d['sssp_iters']} it) | "
                  f"PR {d['pagerank_ms']:.2f} ms ({d['pagerank_iters']} it)")
            continue
        if "sssp_lb_ms" not in d and "pagerank_lb_ms" not in d:   # other tools' lines (algos_c4)
            print("  " + ", ".join(f"{k}={v:.3g}" if isinstance(v, float) else f"{k}={v}" for k, v in d.items()
                                   if k not in ("config", "graph", "n", "m")))
            continue
        if d["knob"] == "exact":
            pbx = f" pb {d['pr_pb_ms']:.2f}" if "pr_pb_ms" in d else ""
            print(f"  {d['graph']} exact: SSSP lb {d['sssp_lb_ms']:.2f} ms tpv {d['sssp_tpv_ms']:.2f} | PR lb {d['pr_lb_ms']:.2f} tpv {d['pr_tpv_ms']:.2f}{pbx} ({d['pr_iters']} it)")
            continue
        print(f"  {d['knob']:30s} tr {d['transform_s']:5.1f}s +{d['extra_space_pct']:5.2f}% | SSSP tpv {d['sssp_tpv_ms']:7.2f} "
              f"({d['sssp_tpv_speedup_same_mapping']:.2f}x) lb {d['sssp_lb_ms']:6.2f} ({d['sssp_lb_speedup_same_mapping']:.2f}x) "
              f"inacc {d['sssp_inacc_pct']:.2f}% | PR tpv {d['pagerank_tpv_ms']:7.2f} ({d['pagerank_tpv_speedup_same_mapping']:.2f}x) "
              f"lb {d['pagerank_lb_ms']:6.2f} ({d['pagerank_lb_speedup_same_mapping']:.2f}x)"
              + (f" pb {d['pagerank_pb_ms']:6.2f} ({d['pagerank_pb_speedup_same_mapping']:.2f}x, "
                 f"{d['pagerank_pb_speedup_vs_best_exact']:.2f}x best)" if "pagerank_pb_ms" in d else "")
              + f" inacc {d['pr_inacc_pct']:.2f}% it {d['pr_lb_iters']}")
