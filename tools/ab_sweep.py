"""The paper's A/B methodology on B200.

Times every search variant x {XSBench order, (material, energy) order} x 3 grid types on
one workload (median of 5 after 2 warm-ups, CUDA-event time of the lookup kernel alone) and
writes JSON lines.  `--ncu` mode instead runs each configuration twice so an outer
`ncu -k regex:k_lookup` capture sees one launch per configuration (in this order).
usage: python tools/ab_sweep.py [--workload small] [--ncu] > out.jsonl"""
import argparse, json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED

SEARCHES = ["M", "M2", "M4", "M8", "U1", "U2", "U4", "U8", "B", "W", "H"]
SORTS = ["none", "material_energy"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="small")
    ap.add_argument("--ncu", action="store_true")
    ap.add_argument("--lookups", type=int, default=0)
    a = ap.parse_args()
    w = WORKLOADS[a.workload]
    n = a.lookups or w.lookups
    for gt in (1, 0, 2):
        g = xs.Grid(w.n_nuclides, w.n_gridpoints, gt, GRID_SEED)
        for srt in SORTS:
            for s in SEARCHES:
                if a.ncu:
                    st = g.lookup_range(0, n, LOOKUP_SEED, search=s, sort=srt)
                    print(json.dumps({"grid": gt, "sort": srt, "search": s, "hash": st.hash}), flush=True)
                    continue
                for _ in range(2):
                    g.lookup_range(0, n, LOOKUP_SEED, search=s, sort=srt)
                ms = [g.lookup_range(0, n, LOOKUP_SEED, search=s, sort=srt, timing=True) for _ in range(5)]
                print(json.dumps({"workload": a.workload, "grid": gt, "sort": srt, "search": s,
                                  "lookup_ms": statistics.median(x.lookup_ms for x in ms),
                                  "total_ms": statistics.median(x.device_ms for x in ms),
                                  "hash": ms[0].hash}), flush=True)
        g.close()


if __name__ == "__main__":
    main()
