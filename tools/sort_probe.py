"""Sort-phase probe: event-timed sort phase with and without an L2 flush before the step
(development aid; not the bench contract).  usage: python tools/sort_probe.py [WORKLOAD]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED

w = WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "small"]
g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
flush = torch.empty(256 << 18, dtype=torch.int32, device="cuda")
for fl in (False, True):
    for sort in ("material_energy", "material"):
        res = []
        for k in range(12):
            if fl:
                flush.fill_(k)
            st = g.lookup_range(0, w.lookups, LOOKUP_SEED, sort=sort, timing=True)
            res.append((st.sample_ms, st.lookup_ms, st.device_ms))
        res = res[2:]
        print(f"{w.name} flush={fl} sort={sort}: sort {statistics.median(r[0] for r in res):.3f} ms, "
              f"lookup {statistics.median(r[1] for r in res):.3f} ms, device {statistics.median(r[2] for r in res):.3f} ms",
              flush=True)
