"""Lookup-kernel A/B of search variants on one workload (refined sorted order): median
sort / lookup / step event times of N steps, L2 flushed before each; hashes must agree.
usage: python tools/search_ab.py WORKLOAD STEPS SEARCH [SEARCH ...]"""
import os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED

w = WORKLOADS[sys.argv[1]]
steps = int(sys.argv[2])
g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
flush = torch.empty(256 << 18, dtype=torch.int32, device="cuda")
for search in sys.argv[3:] * 2:
    s_ms, l_ms, t_ms, hashes = [], [], [], set()
    for k in range(steps + 2):
        flush.fill_(k)
        st = g.lookup_range(0, w.lookups, LOOKUP_SEED, search=search, timing=True)
        if k >= 2:
            s_ms.append(st.sample_ms); l_ms.append(st.lookup_ms); t_ms.append(st.device_ms)
        hashes.add(st.hash)
    print(f"{sys.argv[1]:8s} {search:3s} sort {statistics.median(s_ms):.3f} ms  lookup {statistics.median(l_ms):.3f} ms  "
          f"total {statistics.median(t_ms):.3f} ms  hash {sorted(hashes)}", flush=True)
