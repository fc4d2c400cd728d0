"""Short target for ncu captures: build one grid, run the hot path a few times.
usage: python tools/ncu_target.py WORKLOAD SEARCH SORT [REPS] [LOOKUPS]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED
w = WORKLOADS[sys.argv[1]]
search, sort = sys.argv[2], sys.argv[3]
split = os.environ.get("XS_SPLIT", "0") == "1"
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
n = int(sys.argv[5]) if len(sys.argv) > 5 else w.lookups
g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
for _ in range(reps):
    st = g.lookup_range(0, n, LOOKUP_SEED, search=search, sort=sort, split=split)
print("hash", st.hash, "device_ms", st.device_ms)
