"""A/B of the k_bucket_refine pass (XS_FLAG_COARSE off/on) on one workload: sort and lookup
kernel event times (median of N steps, L2 flushed before each), hash equality.
usage: python tools/refine_ab.py WORKLOAD [SEARCH] [STEPS]"""
import os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED

w = WORKLOADS[sys.argv[1]]
search = sys.argv[2] if len(sys.argv) > 2 else "S"
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 10
g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
flush = torch.empty(256 << 18, dtype=torch.int32, device="cuda")
res = {}
for coarse in (True, False, True, False):
    s_ms, l_ms, t_ms, hashes = [], [], [], set()
    for k in range(steps + 2):
        flush.fill_(k)
        st = g.lookup_range(0, w.lookups, LOOKUP_SEED, search=search, timing=True, coarse=coarse)
        if k >= 2:
            s_ms.append(st.sample_ms); l_ms.append(st.lookup_ms); t_ms.append(st.device_ms)
        hashes.add(st.hash)
    key = "coarse" if coarse else "refined"
    res.setdefault(key, []).append((statistics.median(s_ms), statistics.median(l_ms), statistics.median(t_ms), hashes))
for key, runs in res.items():
    for s, l, t, h in runs:
        print(f"{sys.argv[1]:8s} {search} {key:8s} sort {s:.3f} ms  lookup {l:.3f} ms  total {t:.3f} ms  hash {sorted(h)}")
