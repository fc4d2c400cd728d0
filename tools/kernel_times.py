"""Per-kernel device timeline of one lookup step (CUPTI through torch.profiler): kernel
durations and the idle gaps between them.  Development aid.
usage: python tools/kernel_times.py [WORKLOAD] [SEARCH] [SORT] [LOOKUPS]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from torch.profiler import profile, ProfilerActivity
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED

w = WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "small"]
search = sys.argv[2] if len(sys.argv) > 2 else "S"
sort = sys.argv[3] if len(sys.argv) > 3 else "material_energy"
n = int(sys.argv[4]) if len(sys.argv) > 4 else w.lookups
g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
for _ in range(3):
    g.lookup_range(0, n, LOOKUP_SEED, search=search, sort=sort)
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for _ in range(2):
        g.lookup_range(0, n, LOOKUP_SEED, search=search, sort=sort)
    torch.cuda.synchronize()
evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
evs.sort(key=lambda e: e.time_range.start)
prev = None
for e in evs:
    gap = (e.time_range.start - prev) if prev is not None else 0
    print(f"{e.time_range.start:14.1f} +{gap:7.1f} us  {e.time_range.elapsed_us():9.1f} us  {e.name[:90]}")
    prev = e.time_range.end
