"""Energy-bin / block-size sweep for one search variant (development aid)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED
cfgs = sys.argv[1].split(","); search = sys.argv[2]
bins = [int(x) for x in sys.argv[3].split(",")]; blocks = [int(x) for x in sys.argv[4].split(",")] if len(sys.argv) > 4 else [256]
for c in cfgs:
    w = WORKLOADS[c]
    g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
    for nb in bins:
        for bl in blocks:
            for _ in range(2):
                g.lookup_range(0, w.lookups, LOOKUP_SEED, search=search, energy_bins=nb, block=bl)
            r = sorted((lambda st: (st.device_ms, st.sample_ms, st.lookup_ms))(
                g.lookup_range(0, w.lookups, LOOKUP_SEED, search=search, energy_bins=nb, block=bl, timing=True)) for _ in range(5))[2]
            print(json.dumps({"cfg": c, "search": search, "bins": nb, "block": bl, "total_ms": round(r[0], 3),
                              "sort_ms": round(r[1], 3), "lookup_ms": round(r[2], 3), "Glookups_s": round(w.lookups / r[0] / 1e6, 3)}), flush=True)
    g.close()
