"""Quick variant/size timing probe (development aid; not the bench contract)."""
import sys, os, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_murtovigplls24_b200 as xs
from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED

def main():
    cfgs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["small", "large"]
    searches = sys.argv[2].split(",") if len(sys.argv) > 2 else ["M", "U1", "U2", "U4", "U8", "B", "M2"]
    sorts = sys.argv[3].split(",") if len(sys.argv) > 3 else ["none", "material", "material_energy"]
    fused_opts = [bool(int(x)) for x in sys.argv[4].split(",")] if len(sys.argv) > 4 else [False]
    for c in cfgs:
        w = WORKLOADS[c]
        t0 = time.time()
        g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
        print(f"{c}: grid build {time.time()-t0:.2f}s, {g.info.device_bytes/1e6:.1f} MB", flush=True)
        n = w.lookups
        for srt in sorts:
          for fu in (fused_opts if srt != "none" else [True]):
            for s in searches:
                for _ in range(2):
                    g.lookup_range(0, n, LOOKUP_SEED, search=s, sort=srt, split=not fu)
                ms = []
                for _ in range(5):
                    st = g.lookup_range(0, n, LOOKUP_SEED, search=s, sort=srt, timing=True, split=not fu)
                    ms.append((st.device_ms, st.sample_ms, st.lookup_ms, st.search_ms))
                ms.sort()
                d, a, b, c2 = ms[len(ms)//2]
                print(json.dumps({"cfg": c, "sort": srt, "fused": fu, "search": s, "total_ms": round(d,3), "sort_ms": round(a,3),
                                  "lookup_ms": round(b,3), "search_ms": round(c2, 3), "Mlookups_s": round(n/d/1e3,1), "hash": st.hash}), flush=True)
        g.close()

if __name__ == "__main__":
    main()
