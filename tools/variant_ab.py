"""A/B of experimental libxs builds: for each XS_LIB_VARIANT (libxs_<v>.so; '' = libxs.so)
and workload, the lookup-kernel and sort times of the default path (median of 7 after 3
warm-ups, CUDA events inside the library) and the hash.  Development aid.
usage: python tools/variant_ab.py VARIANTS WORKLOADS [SEARCH] [LOOKUPS]   e.g.  "',lr0'" small,XL"""
import json, os, statistics, subprocess, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(workload, search, n=0):
    sys.path.insert(0, ROOT)
    import paper_conf_cgo_murtovigplls24_b200 as xs
    from xs_workloads import WORKLOADS, GRID_SEED, LOOKUP_SEED
    w = WORKLOADS[workload]
    n = int(n) or w.lookups
    g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
    for _ in range(3):
        g.lookup_range(0, n, LOOKUP_SEED, search=search)
    st = [g.lookup_range(0, n, LOOKUP_SEED, search=search, timing=True) for _ in range(7)]
    print(json.dumps({"variant": os.environ.get("XS_LIB_VARIANT", ""), "workload": workload, "lookups": n, "search": search,
                      "lookup_ms": statistics.median(s.lookup_ms for s in st),
                      "sort_ms": statistics.median(s.sample_ms for s in st),
                      "device_ms": statistics.median(s.device_ms for s in st), "hash": st[0].hash}), flush=True)


def main():
    if sys.argv[1] == "--child":
        return child(sys.argv[2], sys.argv[3], sys.argv[4] if len(sys.argv) > 4 else 0)
    variants = sys.argv[1].split(",")
    workloads = sys.argv[2].split(",")
    search = sys.argv[3] if len(sys.argv) > 3 else "S"
    n = sys.argv[4] if len(sys.argv) > 4 else "0"
    for w in workloads:
        for v in variants:
            env = dict(os.environ)
            if v:
                env["XS_LIB_VARIANT"] = v
            else:
                env.pop("XS_LIB_VARIANT", None)
            subprocess.run([sys.executable, __file__, "--child", w, search, n], env=env)


if __name__ == "__main__":
    main()
