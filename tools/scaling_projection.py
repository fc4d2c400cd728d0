"""Per-rank work of the N-GPU configurations, timed on ONE GPU (no 8-GPU node this round).

For N in {1, 2, 4, 8}, every rank's exact lookup range (strong scaling for
large-U / large / small, weak at 125M per rank for XL) is run through the bench protocol
(L2 flushed, CUDA events, median of K steps) on this GPU, one rank after another.  The
projected job throughput is (lookups of all ranks) / (max over ranks of the rank's step
time): what `bench.py --gpus N` would report if the ranks did not interfere and the one
24-byte all-reduce per step (measured separately on NVLink by bench.py) cost nothing.
A projection, not a measurement of N GPUs.

usage: python tools/scaling_projection.py [WORKLOADS] [STEPS] [index|keys] > out.jsonl"""
import json, os, statistics, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import paper_conf_cgo_murtovigplls24_b200 as xs
    from paper_conf_cgo_murtovigplls24_b200 import driver
    from xs_workloads import GRID_SEED, LOOKUP_SEED, WORKLOADS
    names = (sys.argv[1] if len(sys.argv) > 1 else "large-U,XL").split(",")
    steps = int(sys.argv[2]) if len(sys.argv) > 2 else 7
    # split of the strong configurations: "index" = [floor(rT/N), floor((r+1)T/N)) (SURVEY.md
    # §8e), "keys" = key-range shards of the whole range (xs_opts.shard_*)
    split = sys.argv[3] if len(sys.argv) > 3 else "index"
    flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream()
    for name in names:
        w = WORKLOADS[name]
        g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
        base = None
        for N in (1, 2, 4, 8):
            ranks = []
            for r in range(N):
                keys = w.scaling == "strong" and split == "keys"
                if keys:
                    first, count, opt = 0, w.lookups, dict(shard=(r, N))
                else:
                    first, count = (driver.shard(w.lookups, r, N) if w.scaling == "strong"
                                    else driver.weak_range(w.lookups, r))
                    opt = {}
                for _ in range(3):
                    g.lookup_range(first, count, LOOKUP_SEED, **opt)
                ms = []
                for k in range(steps):
                    flush.fill_(k)
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                    st = g.lookup_range(first, count, LOOKUP_SEED, **opt)
                    b.record(stream)
                    torch.cuda.synchronize()
                    ms.append(a.elapsed_time(b))
                ranks.append({"rank": r, "first": first, "count": int(st.lookups), "ms": statistics.median(ms),
                              "hash": st.hash, "pairs": st.pairs, "split": "keys" if keys else "index"})
            total = sum(x["count"] for x in ranks)
            tmax = max(x["ms"] for x in ranks)
            val = total / (tmax / 1e3)
            base = base or val
            print(json.dumps({"workload": name, "scaling": w.scaling, "n_gpus": N, "lookups_total": total,
                              "max_rank_ms": tmax, "projected_lookups_per_s": val,
                              "projected_efficiency": val / (base * N), "ranks": ranks}), flush=True)
        g.close()


if __name__ == "__main__":
    main()
