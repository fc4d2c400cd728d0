#!/usr/bin/env python
"""bench.py -- lookups/s of the XSBench-style macroscopic XS lookup on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload small] [--search U4] [--sort material_energy]

One step = one pass of the whole hot path (sampling,
(material, energy) ordering, search, interpolation, accumulation, verification) over
one batch of lookups on every rank, inputs (the grid) resident in HBM.  Weak scaling:
rank r owns lookups [r*L, (r+1)*L) of each batch (L = the workload's per-GPU count).
Rank 0 prints ONE JSON line.  Timing: W untimed warm-up steps, then K steps, each
bracketed by CUDA events on the launching stream with the 126 MB L2 flushed (a
256 MiB write) before it, outside the events; barrier + synchronize on both sides;
the max over ranks of the summed step times.  Grid creation is untimed (XSBench's
grid_init_do_not_profile [XSB]).

--impl reference times the CPU oracle (oracle/, plain C + OpenMP) on the box's host
cores on a bounded sample of the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from xs_workloads import GRID_SEED, LOOKUP_SEED, MEAN_NUCS, WORKLOADS, GRID_NAMES  # noqa: E402

METRIC = "lookups/sec (device-timed, max over ranks)"
UNIT = "lookups/s"
L2_FLUSH_BYTES = 256 << 20
BYTES_PER_PAIR = 96  # two 48 B point records per (lookup, nuclide)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--workload", default="small", choices=sorted(WORKLOADS))
    p.add_argument("--lookups", type=int, default=0, help="override lookups per GPU")
    p.add_argument("--search", default="S")
    p.add_argument("--sort", default="material_energy")
    p.add_argument("--energy-bins", type=int, default=0)
    p.add_argument("--no-flush", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--ab", default="M,U1,U2,U4,U8,B,W,H,S", help="search variants for the A/B sub-object ('' = off)")
    p.add_argument("--ab-steps", type=int, default=5)
    p.add_argument("--cpu-seconds", type=float, default=12.0, help="target wall time of the CPU sample")
    return p.parse_args()


def algorithmic_bytes_per_lookup(w) -> float:
    """the useful bytes of a random gather -- E[n_nuc] x 96 B (nuclide),
    + 4 B of IDX per pair (unionized), + 8*ceil(log2(W+1)) B of window probes (hash).
    Probes into L2-resident search arrays are excluded."""
    m = MEAN_NUCS[68 if w.n_nuclides == 68 else 355]
    if w.grid_type == 1:
        per_pair = BYTES_PER_PAIR
    elif w.grid_type == 0:
        per_pair = BYTES_PER_PAIR + 4
    else:
        W = w.n_gridpoints / 10000
        per_pair = BYTES_PER_PAIR + 8 * math.ceil(math.log2(W + 1))
    return m * per_pair


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_record(workload: str, search: str, sort: str):
    """The committed ncu --set full capture of k_lookup for this configuration
    (profiles/ncu_traffic.json: DRAM bytes and warp instructions per launch)."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            d = json.load(f)
        return d.get(f"{workload}/{search}/{sort}")
    except Exception:
        return None


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.p = None
        self.path = os.path.join("/tmp", f"xs_clocks_{os.getpid()}.csv")

    def __enter__(self):
        try:
            self.f = open(self.path, "w")
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
            time.sleep(0.3)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        if self.p:
            self.p.terminate()
            try:
                self.p.wait(timeout=5)
            except Exception:
                self.p.kill()
            self.f.close()

    def summary(self):
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        rows = []
        for line in open(self.path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 9:
                rows.append(parts)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = max(float(r[2]) for r in rows if r[2].replace(".", "").isdigit())
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if r[5 + k].lower() == "active"})
        loaded = [s for s in sm if s > 0.5 * mx] or sm
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(rows)}


def cpu_baseline(w, lookups_cap: int, seconds: float):
    """The oracle as it stands on this host's cores: a bounded sample of the workload."""
    import oracle
    t0 = time.time()
    P = oracle.Problem(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED, build_idx=False)
    setup_s = time.time() - t0
    threads = oracle.max_threads()
    n = 20_000
    t0 = time.perf_counter()
    P.run_range(LOOKUP_SEED, 0, n, macro=False)
    rate = n / max(time.perf_counter() - t0, 1e-6)
    n = int(min(lookups_cap, max(n, rate * seconds)))
    t0 = time.perf_counter()
    r = P.run_range(LOOKUP_SEED, 0, n, macro=False)
    dt = time.perf_counter() - t0
    # plus one single-thread run (a ~1/threads-sized sample, same rate basis)
    n1 = max(1000, n // max(threads, 1))
    t0 = time.perf_counter()
    P.run_range(LOOKUP_SEED, 0, n1, macro=False, threads=1)
    dt1 = time.perf_counter() - t0
    return {"value": n / dt, "unit": UNIT, "cores": threads, "kind": "oracle",
            "single_thread": {"value": n1 / dt1, "unit": UNIT, "sample": f"lookups [0, {n1})"},
            "sample": f"lookups [0, {n}) of {w.name} ({w.n_nuclides}x{w.n_gridpoints} "
                      f"{GRID_NAMES[w.grid_type]}), OpenMP static over lookups, {dt:.1f} s wall "
                      f"(grid build {setup_s:.1f} s untimed)",
            "_hash": r["hash"], "_n": n}


def run_reference(a, w):
    """--impl reference: the oracle as the reference arm (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    P = oracle.Problem(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED, build_idx=False)
    threads = oracle.max_threads()
    n = 20_000
    t0 = time.perf_counter()
    P.run_range(LOOKUP_SEED, 0, n, macro=False)
    rate = n / max(time.perf_counter() - t0, 1e-6)
    budget = 150.0 / max(a.steps + a.warmup, 1)  # whole run within a few minutes
    n = int(max(10_000, min(w.lookups, rate * budget)))
    times = []
    for k in range(a.warmup + a.steps):
        t0 = time.perf_counter()
        P.run_range(LOOKUP_SEED, 0, n, macro=False)
        if k >= a.warmup:
            times.append(time.perf_counter() - t0)
    total = sum(times)
    value = n * len(times) / total
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": a.gpus,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * total / len(times),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (XSBench LCG grid + lookups, seeds 42/1070)",
        "config": {"workload": w.name, "n_nuclides": w.n_nuclides, "n_gridpoints": w.n_gridpoints,
                   "grid": GRID_NAMES[w.grid_type], "lookups_per_step": n},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                         "sample": f"lookups [0, {n}) of {w.name} per step"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def run_ours(a, w):
    import torch
    import paper_conf_cgo_murtovigplls24_b200 as xs
    from paper_conf_cgo_murtovigplls24_b200 import driver

    R = driver.init()
    dev = torch.device("cuda", torch.cuda.current_device())
    L = a.lookups or w.lookups
    first, count = driver.weak_range(L, R.rank)
    g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
    assert driver.replicas_identical(g.checksum()), "grid replicas differ across ranks"
    stream = torch.cuda.current_stream()
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.int32, device=dev)
    opts = dict(search=a.search, sort=a.sort, energy_bins=a.energy_bins, timing=True)

    def step(**o):
        return g.lookup_range(first, count, LOOKUP_SEED, None, **{**opts, **o})

    def timed_steps(k_steps, **o):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(k_steps)]
        out = []
        for k in range(k_steps):
            if not a.no_flush:
                flush.fill_(k)
            evs[k][0].record(stream)
            out.append(step(**o))
            evs[k][1].record(stream)
        torch.cuda.synchronize()
        return [s_.elapsed_time(e_) for s_, e_ in evs], out

    ref_stats = None
    for _ in range(a.warmup):
        ref_stats = step()
    driver.barrier()
    torch.cuda.synchronize()
    with Clocks(torch.cuda.current_device()) as clk:
        step_ms, stats = timed_steps(a.steps)
    driver.barrier()
    total_ms = driver.max_over_ranks(sum(step_ms))
    lookup_ms = [s.lookup_ms for s in stats]
    hashes = {s.hash for s in stats}
    assert len(hashes) == 1 and (ref_stats is None or ref_stats.hash in hashes), "non-deterministic hash"
    h, nl, npairs, _ = driver.reduce_stats(stats[0].hash, stats[0].lookups, stats[0].pairs, 0.0)

    # ---- the paper's A/B on this workload: every search variant, same protocol, fewer steps
    ab = {}
    for v in [x for x in a.ab.split(",") if x]:
        for _ in range(2):
            step(search=v)
        ms, sts = timed_steps(a.ab_steps, search=v)
        ms_max = driver.max_over_ranks(sum(ms))
        ab[v] = {"value": R.world * count * a.ab_steps / (ms_max / 1e3),
                 "lookup_ms": statistics.mean(x.lookup_ms for x in sts), "hash_ok": all(x.hash == stats[0].hash for x in sts)}
    if a.ab:
        for _ in range(2):
            step(search="H", sort="history")
        ms, sts = timed_steps(a.ab_steps, search="H", sort="history")
        ms_max = driver.max_over_ranks(sum(ms))
        ab["H/history (XSBench history order, 34 lookups/particle)"] = {
            "value": R.world * count * a.ab_steps / (ms_max / 1e3),
            "lookup_ms": statistics.mean(x.lookup_ms for x in sts), "hash_ok": all(x.hash == stats[0].hash for x in sts)}
        for _ in range(2):
            step(coarse=True)
        ms, sts = timed_steps(a.ab_steps, coarse=True)
        ms_max = driver.max_over_ranks(sum(ms))
        ab[f"{a.search}/coarse (bucket order without the k_bucket_refine pass)"] = {
            "value": R.world * count * a.ab_steps / (ms_max / 1e3), "sort_ms": statistics.mean(x.sample_ms for x in sts),
            "lookup_ms": statistics.mean(x.lookup_ms for x in sts), "hash_ok": all(x.hash == stats[0].hash for x in sts)}
        for _ in range(2):
            step(search="M", sort="none")
        ms, sts = timed_steps(a.ab_steps, search="M", sort="none")
        ms_max = driver.max_over_ranks(sum(ms))
        ab["M/unsorted (XSBench order)"] = {"value": R.world * count * a.ab_steps / (ms_max / 1e3),
                                            "lookup_ms": statistics.mean(x.lookup_ms for x in sts),
                                            "hash_ok": all(x.hash == stats[0].hash for x in sts)}

    # ---- e2e: the public API with HOST output buffers (D2H of every macro XS in the region)
    e2e = None
    if not a.no_e2e:
        host = torch.empty((count, 5), dtype=torch.float64).pin_memory()
        for _ in range(2):
            g.lookup_range(first, count, LOOKUP_SEED, host, search=a.search, sort=a.sort)
        driver.barrier()
        torch.cuda.synchronize()
        t = []
        for k in range(max(3, a.steps // 4)):
            if not a.no_flush:
                flush.fill_(k)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            g.lookup_range(first, count, LOOKUP_SEED, host, search=a.search, sort=a.sort)
            t.append(time.perf_counter() - t0)
        e2e_s = driver.max_over_ranks(sum(t))
        # the hash-only public call (XSBench's own result: the verification hash)
        th = []
        for k in range(max(3, a.steps // 4)):
            if not a.no_flush:
                flush.fill_(k)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            hh = xs.xs_lookup_batch(g.handle, count, LOOKUP_SEED, None) if R.world == 1 else \
                g.lookup_range(first, count, LOOKUP_SEED, None, search=a.search, sort=a.sort).hash
            th.append(time.perf_counter() - t0)
        e2e_h = driver.max_over_ranks(sum(th))
        e2e = {"value": R.world * count * len(t) / e2e_s, "unit": UNIT, "h2d_bytes_per_step": 0,
               "d2h_bytes_per_step": count * 5 * 8 + 16,
               "note": "xs_lookup_range writing every macroscopic XS into pinned HOST memory (D2H "
                       "overlapped with compute in 4M-lookup chunks), host wall clock; inputs are the "
                       "(seed, range) scalars -- lookups are drawn on device by the method's "
                       "counter-based LCG (DESIGN.md §8)",
               "hash_only": {"value": R.world * count * len(th) / e2e_h, "d2h_bytes_per_step": 16,
                             "call": "xs_lookup_batch (default options), host wall clock"}}

    if R.rank != 0:
        driver.finalize()
        return
    value = R.world * count * a.steps / (total_ms / 1e3)
    peak, peak_src = measured_peaks()
    bpl = algorithmic_bytes_per_lookup(w)
    mean_lookup_ms = statistics.mean(lookup_ms)
    achieved = bpl * count / (mean_lookup_ms / 1e3) / 1e9
    rec = ncu_record(w.name, a.search, a.sort)
    traffic = rec["dram_bytes_per_launch"] if rec else None
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": R.world, "steps": a.steps,
        "warmup": a.warmup, "ms_per_step": total_ms / a.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (XSBench LCG grid + lookups, seeds 42/1070)",
        "config": {"workload": w.name, "n_nuclides": w.n_nuclides, "n_gridpoints": w.n_gridpoints,
                   "grid": GRID_NAMES[w.grid_type], "lookups_per_gpu": count, "search": a.search,
                   "sort": a.sort, "l2_flush": not a.no_flush, "parallelism": f"dp{R.world} (index ranges)"},
        "step_ms": {"median": statistics.median(step_ms), "rsd_pct": 100 * statistics.pstdev(step_ms) /
                    statistics.mean(step_ms), "min": min(step_ms), "max": max(step_ms)},
        "phase_ms": {"sort": statistics.mean(s.sample_ms for s in stats), "lookup": mean_lookup_ms},
        "roofline": {"bound": "hbm", "kernel": "k_lookup_staged" if a.search == "S" and a.sort == "material_energy" else "k_lookup", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic,
                     "bytes_per_lookup_alg": bpl, "peak_source": peak_src,
                     "note": "achieved = SURVEY.md §8d random-gather bytes (E[nuclides] x 96 B per lookup) / "
                             "k_lookup event time.  The (material, energy) sort makes warps share grid "
                             "points, so DRAM traffic (`traffic`, ncu) is far below the algorithmic bytes "
                             "and frac can exceed 1; the kernel is latency-bound (DESIGN.md §7)"},
        "ab": ab,
        "verification": {"hash": h, "lookups": nl, "pairs": npairs},
        "gpu_launches": int(sum(s.launches for s in stats)),
        "e2e": e2e,
    }
    line["clocks"] = clk.summary()
    if rec and rec.get("warp_inst_per_launch") and line["clocks"].get("sm_mhz"):
        sms = torch.cuda.get_device_properties(dev).multi_processor_count
        ips = rec["warp_inst_per_launch"] / (mean_lookup_ms / 1e3)
        peak_ips = sms * 4 * line["clocks"]["sm_mhz"] * 1e6  # 4 schedulers x 1 warp-instruction/clk
        line["roofline"]["issue"] = {"achieved_warp_inst_per_s": ips, "peak": peak_ips, "frac": ips / peak_ips,
                                     "source": "ncu smsp__inst_executed.sum per launch (profiles/) / live event time"}
        if rec.get("lsu_wavefronts_per_launch"):
            # the unit that binds the staged kernel: one L1/shared-memory
            # data-pipe wavefront per SM per clock
            wps = rec["lsu_wavefronts_per_launch"] / (mean_lookup_ms / 1e3)
            peak_wps = sms * line["clocks"]["sm_mhz"] * 1e6
            line["roofline"]["l1_data_pipe"] = {
                "achieved_wavefronts_per_s": wps, "peak": peak_wps, "frac": wps / peak_wps,
                "ncu_pct_of_peak": rec.get("lsu_wavefronts_pct_of_peak"),
                "source": "ncu shared + global + local LSU wavefronts per launch (profiles/) / live event time"}
    try:  # SURVEY.md §8d's measured random-gather roofline (tools/l2_gather.cu on this pool's B200)
        with open(os.path.join(ROOT, "profiles", "l2_gather.json")) as f:
            lg = json.load(f)
        key = {"small": "small_points_37MB", "large": "large_points_193MB", "large-U": "large_points_193MB",
               "XL": "xl_points_4.07GB"}.get(w.name)
        if key and lg["gathers"].get(key):
            gp = lg["gathers"][key]["GBps_useful"]
            line["roofline"]["random_gather"] = {
                "peak": gp, "unit": "GB/s", "frac": achieved / gp, "buffer": key,
                "source": "profiles/l2_gather.json: random 96 B record gathers over a buffer the size of this "
                          "workload's point records (L2-resident for small); frac > 1 = the sort turns the "
                          "random gather into shared accesses"}
    except Exception:
        pass
    if not a.no_cpu_baseline and R.world == 1:
        cb = cpu_baseline(w, count, a.cpu_seconds)
        # parity of the bench's own configuration on the oracle's sample range
        gs = g.lookup_range(0, cb["_n"], LOOKUP_SEED, None, search=a.search, sort=a.sort)
        line["verification"]["oracle_sample_hash_match"] = bool(gs.hash == cb["_hash"])
        line["cpu_baseline"] = {k: v for k, v in cb.items() if not k.startswith("_")}
    print(json.dumps(line), flush=True)
    g.close()
    driver.finalize()


def main():
    a = parse()
    w = WORKLOADS[a.workload]
    if a.impl == "reference":
        run_reference(a, w)
    else:
        run_ours(a, w)


if __name__ == "__main__":
    main()
