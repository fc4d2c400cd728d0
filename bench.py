#!/usr/bin/env python
"""bench.py -- lookups/s of the XSBench-style macroscopic XS lookup on 1..8 B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload large-U] [--scaling strong|strong-index|weak] [--search S]
                    [--workloads small,large,XL]

One step = one pass of the whole hot path (sampling,
(material, energy) ordering, search, interpolation, accumulation, verification) over one
batch of lookups on every rank, the grid resident in HBM.  With --gpus N > 1 and no
torchrun environment, bench.py re-launches itself under torch.distributed.run with one
process per GPU; XS_DIST_BACKEND=gloo runs the ranks over gloo instead of
NCCL (ranks share the visible GPUs round-robin, so a 1-GPU box can run 2 ranks).

Scaling: strong (the default except XL) splits the workload's fixed total T into key-range
shards -- every rank draws all T lookups and orders / looks up its cost-weighted share of the
(material, energy) buckets (xs_opts.shard_*); strong-index into rank ranges
[floor(rT/N), floor((r+1)T/N)); weak gives every rank its own block of the
workload's per-rank count (XL: 125M per rank, so N = 8 is exactly the 1B-lookup configuration
of BASELINE.json configs[4]).  Counter-based sampling makes the results independent of the
split; the job's hash is checked against the CPU oracle's golden hashes
(tests/golden/hashes.json, written by tools/oracle_golden.py from oracle/ only): every rank's
index range against its eighths, or the ranks' sum against the total for key-range shards.

Timing: W untimed warm-up steps, then K steps, each bracketed by CUDA events on the
launching stream with the L2 flushed (a 256 MiB write) before it, outside the events;
barrier + synchronize on both sides; value = lookups of all ranks / the max over ranks of
the summed step times.  Grid creation is untimed (XSBench's grid_init_do_not_profile).

--impl reference times the CPU oracle (oracle/, plain C + OpenMP) on the box's host cores
on a bounded sample of the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import hashlib
import json
import math
import os
import socket
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
BYTES_PER_PAIR = 96      # two 48 B point records per (lookup, nuclide)
POINT_RECORD_BYTES = 48  # {E, 5 channels} fp64 per grid point
STREAM_BYTES = 12        # sorted slot (u32) + energy (f64) per lookup, read by the lookup kernel
# FP64 flops per (lookup, nuclide) pair that any bit-exact evaluation of reading R8 must
# execute, with d = E_hi - E_lo, y = RN(1/d) and dX_c precomputed:
# a = E_hi - q (1), Markstein's quotient q0 = a y, r = fma(-d, q0, a), f = fma(r, y, q0)
# (1 + 2 + 2), micro_c = fma(-f, dX_c, X_c) (5 x 2), acc_c = fma(micro_c, conc, acc_c) (5 x 2)
FLOPS_PER_PAIR = 26
FP64_LANES_PER_SM = 64   # B200: 64 FP64 FMA lanes per SM per clock
GOLDEN = os.path.join(ROOT, "tests", "golden", "hashes.json")


def parse(argv=None):
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--workload", default="large-U", choices=sorted(WORKLOADS))
    p.add_argument("--scaling", default="", choices=["", "strong", "weak", "strong-index"],
                   help="default: the workload's (XL weak at 125M per rank, the rest strong). strong: "
                        "key-range shards (every rank draws the whole range and looks up its share of the "
                        "(material, energy) buckets, DESIGN.md §9); strong-index: index ranges "
                        "[floor(rT/N), floor((r+1)T/N)) (SURVEY.md §8e)")
    p.add_argument("--lookups", type=int, default=0, help="override: job total (strong) or per rank (weak)")
    p.add_argument("--search", default="S")
    p.add_argument("--sort", default="material_energy")
    p.add_argument("--energy-bins", type=int, default=0)
    p.add_argument("--no-flush", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--ab", default="M,U1,U2,U4,U8,B,W,H,S", help="search variants for the A/B sub-object ('' = off)")
    p.add_argument("--ab-steps", type=int, default=5)
    p.add_argument("--workloads", default="small,large,XL",
                   help="other configurations measured into the `workloads` sub-object ('' = off)")
    p.add_argument("--cpu-seconds", type=float, default=12.0, help="target wall time of the CPU sample")
    return p.parse_args(argv)


# ------------------------------------------------------------------ sizes and rooflines
def scaling_of(a, w) -> str:
    """strong (key-range shards), strong-index or weak"""
    return a.scaling or w.scaling


def scaling_kind(scaling: str) -> str:
    """the contract's `scaling` field: strong or weak"""
    return "weak" if scaling == "weak" else "strong"


def rank_range(w, scaling: str, total_override: int, rank: int, world: int):
    """(first, count) of this rank's index range: strong splits the job's total,
    weak gives every rank its own per-rank count"""
    from paper_conf_cgo_murtovigplls24_b200 import driver
    n = total_override or w.lookups
    return driver.shard(n, rank, world) if scaling_kind(scaling) == "strong" else driver.weak_range(n, rank)


def job_lookups(w, scaling: str, total_override: int, world: int) -> int:
    n = total_override or w.lookups
    return n if scaling_kind(scaling) == "strong" else n * world


def algorithmic_bytes_per_lookup(w) -> float:
    """the useful bytes of a RANDOM gather -- E[n_nuc] x 96 B (nuclide),
    + 4 B of IDX per pair (unionized), + 8*ceil(log2(W+1)) B of window probes (hash).
    Valid for XSBench's unsorted order only."""
    m = MEAN_NUCS[68 if w.n_nuclides == 68 else 355]
    if w.grid_type == 1:
        per_pair = BYTES_PER_PAIR
    elif w.grid_type == 0:
        per_pair = BYTES_PER_PAIR + 4
    else:
        W = w.n_gridpoints / 10000
        per_pair = BYTES_PER_PAIR + 8 * math.ceil(math.log2(W + 1))
    return m * per_pair


def hbm_min_bytes(w, lookups: int) -> float:
    """A lower bound on the DRAM bytes one lookup-kernel launch over `lookups` sorted lookups
    must move: every point record once (at these sizes every interval of
    every nuclide is visited: >= 2.4M lookups per fuel nuclide per launch) plus the sorted
    (slot, energy) stream.  Search structures (E, bins, U, IDX, H) are left out, so the
    fraction is an underestimate."""
    return w.n_points * POINT_RECORD_BYTES + STREAM_BYTES * lookups


def measured_hbm_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def fp64_peak_tflops(sms: int):
    """FP64 peak: the guide's unit count (64 FMA lanes/SM/clk) x 2 flops x SMs x max SM clock;
    profiles/fp64_peak.json (tools/fp64_peak.cu, a DFMA microbenchmark on this pool's B200)
    when present."""
    try:
        with open(os.path.join(ROOT, "profiles", "fp64_peak.json")) as f:
            d = json.load(f)
        return float(d["tflops"]), "measured (profiles/fp64_peak.json: DFMA microbenchmark)"
    except Exception:
        mhz = 1965.0
        try:
            with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
                mhz = float(json.load(f).get("sm_max_mhz", mhz))
        except Exception:
            pass
        return sms * FP64_LANES_PER_SM * 2 * mhz * 1e6 / 1e12, \
            f"derived: {sms} SMs x {FP64_LANES_PER_SM} FP64 lanes x 2 flops x {mhz:.0f} MHz"


def libxs_sha() -> str:
    """The build identity of libxs.so (build.py source_digest: sources + flags)."""
    try:
        import importlib.util
        spec = importlib.util.spec_from_file_location(
            "_xs_build", os.path.join(ROOT, "paper_conf_cgo_murtovigplls24_b200", "build.py"))
        b = importlib.util.module_from_spec(spec)
        spec.loader.exec_module(b)
        return b.source_digest()
    except Exception:
        return ""


def ncu_record(workload: str, search: str, sort: str):
    """The committed ncu --set full capture of this configuration's lookup kernel
    (profiles/ncu_traffic.json), used only if it was taken on THIS libxs.so build."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            d = json.load(f)
        rec = d.get(f"{workload}/{search}/{sort}")
        if rec and rec.get("libxs_sha") == libxs_sha():
            return rec
    except Exception:
        pass
    return None


def roofline(w, search, sort, lookups, pairs, kernel_ms, sms, clocks=None, with_ncu=True):
    """The lookup kernel against what the work needs: FP64 flops (alu) and
    the HBM minimum; `bound` is whichever fraction is higher.  SURVEY.md §8d's random-gather
    bytes are kept as `random_gather_equiv` (valid as a roofline for unsorted order only)."""
    sec = kernel_ms / 1e3
    hbm_peak, hbm_src = measured_hbm_peak()
    fp_peak, fp_src = fp64_peak_tflops(sms)
    flops = FLOPS_PER_PAIR * pairs
    alu = {"achieved": flops / sec / 1e12, "peak": fp_peak, "unit": "TFLOP/s",
           "frac": flops / sec / 1e12 / fp_peak, "flops_per_pair": FLOPS_PER_PAIR, "pairs": pairs,
           "peak_source": fp_src}
    hb = hbm_min_bytes(w, lookups)
    hbm = {"achieved": hb / sec / 1e9, "peak": hbm_peak, "unit": "GB/s", "frac": hb / sec / 1e9 / hbm_peak,
           "bytes_per_launch": hb, "peak_source": hbm_src}
    rg_b = algorithmic_bytes_per_lookup(w) * lookups
    rg = {"achieved": rg_b / sec / 1e9, "unit": "GB/s", "bytes_per_lookup": algorithmic_bytes_per_lookup(w),
          "frac_of_hbm": rg_b / sec / 1e9 / hbm_peak}
    try:
        with open(os.path.join(ROOT, "profiles", "l2_gather.json")) as f:
            lg = json.load(f)
        key = {"small": "small_points_37MB", "large": "large_points_193MB", "large-U": "large_points_193MB",
               "XL": "xl_points_4.07GB"}.get(w.name)
        if key and lg["gathers"].get(key):
            gp = lg["gathers"][key]["GBps_useful"]
            rg.update(measured_gather_peak=gp, frac_of_measured_gather=rg_b / sec / 1e9 / gp, buffer=key)
    except Exception:
        pass
    rg["note"] = ("SURVEY.md §8d random-gather bytes; in (material, energy) order warps share their grid "
                  "points, so this exceeds any bandwidth and is not a roofline there")
    kernel = "k_lookup_staged" if search == "S" and sort in ("material_energy", "material") else "k_lookup"
    top = alu if alu["frac"] >= hbm["frac"] else hbm
    line = {"bound": "alu" if top is alu else "hbm", "kernel": kernel, "achieved": top["achieved"],
            "peak": top["peak"], "unit": top["unit"], "frac": top["frac"], "traffic": None,
            "alu_fp64": alu, "hbm_min": hbm, "random_gather_equiv": rg}
    rec = ncu_record(w.name, search, sort) if with_ncu else None
    if rec:
        line["traffic"] = rec["dram_bytes_per_launch"] * lookups / rec.get("lookups", lookups)
        line["ncu"] = {k: rec.get(k) for k in ("libxs_sha", "report", "round", "dram_bytes_per_launch",
                                               "l2_hit_pct", "l1_hit_pct", "sectors_per_request",
                                               "lsu_wavefronts_pct_of_peak", "fp64_pipe_pct", "issue_active_pct",
                                               "branch_uniform_pct")}
        line["hbm_min"]["refetch"] = rec["dram_bytes_per_launch"] / hb
    else:
        line["ncu"] = {"note": "no ncu capture of this libxs.so build for this configuration"}
    return line


def golden_expect(name: str, first: int, count: int):
    """The oracle's hash / pairs over [first, first + count) when the range is a union of the
    golden eighths (tests/golden/hashes.json), else None."""
    try:
        with open(GOLDEN) as f:
            g = json.load(f)[name]
    except Exception:
        return None
    b = g["bounds"]
    if first not in b or (first + count) not in b:
        return None
    i, j = b.index(first), b.index(first + count)
    return sum(g["hash"][i:j]), sum(g["pairs"][i:j])


# ------------------------------------------------------------------ clocks
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


# ------------------------------------------------------------------ the reference arm
def config_of(a, w, world: int) -> dict:
    """The workload `config` both arms print (identical, so the driver can pair them)."""
    sc = scaling_of(a, w)
    split = ("key-range shards: every rank draws all lookups, orders and looks up its 1/N of the "
             "(material, energy) buckets by expected cost" if sc == "strong" and world > 1 else "lookup index ranges")
    return {"workload": w.name, "n_nuclides": w.n_nuclides, "n_gridpoints": w.n_gridpoints,
            "grid": GRID_NAMES[w.grid_type], "lookups_total": job_lookups(w, sc, a.lookups, world),
            "scaling": scaling_kind(sc), "l2_flush": not a.no_flush, "parallelism": f"dp{world} ({split})"}


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
    """--impl reference: the oracle as the reference arm (rank 0 only; other ranks exit 0)."""
    if int(os.environ.get("RANK", "0")) != 0:
        return
    import oracle
    world = int(os.environ.get("WORLD_SIZE", str(a.gpus)))
    P = oracle.Problem(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED, build_idx=False)
    threads = oracle.max_threads()
    n = 20_000
    t0 = time.perf_counter()
    P.run_range(LOOKUP_SEED, 0, n, macro=False)
    rate = n / max(time.perf_counter() - t0, 1e-6)
    budget = 150.0 / max(a.steps + a.warmup, 1)  # whole run within a few minutes
    total = job_lookups(w, scaling_of(a, w), a.lookups, world)
    n = int(max(10_000, min(total, rate * budget)))
    times = []
    for k in range(a.warmup + a.steps):
        t0 = time.perf_counter()
        P.run_range(LOOKUP_SEED, 0, n, macro=False)
        if k >= a.warmup:
            times.append(time.perf_counter() - t0)
    tsum = sum(times)
    value = n * len(times) / tsum
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * tsum / len(times),
        "higher_is_better": True, "scaling": scaling_kind(scaling_of(a, w)), "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (XSBench LCG grid + lookups, seeds 42/1070)",
        "config": config_of(a, w, world),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                         "sample": f"lookups [0, {n}) of {w.name} per step (the job's {total} lookups "
                                   f"bounded to ~{budget:.0f} s of CPU work per step), host cores only"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm
class Runner:
    """One grid on this rank's GPU and the timed-step protocol."""

    def __init__(self, a, w, R, scaling):
        import torch
        import paper_conf_cgo_murtovigplls24_b200 as xs
        from paper_conf_cgo_murtovigplls24_b200 import driver
        self.torch, self.xs, self.driver, self.a, self.w, self.R = torch, xs, driver, a, w, R
        self.scaling = scaling
        # index range of this rank (weak, strong-index, and the passes key shards do not serve)
        self.first, self.count = rank_range(w, scaling, a.lookups, R.rank, R.world)
        self.total = int(driver.sum_over_ranks(self.count))
        # strong at N > 1: key-range shard (rank, N) of the whole range [0, total)
        self.keys = scaling == "strong" and R.world > 1
        self.g = xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
        assert driver.replicas_identical(self.g.checksum()), "grid replicas differ across ranks"
        self.stream = torch.cuda.current_stream()
        self.flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.int32, device=self.g.device)
        self.opts = dict(search=a.search, sort=a.sort, energy_bins=a.energy_bins, timing=True)

    def uses_keys(self, o) -> bool:
        """key-range shards serve the refined order with the staged kernel (xs.h)"""
        oo = {**self.opts, **o}
        return self.keys and oo["search"] == "S" and oo["sort"] == "material_energy" and not oo.get("coarse")

    def step(self, **o):
        if self.uses_keys(o):
            return self.g.lookup_range(0, self.total, LOOKUP_SEED, None,
                                       **{**self.opts, **o, "shard": (self.R.rank, self.R.world)})
        return self.g.lookup_range(self.first, self.count, LOOKUP_SEED, None, **{**self.opts, **o})

    def timed(self, k_steps, warm, **o):
        torch = self.torch
        for _ in range(warm):
            self.step(**o)
        self.driver.barrier()
        torch.cuda.synchronize()
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(k_steps)]
        out = []
        for k in range(k_steps):
            if not self.a.no_flush:
                self.flush.fill_(k)
            evs[k][0].record(self.stream)
            out.append(self.step(**o))
            evs[k][1].record(self.stream)
        torch.cuda.synchronize()
        self.driver.barrier()
        ms = [s_.elapsed_time(e_) for s_, e_ in evs]
        return ms, out, self.driver.max_over_ranks(sum(ms))

    def golden(self, stats, keys=False):
        """Index ranges: every rank's hash and pairs against the oracle's golden eighths; key
        shards: the sums over ranks against the golden total of the whole range.  True / False
        / None (None: the split does not fall on the golden boundaries)."""
        if keys:
            h, nl, pr, _ = self.driver.reduce_stats(stats.hash, stats.lookups, stats.pairs, 0.0)
            exp = golden_expect(self.w.name, 0, self.total)
            return None if exp is None else bool(h == exp[0] and pr == exp[1] and nl == self.total)
        exp = golden_expect(self.w.name, self.first, self.count)
        ok = -1 if exp is None else int(stats.hash == exp[0] and stats.pairs == exp[1])
        lo = self.driver.min_over_ranks(ok)
        return None if lo < 0 else bool(lo)

    def close(self):
        self.g.close()


def summarize(run: Runner, ms_max, stats, steps, sms, clocks=None, **o):
    s0 = stats[0]
    h, nl, npairs, _ = run.driver.reduce_stats(s0.hash, s0.lookups, s0.pairs, 0.0)
    lookup_ms = statistics.mean(x.lookup_ms for x in stats)
    search = o.get("search", run.a.search)
    sort = o.get("sort", run.a.sort)
    keys = run.uses_keys(o)
    return {"value": run.total * steps / (ms_max / 1e3), "ms_per_step": ms_max / steps,
            "lookups_per_gpu": int(s0.lookups), "sort_ms": statistics.mean(x.sample_ms for x in stats),
            "lookup_ms": lookup_ms, "hash": h, "pairs": npairs, "lookups": nl,
            "split": "key-range shards" if keys else "index ranges",
            "hash_consistent": all(x.hash == s0.hash for x in stats),
            "golden_match": run.golden(s0, keys),
            "roofline": roofline(run.w, search, sort, int(s0.lookups), s0.pairs, lookup_ms, sms, clocks)}


def run_ours(a, w):
    import torch
    from paper_conf_cgo_murtovigplls24_b200 import driver

    R = driver.init(backend=os.environ.get("XS_DIST_BACKEND") or None)
    if R.world != a.gpus:
        raise SystemExit(f"bench.py: --gpus {a.gpus} but WORLD_SIZE={R.world}")
    dev = torch.device("cuda", torch.cuda.current_device())
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    scaling = scaling_of(a, w)
    run = Runner(a, w, R, scaling)

    with Clocks(torch.cuda.current_device()) as clk:
        step_ms, stats, total_ms = run.timed(a.steps, a.warmup)
    clocks = clk.summary()
    assert len({s.hash for s in stats}) == 1, "non-deterministic hash"
    main = summarize(run, total_ms, stats, a.steps, sms)

    # ---- the north-star quantity: the unmerged (u&u, u=2) Listing-1 search, same config and N
    north = {}
    for label, o in (("U2 (material, energy) order", dict(search="U2")),
                     ("U2 XSBench order (unsorted)", dict(search="U2", sort="none"))):
        ms, sts, mx = run.timed(a.ab_steps, 2, **o)
        north[label] = summarize(run, mx, sts, a.ab_steps, sms, **o)
        # the job's hash (reduced over ranks) is the same whatever the split or search
        north[label]["hash_ok"] = north[label]["hash"] == main["hash"] and north[label]["hash_consistent"]

    # ---- the paper's A/B on this workload: every search variant, same protocol, fewer steps
    ab = {}
    variants = [x for x in a.ab.split(",") if x]
    extra = [("H/history (XSBench history order, 34 lookups/particle)", dict(search="H", sort="history")),
             (f"{a.search}/coarse (bucket order without the k_bucket_refine pass)", dict(coarse=True)),
             ("M/unsorted (XSBench order)", dict(search="M", sort="none"))] if variants else []
    for label, o in [(v, dict(search=v)) for v in variants] + extra:
        ms, sts, mx = run.timed(a.ab_steps, 2, **o)
        h_job = driver.reduce_stats(sts[0].hash, sts[0].lookups, sts[0].pairs, 0.0)[0]
        ab[label] = {"value": run.total * a.ab_steps / (mx / 1e3), "sort_ms": statistics.mean(x.sample_ms for x in sts),
                     "lookup_ms": statistics.mean(x.lookup_ms for x in sts),
                     "hash_ok": h_job == main["hash"] and all(x.hash == sts[0].hash for x in sts)}

    # ---- e2e: the public API with HOST output buffers (D2H of every macro XS in the region)
    e2e = None
    if not a.no_e2e:
        host = torch.empty((run.count, 5), dtype=torch.float64).pin_memory()
        for _ in range(2):
            run.g.lookup_range(run.first, run.count, LOOKUP_SEED, host, search=a.search, sort=a.sort)
        driver.barrier()
        torch.cuda.synchronize()
        t = []
        for k in range(max(3, a.steps // 4)):
            if not a.no_flush:
                run.flush.fill_(k)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            run.g.lookup_range(run.first, run.count, LOOKUP_SEED, host, search=a.search, sort=a.sort)
            t.append(time.perf_counter() - t0)
        e2e_s = driver.max_over_ranks(sum(t))
        th = []
        for k in range(max(3, a.steps // 4)):
            if not a.no_flush:
                run.flush.fill_(k)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            if R.world == 1:
                run.xs.xs_lookup_batch(run.g.handle, run.count, LOOKUP_SEED, None)
            else:
                run.step(timing=False)
            th.append(time.perf_counter() - t0)
        e2e_h = driver.max_over_ranks(sum(th))
        e2e = {"value": run.total * len(t) / e2e_s, "unit": UNIT, "h2d_bytes_per_step": 0,
               "d2h_bytes_per_step": run.count * 5 * 8 + 16,
               "note": "xs_lookup_range writing every macroscopic XS into pinned HOST memory (D2H "
                       "overlapped with compute in 4M-lookup chunks; each rank its index range -- key-range "
                       "shards write device memory only), host wall clock, max over ranks; "
                       "inputs are the (seed, range) scalars -- lookups are drawn on device by the "
                       "method's counter-based LCG (DESIGN.md §8)",
               "hash_only": {"value": run.total * len(th) / e2e_h, "d2h_bytes_per_step": 16,
                             "call": "xs_lookup_batch (default options) / xs_lookup_range, host wall clock"}}
        del host

    cb = None
    if not a.no_cpu_baseline and R.world == 1:
        cb = cpu_baseline(w, run.count, a.cpu_seconds)
        gs = run.g.lookup_range(0, cb["_n"], LOOKUP_SEED, None, search=a.search, sort=a.sort)
        cb["_match"] = bool(gs.hash == cb["_hash"])
    run.close()
    del run

    # ---- the other configurations (sub-object), same protocol and N
    workloads = {}
    for name in [x for x in a.workloads.split(",") if x and x != w.name]:
        ww = WORKLOADS[name]
        sa = argparse.Namespace(**{**vars(a), "lookups": 0, "scaling": ""})
        r2 = Runner(sa, ww, R, scaling_of(sa, ww))
        ms, sts, mx = r2.timed(a.steps, a.warmup)
        workloads[name] = {"config": config_of(sa, ww, R.world), **summarize(r2, mx, sts, a.steps, sms)}
        r2.close()
        del r2
        torch.cuda.empty_cache()

    if R.rank != 0:
        driver.finalize()
        return
    line = {
        "metric": METRIC, "value": main["value"], "unit": UNIT, "n_gpus": R.world, "steps": a.steps,
        "warmup": a.warmup, "ms_per_step": main["ms_per_step"], "higher_is_better": True,
        "scaling": scaling_kind(scaling), "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (XSBench LCG grid + lookups, seeds 42/1070)",
        "config": config_of(a, w, R.world),
        "path": {"search": a.search, "sort": a.sort, "backend": driver.backend_name(),
                 "lookups_per_gpu": main["lookups_per_gpu"]},
        "step_ms": {"median": statistics.median(step_ms), "rsd_pct": 100 * statistics.pstdev(step_ms) /
                    statistics.mean(step_ms), "min": min(step_ms), "max": max(step_ms)},
        "phase_ms": {"sort": main["sort_ms"], "lookup": main["lookup_ms"]},
        "roofline": main["roofline"],
        "verification": {"hash": main["hash"], "lookups": main["lookups"], "pairs": main["pairs"],
                         "golden_match": main["golden_match"], "hash_consistent": main["hash_consistent"],
                         "golden": "tests/golden/hashes.json (CPU oracle: every rank's index range, or the "
                                   "ranks' sum over the whole range for key-range shards)"},
        "north_star": north,
        "workloads": workloads,
        "ab": ab,
        "gpu_launches": int(sum(s.launches for s in stats)),
        "e2e": e2e,
        "clocks": clocks,
    }
    if cb:
        line["verification"]["oracle_sample_hash_match"] = cb["_match"]
        line["cpu_baseline"] = {k: v for k, v in cb.items() if not k.startswith("_")}
    print(json.dumps(line), flush=True)
    driver.finalize()


# ------------------------------------------------------------------ launcher
def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch(a) -> int:
    """--gpus N without a torchrun environment: run this script under torch.distributed.run,
    one process per GPU, and return its exit code (rank 0 prints the JSON line)."""
    env = dict(os.environ)
    if (env.get("XS_DIST_BACKEND") or "nccl") == "nccl":
        env.setdefault("NCCL_DEBUG", "INFO")          # the communicator's nranks in the log
        env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd, env=env)


def main():
    a = parse()
    w = WORKLOADS[a.workload]
    if a.impl == "reference":
        run_reference(a, w)
        return 0
    if a.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch(a)
    run_ours(a, w)
    return 0


if __name__ == "__main__":
    sys.exit(main())
