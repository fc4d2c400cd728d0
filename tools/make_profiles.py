"""Turn ncu --set full captures into the committed profile summaries.

usage: python tools/make_profiles.py ROUND KEY=REPORT.ncu-rep[@LOOKUPS] [KEY=REPORT ...]
  KEY = workload/search/sort (e.g. large-U/S/material_energy); LOOKUPS = lookups of the captured
  launch (default: the workload's bench count per GPU)
Writes/updates profiles/ncu_traffic.json (per-launch counters of the lookup kernel, keyed by the
configuration AND the source digest (build.py source_digest) of the libxs.so that was captured -- bench.py refuses records of
another build) and profiles/<ROUND>_ncu_<workload>_<search>[_<sort>].md (key metrics, stalls).

Counters named by BASELINE.json north_star: achieved DRAM GB/s, L2 hit rate, sectors per
request (global loads: l1tex sectors / requests), branch uniformity (divergence efficiency)."""
import json, os, sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import rows, to_mb  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.environ.get("XS_PROF_DIR") or os.path.join(ROOT, "profiles")
sys.path.insert(0, ROOT)


def libxs_sha():
    """build.py source_digest(): the build identity bench.py matches records against"""
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "_xs_build", os.path.join(ROOT, "paper_conf_cgo_murtovigplls24_b200", "build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    return b.source_digest()


def main():
    from xs_workloads import WORKLOADS
    rnd = sys.argv[1]
    os.makedirs(PROF, exist_ok=True)
    path = os.path.join(PROF, "ncu_traffic.json")
    db = json.load(open(path)) if os.path.exists(path) else {}
    sha = libxs_sha()
    for arg in sys.argv[2:]:
        key, rep = arg.split("=", 1)
        lookups = None
        if "@" in rep:
            rep, lookups = rep.split("@")
            lookups = int(lookups)
        w, s, srt = key.split("/")
        lookups = lookups or WORKLOADS[w].lookups
        hdr, units, data = rows(rep)
        md = [f"# ncu --set full: {key} ({os.path.basename(rep)}; libxs build {sha}; {lookups} lookups per launch)", ""]
        for row in data:
            d = dict(zip(hdr, row)); u = dict(zip(hdr, units))
            name = d.get("Kernel Name", "?")

            def num(k):
                v = d.get(k, "")
                try:
                    return float(v.replace(",", "")) if v not in ("", "n/a") else None
                except ValueError:
                    return None
            rd = to_mb(num("dram__bytes_read.sum") or 0, u.get("dram__bytes_read.sum", "")) * 1e6
            wr = to_mb(num("dram__bytes_write.sum") or 0, u.get("dram__bytes_write.sum", "")) * 1e6
            dur = num("gpu__time_duration.sum")
            dur_us = dur * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}.get(u.get("gpu__time_duration.sum", ""), 1e-3)
            inst = num("smsp__inst_executed.sum")
            sec, req = num("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"), num("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")
            spr = sec / req if sec and req else None
            stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): num(k) or 0 for k in hdr
                      if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
            tot = sum(stalls.values()) or 1
            top = sorted(stalls.items(), key=lambda x: -x[1])[:6]
            lsu_pct = num("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed")
            rec = {"libxs_sha": sha, "report": os.path.basename(rep), "round": rnd, "kernel": name.split("(")[0][:80],
                   "lookups": lookups, "ncu_duration_us": dur_us, "dram_bytes_per_launch": rd + wr,
                   "dram_read_bytes": rd, "dram_write_bytes": wr,
                   "dram_gbps": (rd + wr) / (dur_us * 1e-6) / 1e9 if dur_us else None,
                   "dram_pct_of_peak": num("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
                   "warp_inst_per_launch": inst, "ipc": num("sm__inst_executed.avg.per_cycle_active"),
                   "occupancy_pct": num("sm__warps_active.avg.pct_of_peak_sustained_active"),
                   "registers": num("launch__registers_per_thread"),
                   "l1_hit_pct": num("l1tex__t_sector_hit_rate.pct"), "l2_hit_pct": num("lts__t_sector_hit_rate.pct"),
                   "sectors_per_request": spr,
                   "threads_per_warp_inst": num("smsp__thread_inst_executed_per_inst_executed.ratio"),
                   "branch_uniform_pct": num("smsp__sass_average_branch_targets_threads_uniform.pct"),
                   "fp64_pipe_pct": num("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active"),
                   "lsu_wavefronts_pct_of_peak": lsu_pct,
                   "issue_active_pct": num("sm__inst_issued.avg.pct_of_peak_sustained_active"),
                   "stalls_pct": {k: round(100 * v / tot, 1) for k, v in top}}
            md += [f"## {name[:120]}", "",
                   "| metric | value |", "|---|---|",
                   f"| duration (ncu, serialised, cold) | {dur_us:.1f} us |",
                   f"| DRAM read / write | {rd/1e6:.1f} MB / {wr/1e6:.1f} MB ({rec['dram_gbps'] or 0:.0f} GB/s, {rec['dram_pct_of_peak']} % of peak) |",
                   f"| warp instructions | {inst:.4g} |" if inst else "| warp instructions | n/a |",
                   f"| IPC (active) | {rec['ipc']} |",
                   f"| achieved occupancy % | {rec['occupancy_pct']} |",
                   f"| registers / thread | {rec['registers']} |",
                   f"| L1 hit % / L2 hit % | {rec['l1_hit_pct']} / {rec['l2_hit_pct']} |",
                   f"| sectors per request (global loads) | {spr:.2f} |" if spr else "| sectors per request | n/a |",
                   f"| threads per warp instruction (warp efficiency x 32) | {rec['threads_per_warp_inst']} |",
                   f"| branch targets uniform % | {rec['branch_uniform_pct']} |",
                   f"| FP64 pipe % | {rec['fp64_pipe_pct']} |",
                   f"| L1/shared data pipe (LSU wavefronts) % of peak | {lsu_pct} |",
                   "", "stall samples: " + ", ".join(f"{k} {100*v/tot:.1f}%" for k, v in top), ""]
            if "k_lookup" in name:
                db[key] = rec
        suffix = "" if srt == "material_energy" else "_" + srt
        with open(os.path.join(PROF, f"{rnd}_ncu_{w}_{s}{suffix}.md"), "w") as f:
            f.write("\n".join(md) + "\n")
    json.dump(db, open(path, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
