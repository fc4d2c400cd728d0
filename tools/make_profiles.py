"""Turn ncu --set full captures into the committed profile summaries.

usage: python tools/make_profiles.py ROUND KEY=REPORT.ncu-rep [KEY=REPORT ...]
  KEY = workload/search/sort (e.g. small/W/material_energy)
Writes/updates profiles/ncu_traffic.json (per-launch DRAM bytes and warp instructions of
k_lookup) and profiles/<ROUND>_ncu_<workload>_<search>.md (key metrics + stall mix)."""
import json, os, subprocess, sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import rows, to_mb  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")


def main():
    rnd = sys.argv[1]
    os.makedirs(PROF, exist_ok=True)
    path = os.path.join(PROF, "ncu_traffic.json")
    db = json.load(open(path)) if os.path.exists(path) else {}
    for arg in sys.argv[2:]:
        key, rep = arg.split("=", 1)
        hdr, units, data = rows(rep)
        md = [f"# ncu --set full: {key} ({os.path.basename(rep)})", ""]
        for row in data:
            d = dict(zip(hdr, row)); u = dict(zip(hdr, units))
            name = d.get("Kernel Name", "?")
            def num(k):
                v = d.get(k, "")
                return float(v.replace(",", "")) if v not in ("", "n/a") else None
            rd = to_mb(num("dram__bytes_read.sum") or 0, u.get("dram__bytes_read.sum", "")) * 1e6
            wr = to_mb(num("dram__bytes_write.sum") or 0, u.get("dram__bytes_write.sum", "")) * 1e6
            dur = num("gpu__time_duration.sum")
            dur_us = dur * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}.get(u.get("gpu__time_duration.sum", ""), 1e-3)
            inst = num("smsp__inst_executed.sum")
            stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): num(k) or 0 for k in hdr
                      if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
            tot = sum(stalls.values()) or 1
            top = sorted(stalls.items(), key=lambda x: -x[1])[:6]
            md += [f"## {name[:120]}", "",
                   f"| metric | value |", "|---|---|",
                   f"| duration (ncu, serialised, cold) | {dur_us:.1f} us |",
                   f"| DRAM read / write | {rd/1e6:.1f} MB / {wr/1e6:.1f} MB |",
                   f"| warp instructions | {inst:.4g} |" if inst else "| warp instructions | n/a |",
                   f"| IPC (active) | {num('sm__inst_executed.avg.per_cycle_active')} |",
                   f"| achieved occupancy % | {num('sm__warps_active.avg.pct_of_peak_sustained_active')} |",
                   f"| registers / thread | {num('launch__registers_per_thread')} |",
                   f"| L1 hit % / L2 hit % | {num('l1tex__t_sector_hit_rate.pct')} / {num('lts__t_sector_hit_rate.pct')} |",
                   f"| DRAM throughput % of peak | {num('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed')} |",
                   f"| threads per warp instruction | {num('smsp__thread_inst_executed_per_inst_executed.ratio')} |",
                   f"| branch targets uniform % | {num('smsp__sass_average_branch_targets_threads_uniform.pct')} |",
                   f"| FP64 pipe % | {num('sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active')} |",
                   "", "stall samples: " + ", ".join(f"{k} {100*v/tot:.1f}%" for k, v in top), ""]
            lsu_pct = num("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed")
            md.insert(-2, f"L1/shared data pipe (LSU wavefronts) % of peak: {lsu_pct}")
            if "k_lookup" in name:
                db[key] = {"dram_bytes_per_launch": rd + wr, "warp_inst_per_launch": inst,
                           "ncu_duration_us": dur_us, "report": os.path.basename(rep), "round": rnd,
                           "lsu_wavefronts_pct_of_peak": lsu_pct,
                           "lsu_wavefronts_per_launch": sum(num(k) or 0 for k in (
                               "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
                               "l1tex__t_output_wavefronts_pipe_lsu_mem_global_op_ld.sum",
                               "l1tex__t_output_wavefronts_pipe_lsu_mem_local_op_ld.sum",
                               "l1tex__t_output_wavefronts_pipe_lsu_mem_local_op_st.sum"))}
        w, s, _ = key.split("/")
        with open(os.path.join(PROF, f"{rnd}_ncu_{w}_{s}.md"), "w") as f:
            f.write("\n".join(md) + "\n")
    json.dump(db, open(path, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
