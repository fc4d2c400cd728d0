"""Summarise an ncu --set full report: per kernel the key SOL / occupancy / stall metrics.
usage: python tools/ncu_summary.py REPORT.ncu-rep [--stalls] [--json]"""
import csv, io, json, subprocess, sys

KEYS = [
    ("gpu__time_duration.sum", "dur_us", 1e-3),
    ("dram__bytes_read.sum", "dram_rd_MB", None),
    ("dram__bytes_write.sum", "dram_wr_MB", None),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct", 1),
    ("lts__t_sector_hit_rate.pct", "l2_hit_pct", 1),
    ("l1tex__t_sector_hit_rate.pct", "l1_hit_pct", 1),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_pct", 1),
    ("sm__inst_executed.avg.per_cycle_active", "ipc", 1),
    ("smsp__inst_executed.sum", "warp_inst", 1),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occ_pct", 1),
    ("launch__registers_per_thread", "regs", 1),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "thr_per_inst", 1),
    ("smsp__sass_average_branch_targets_threads_uniform.pct", "branch_uniform_pct", 1),
    ("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "fp64_pipe_pct", 1),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1_ld_sectors", 1),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1_ld_requests", 1),
]


def rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units = r[0], r[1]
    return hdr, units, r[2:]


def to_mb(v, unit):
    scale = {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1, "Gbyte": 1e3, "KB": 1e-3, "MB": 1, "GB": 1e3}
    return v * scale.get(unit, 1)


def main():
    rep = sys.argv[1]
    hdr, units, data = rows(rep)
    res = []
    for row in data:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        name = d.get("Kernel Name", "?")
        item = {"kernel": name.split("(")[0][:60]}
        for k, short, sc in KEYS:
            if k in d and d[k] not in ("", "n/a"):
                v = float(d[k].replace(",", ""))
                if sc is None:
                    v = to_mb(v, u.get(k, ""))
                elif k == "gpu__time_duration.sum":
                    v = v * ({"nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}.get(u.get(k, ""), 1e-3))
                item[short] = round(v, 3)
        if "--stalls" in sys.argv:
            st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(d[k].replace(",", "") or 0)
                  for k in hdr if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
            tot = sum(st.values()) or 1
            item["stalls"] = {k: round(100 * v / tot, 1) for k, v in sorted(st.items(), key=lambda x: -x[1])[:6]}
        res.append(item)
    if "--json" in sys.argv:
        print(json.dumps(res, indent=1))
    else:
        for it in res:
            print(json.dumps(it))


if __name__ == "__main__":
    main()
