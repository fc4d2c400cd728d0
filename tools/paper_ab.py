"""The paper's A/B methodology on B200, reported (PAPER.md:234-246,
306-324, 344-352): lookup-kernel times of every search variant x {XSBench order, (material,
energy) order} x 3 grid types (tools/ab_sweep.py JSON lines), and the ncu counters of the same
configurations (tools/ab_sweep.py --ncu under `ncu --metrics`, one k_lookup launch per
configuration in ab_sweep's order), mapped as SURVEY.md §5:

  warp execution efficiency = threads per executed warp instruction / 32 (nvprof's
  warp_execution_efficiency); IPC; branch uniformity; `no_instruction` stall
  (PAPER.md:474's stall_inst_fetch); SEL + MOV warp instructions (the paper's inst_misc: selp /
  mov); global-load sectors per request; L2 hit rate.

usage: python tools/paper_ab.py OUT.md --timing small=A.jsonl [--timing large=B.jsonl]
                                --ncu NCU.csv [--ncu-lookups 4000000]"""
import argparse, collections, csv, json, re

SEARCHES = ["M", "M2", "M4", "M8", "U1", "U2", "U4", "U8", "B", "W", "H"]
SORTS = ["none", "material_energy"]
GRIDS = [(1, "nuclide"), (0, "unionized"), (2, "hash")]
METRICS = ["smsp__thread_inst_executed_per_inst_executed.ratio", "smsp__inst_executed.sum",
           "sm__inst_executed.avg.per_cycle_active", "smsp__sass_average_branch_targets_threads_uniform.pct",
           "smsp__warp_issue_stalled_no_instruction_per_warp_active.pct",
           "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
           "lts__t_sector_hit_rate.pct", "dram__bytes_read.sum", "gpu__time_duration.sum",
           "sass__inst_executed_per_opcode"]


def load_ncu(path):
    """launches in order -> {metric: value or {opcode: count}}"""
    launches = collections.OrderedDict()
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    for row in csv.DictReader(lines):
        if "k_lookup" not in row.get("Kernel Name", ""):
            continue
        lid = int(row["ID"])
        d = launches.setdefault(lid, {})
        name, val = row["Metric Name"], row["Metric Value"]
        if name == "sass__inst_executed_per_opcode":
            d[name] = {k: float(v.replace(",", "")) for k, v in re.findall(r"([A-Z][A-Z0-9_]*)\s*[:=]\s*([\d.,eE+]+)", val)}
        else:
            try:
                d[name] = float(val.replace(",", ""))
            except ValueError:
                d[name] = None
    return list(launches.values())


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("out")
    ap.add_argument("--timing", action="append", default=[])
    ap.add_argument("--ncu")
    ap.add_argument("--ncu-lookups", type=int, default=4_000_000)
    a = ap.parse_args()
    times = {}
    for t in a.timing:
        w, p = t.split("=", 1)
        for line in open(p):
            if line.startswith("{"):
                d = json.loads(line)
                times[(w, d["grid"], d["sort"], d["search"])] = d["lookup_ms"]
    workloads = [t.split("=", 1)[0] for t in a.timing]
    ncu = {}
    if a.ncu:
        launches = load_ncu(a.ncu)
        order = [(gt, srt, s) for gt, _ in GRIDS for srt in SORTS for s in SEARCHES]
        for key, d in zip(order, launches):
            ncu[key] = d
    out = ["# The paper's A/B on B200, on HEAD (SURVEY.md §8f rank 1; PAPER.md:234-246, 306-324, 344-352)", "",
           "Lookup-kernel time = CUDA events around `k_lookup` alone, median of 5 after 2 warm-ups "
           "(`tools/ab_sweep.py`); counters: one ncu launch per configuration on "
           f"{a.ncu_lookups:,} lookups of the small workload (`tools/ab_sweep.py --ncu`), mapped as SURVEY.md §5. "
           "Variants (SASS shapes pinned by tests/test_sass.py): M = Listing 3 (select form, Listing 4); "
           "M<k> = unroll only; U1 = unmerge only; U<u> = unroll and unmerge (every one of the 2^u paths with its "
           "own back edge, tools/gen_uu.py; the true-true path of U2 is Listing 5's); B = branchless; W = "
           "warp-cooperative separator tree + U2; H = bin-bounded window + U2.  All hashes equal the oracle's.", "",
           "Columns: `x M` = speedup over M in the same grid and order; warp eff = threads per warp instruction / 32; "
           "SEL+MOV = the paper's inst_misc class; sect/req = global-load sectors per request.", ""]
    for gt, gname in GRIDS:
        out += [f"## {gname} grid", ""]
        hdr = "| order | variant | " + " | ".join(f"{w} ms | x M" for w in workloads) + \
              " | warp eff % | warp inst | SEL+MOV | IPC | branch uniform % | no_instr stall % | sect/req | L2 hit % |"
        out += [hdr, "|" + "---|" * (hdr.count("|") - 1)]
        for srt in SORTS:
            for s in SEARCHES:
                cells = []
                for w in workloads:
                    t = times.get((w, gt, srt, s))
                    m = times.get((w, gt, srt, "M"))
                    cells += [f"{t:.2f}" if t else "", f"{m / t:.2f}x" if t and m else ""]
                d = ncu.get((gt, srt, s), {})
                thr = d.get("smsp__thread_inst_executed_per_inst_executed.ratio")
                ops = d.get("sass__inst_executed_per_opcode") or {}
                selmov = (ops.get("SEL", 0) + ops.get("MOV", 0)) if ops else None
                sec, req = d.get("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"), d.get("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")

                def f(v, fmt):
                    return format(v, fmt) if isinstance(v, (int, float)) else ""
                cells += [f(100 * thr / 32 if thr else None, ".1f"), f(d.get("smsp__inst_executed.sum"), ".3g"),
                          f(selmov, ".3g"), f(d.get("sm__inst_executed.avg.per_cycle_active"), ".2f"),
                          f(d.get("smsp__sass_average_branch_targets_threads_uniform.pct"), ".1f"),
                          f(d.get("smsp__warp_issue_stalled_no_instruction_per_warp_active.pct"), ".1f"),
                          f(sec / req if sec and req else None, ".2f"), f(d.get("lts__t_sector_hit_rate.pct"), ".1f")]
                out.append(f"| {'XSBench' if srt == 'none' else 'sorted'} | {s} | " + " | ".join(cells) + " |")
        out.append("")
    with open(a.out, "w") as fo:
        fo.write("\n".join(out) + "\n")


if __name__ == "__main__":
    main()
