"""Side-by-side key counters of the lookup kernel in two or more ncu reports, plus the SASS
opcode mix (instructions, stall samples, shared wavefronts).  Development aid.
usage: python tools/ncu_compare.py A.ncu-rep B.ncu-rep [...] [--ops]"""
import collections, csv, io, subprocess, sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("smsp__inst_executed.sum", "warp inst"),
    ("sm__inst_executed.avg.per_cycle_active", "IPC"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy %"),
    ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed", "LSU wavefronts %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "shared ld wavefronts"),
    ("smsp__inst_executed_op_shared_ld.sum", "shared ld inst"),
    ("l1tex__lsu_writeback_active.avg.pct_of_peak_sustained_elapsed", "LSU writeback %"),
    ("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "FP64 pipe %"),
    ("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "FP64 cycles %"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit %"),
    ("launch__registers_per_thread", "regs"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads/inst"),
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        if "k_lookup" in d.get("Kernel Name", ""):
            return d, dict(zip(hdr, units))
    return {}, {}


def ops(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[1]
    ix = {k: i for i, k in enumerate(h)}
    agg = collections.defaultdict(lambda: [0.0, 0.0, 0.0])
    for r in rows[2:]:
        if len(r) < len(h):
            continue
        toks = r[1].split()
        if not toks:
            continue
        op = (toks[1] if toks[0].startswith("@") else toks[0]).split(".")[0]
        for i, k in enumerate(("Instructions Executed", "Warp Stall Sampling (All Samples)", "L1 Wavefronts Shared")):
            try:
                agg[op][i] += float(r[ix[k]].replace(",", ""))
            except Exception:
                pass
    return agg


def main():
    reps = [a for a in sys.argv[1:] if not a.startswith("--")]
    ds = [raw(r) for r in reps]
    print(f"{'':28s}" + "".join(f"{r.split('/')[-1][:22]:>24s}" for r in reps))
    for k, name in KEYS:
        vals = []
        for d, u in ds:
            v = d.get(k, "")
            vals.append(f"{v} {u.get(k, '')}".strip()[:23])
        print(f"{name:28s}" + "".join(f"{v:>24s}" for v in vals))
    if "--ops" in sys.argv:
        for r in reps:
            agg = ops(r)
            T = [sum(a[i] for a in agg.values()) or 1 for i in range(3)]
            print("==", r)
            for op, a in sorted(agg.items(), key=lambda x: -x[1][0])[:16]:
                print(f"  {op:10s} inst {100*a[0]/T[0]:5.1f}%  samples {100*a[1]/T[1]:5.1f}%  shared-wf {100*a[2]/T[2]:5.1f}%  ({a[0]:.3g} inst)")


if __name__ == "__main__":
    main()
