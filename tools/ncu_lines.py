"""Per-source-line totals from an ncu report's source page (cuda,sass view): stall samples,
warp instructions, shared-memory wavefronts, global L1 tag requests and L2 sectors.
usage: python tools/ncu_lines.py REPORT.ncu-rep [TOP]"""
import csv, io, subprocess, sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    f = None
    hdr = None
    rows = []
    for rec in csv.reader(io.StringIO(out)):
        if not rec:
            continue
        if rec[0] == "File Path":
            f = rec[1].split("/")[-1]
            continue
        if rec[0] == "Line No":
            hdr = rec
            continue
        if hdr is None or rec[0] == "" or rec[0] == "Function Name":
            continue
        d = dict(zip(hdr, rec))
        def num(k):
            try:
                return float(d.get(k, "0").replace(",", ""))
            except ValueError:
                return 0.0
        rows.append((f, rec[0], rec[1][:70], num("Warp Stall Sampling (All Samples)"), num("Instructions Executed"),
                     num("L1 Wavefronts Shared"), num("L1 Tag Requests Global"), num("L2 Theoretical Sectors Global")))
    tot = [sum(r[i] for r in rows) for i in range(3, 8)]
    print(f"totals: samples {tot[0]:.0f}  warp inst {tot[1]:.3e}  shared wavefronts {tot[2]:.3e}  "
          f"global L1 tag req {tot[3]:.3e}  L2 sectors {tot[4]:.3e}")
    print(f"{'file:line':28s} {'samp%':>6s} {'inst%':>6s} {'shwf%':>6s} {'gtag%':>6s} {'l2s%':>6s}  source")
    for r in sorted(rows, key=lambda r: -r[3])[:top]:
        pc = [100 * r[i] / tot[i - 3] if tot[i - 3] else 0 for i in range(3, 8)]
        print(f"{r[0] + ':' + r[1]:28s} " + " ".join(f"{p:6.1f}" for p in pc) + "  " + r[2])


if __name__ == "__main__":
    main()
