"""A/B of the bezier-surface loop variants (Listing 2) on one GPU.

usage: python tools/bezier_ab.py [--reps R] [--out gpurun_out/bezier_ab.jsonl] [--ncu-target W V DT]
Times every variant (M, M2, U1, U2, S, T) x {fp64, fp32} x {paper, deep} with CUDA events
on the launching stream (warm-up 2, best and median of R), checks every variant bit-equal
to T, and prints one JSON line per case.  --ncu-target runs a single case twice (for
`ncu -k regex:k_bz --launch-skip 1 --launch-count 1`)."""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cgo_murtovigplls24_b200 as xs  # noqa: E402
from xs_workloads import BEZIER_WORKLOADS, bezier_control_net  # noqa: E402

VARIANTS = ["M", "M2", "U1", "U2", "S", "T"]
DT = {"fp64": torch.float64, "fp32": torch.float32}


def blends_per_point(w, variant):
    """Listing-2 loop evaluations per output point: the original program's placement
    (b_i per ki, b_j per (ki, kj)) or T's per-tile hoisting (16 x 16 tiles)."""
    if variant == "T":
        return ((w.ni + 1) + (w.nj + 1)) * 16 / 256
    return (w.ni + 1) + (w.ni + 1) * (w.nj + 1)


def time_case(w, dt, variant, reps):
    P = torch.tensor(bezier_control_net(w.ni, w.nj, dtype="float64"), device="cuda").to(DT[dt])
    out = torch.empty((w.res_i, w.res_j, 3), dtype=DT[dt], device="cuda")
    s = torch.cuda.current_stream()
    for _ in range(2):
        xs.bezier_surface(P, w.res_i, w.res_j, variant=variant, out=out)
    ms = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(s)
        xs.bezier_surface(P, w.res_i, w.res_j, variant=variant, out=out)
        b.record(s)
        b.synchronize()
        ms.append(a.elapsed_time(b))
    return out, ms


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--out", default="")
    ap.add_argument("--ncu-target", nargs=3, metavar=("WORKLOAD", "VARIANT", "DTYPE"))
    a = ap.parse_args()
    if a.ncu_target:
        w, v, dt = a.ncu_target
        time_case(BEZIER_WORKLOADS[w], dt, v, 1)
        return
    lines = []
    for wname in ("paper", "deep"):
        w = BEZIER_WORKLOADS[wname]
        for dt in ("fp64", "fp32"):
            ref, base = None, None
            for v in ["T"] + VARIANTS[:-1]:
                out, ms = time_case(w, dt, v, a.reps)
                if ref is None:
                    ref = out.clone()
                same = bool(torch.equal(out, ref))
                best, med = min(ms), statistics.median(ms)
                pts = w.res_i * w.res_j
                rec = {"workload": wname, "ni": w.ni, "nj": w.nj, "res": [w.res_i, w.res_j], "dtype": dt,
                       "variant": v, "ms_best": round(best, 4), "ms_median": round(med, 4),
                       "points_per_s": pts / (med * 1e-3),
                       "loop_evals_per_s": pts * blends_per_point(w, v) / (med * 1e-3),
                       "bit_equal_to_T": same}
                if v == "M":
                    base = med
                lines.append(rec)
            for rec in lines:
                if rec["workload"] == wname and rec["dtype"] == dt:
                    m = next(r for r in lines if r["workload"] == wname and r["dtype"] == dt and r["variant"] == "M")
                    rec["speedup_vs_M"] = round(m["ms_median"] / rec["ms_median"], 3)
    for rec in lines:
        print(json.dumps(rec))
    if a.out:
        with open(a.out, "w") as f:
            f.write("\n".join(json.dumps(r) for r in lines) + "\n")
    if not all(r["bit_equal_to_T"] for r in lines):
        sys.exit("variants disagree")


if __name__ == "__main__":
    main()
