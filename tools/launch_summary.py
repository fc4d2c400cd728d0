"""Summarise an `ncu --metrics gpu__time_duration.sum --csv --log-file X.csv` launch list
into a markdown table (kernel, launches, mean duration, share of the lookup step).
usage: python tools/launch_summary.py LAUNCHES.csv TITLE > profiles/<round>_launches_<w>.md
Step kernels are the sort kernels and k_lookup; everything else is setup or L2 flush."""
import csv
import sys
from collections import OrderedDict

STEP = ("k_bucket_count", "k_bucket_colscan", "k_bucket_base", "k_zero_window", "k_bucket_scatter", "k_bucket_gather",
        "k_bucket_refine", "k_lookup", "k_history", "k_search", "k_interp")
# the OUTS instantiations (k_lookup*<grid, 1>) write outputs: the e2e pass, not the timed step
E2E = ("<1, 1>", "<0, 1>", "<2, 1>", "true>")
UNIT = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}


def main():
    path, title = sys.argv[1], sys.argv[2]
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.DictReader(lines))
    agg = OrderedDict()
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        us = float(r["Metric Value"].replace(",", "")) * UNIT.get(r["Metric Unit"], 1e-3)
        a = agg.setdefault(r["Kernel Name"][:90], [0, 0.0])
        a[0] += 1
        a[1] += us
    is_step = lambda k: any(s in k for s in STEP) and not any(e in k for e in E2E)
    # the default step is the sort + the staged kernel (XS_SEARCH_S); any other lookup kernel in
    # the list belongs to the bench's north-star / A/B passes
    main_lookup = "k_lookup_staged" if any("k_lookup_staged" in k for k in agg) else "k_lookup"
    is_sort = lambda k: "k_bucket" in k or "k_zero_window" in k
    in_default = lambda k: is_step(k) and (is_sort(k) or main_lookup in k)
    # one step = the lookup kernel's mean launch + each sort kernel's launches per sort (the
    # sort also runs for the sorted north-star / A/B passes: per sort = launches / count launches)
    sorts = max((v[0] for k, v in agg.items() if "k_bucket_count" in k), default=1)
    per_step = {k: (v[1] / sorts if is_sort(k) else v[1] / v[0]) for k, v in agg.items() if in_default(k)}
    step_total = sum(per_step.values())
    steps = max((v[0] for k, v in agg.items() if main_lookup in k and in_default(k)), default=1)
    print(f"# {title}\n")
    print("`ncu --metrics gpu__time_duration.sum --clock-control none` (serialised, cold: compare SHARES;"
          " ncu flushes the caches between launches, which undoes what `k_zero_window` leaves in L2 for"
          " the scatter window that follows it)\n")
    print(f"Default step (sort + `{main_lookup}`): {step_total:.1f} us ({steps} lookup launches, {sorts} sorts).\n")
    print("| kernel | launches | mean us (ncu) | share of a default step |\n|---|---|---|---|")
    for k, (n, us) in agg.items():
        if in_default(k):
            share = f"{100 * per_step[k] / step_total:.1f}%"
        elif is_step(k):
            share = "north-star / A/B pass"
        else:
            share = "setup / L2 flush / e2e"
        print(f"| `{k}` | {n} | {us / n:.1f} | {share} |")


if __name__ == "__main__":
    main()
