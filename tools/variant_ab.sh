# A/B of experimental library builds (XS_LIB_VARIANT) on the bench's lookup path.
# usage: bash tools/variant_ab.sh "v1 v2 ..." "small large" [reps]
mkdir -p gpurun_out
reps=${3:-2}
for r in $(seq 1 $reps); do
  for v in $1; do
    for w in $2; do
      [ "$v" = base ] && lv= || lv=$v
      XS_LIB_VARIANT=$lv timeout 300 python bench.py --workload $w --steps 10 --ab '' --no-e2e --no-cpu-baseline \
        | grep '^{' > gpurun_out/vab_${v}_${w}_$r.json
    done
  done
done
python - <<'PY'
import glob, json, collections
res = collections.defaultdict(list)
for f in sorted(glob.glob("gpurun_out/vab_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    _, v, w, r = f[:-5].split("/")[-1].split("_", 3)
    res[(v, w)].append((d["value"], d["phase_ms"]["lookup"], d["verification"]["hash"]))
for (v, w), xs in sorted(res.items()):
    print(v, w, " ".join("%.4g/%.3fms/%d" % x for x in xs))
PY
