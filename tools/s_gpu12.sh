mkdir -p gpurun_out
python tools/sort_probe.py small > gpurun_out/s12_sortprobe_small.log 2>&1
python tools/sort_probe.py large > gpurun_out/s12_sortprobe_large.log 2>&1
for v in cap64 sm32 sm128; do
  for w in small large XL; do
    XS_LIB_VARIANT=$v timeout 300 python bench.py --workload $w --search S --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s12_${v}_${w}.json 2>&1
  done
done
