mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bezier.py -x -q > gpurun_out/bz_tests2.log 2>&1
timeout 600 python tools/bezier_ab.py --out gpurun_out/bz_ab2.jsonl > gpurun_out/bz_ab2.log 2>&1
for v in "" wq4 wq8 wq16; do
  for w in small large; do
    XS_LIB_VARIANT=$v timeout 300 python bench.py --workload $w --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/wq_${v:-base}_$w.json 2>&1
  done
done
