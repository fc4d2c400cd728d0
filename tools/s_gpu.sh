# XS_SEARCH_S bring-up: parity on tiny/chunks, then A/B vs H (small, large), two register budgets
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_chunks.py -x -q -m gpu -k "S or chunk" > gpurun_out/s_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/s_tests.log
for v in "" s3; do
  for w in small large; do
    for s in S H; do
      XS_LIB_VARIANT=$v timeout 300 python bench.py --workload $w --search $s --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s_${v:-base}_${w}_$s.json 2>&1
    done
  done
done
