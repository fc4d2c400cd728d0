mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_chunks.py -x -q -m gpu -k "S or chunk or ragged or bins" > gpurun_out/s5_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/s5_tests.log
for v in "" b4l1 b3l1 b3l2 b2l2; do
  for w in small large; do
      XS_LIB_VARIANT=$v timeout 300 python bench.py --workload $w --search S --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s5_${v:-b4l2}_${w}_S.json 2>&1
  done
done
