mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_chunks.py -x -q -m gpu -k "S or chunk or ragged or bins" > gpurun_out/s2_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/s2_tests.log
for v in s2; do
  for w in small large; do
      XS_LIB_VARIANT=$v timeout 300 python bench.py --workload $w --search S --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s_${v:-base}_${w}_S.json 2>&1
  done
done
for w in small large; do
  XS_LIB_VARIANT=s3 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lookup --launch-skip 1 --launch-count 1 -f -o gpurun_out/s3_S_$w python tools/ncu_target.py $w S material_energy 2 > gpurun_out/s3_ncu_$w.log 2>&1
done
