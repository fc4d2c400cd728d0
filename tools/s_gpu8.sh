mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_chunks.py -x -q -m gpu -k "S or chunk or ragged or bins or small_full" > gpurun_out/s8_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/s8_tests.log
for w in small large large-U XL; do
  timeout 300 python bench.py --workload $w --search S --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s8_${w}_S.json 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lookup --launch-skip 1 --launch-count 1 -f -o gpurun_out/s8_S_large python tools/ncu_target.py large S material_energy 2 > gpurun_out/s8_ncu_large.log 2>&1
