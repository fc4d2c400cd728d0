mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_chunks.py -x -q -m gpu -k "S or chunk or ragged or bins or small_full" > gpurun_out/s7_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/s7_tests.log
for w in small large; do
  timeout 300 python bench.py --workload $w --search S --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s7_${w}_S.json 2>&1
done
