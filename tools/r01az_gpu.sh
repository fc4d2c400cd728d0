# r01az: hash-window fast path (XS_HASH_FAST) -- GPU suite, XL A/B against the R7-as-written build
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/r01az_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01az_gpu_tests.log
for v in "" hf0 "" hf0; do
  echo "variant '$v': $(XS_LIB_VARIANT=$v timeout 600 python tools/search_ab.py XL 5 S H 2>&1 | tr '\n' ' ')" >> gpurun_out/r01az_ab.log
done
timeout 900 python bench.py --workload XL --ab "" --no-cpu-baseline > gpurun_out/r01az_bench_XL.json 2> gpurun_out/r01az_bench_XL.err
