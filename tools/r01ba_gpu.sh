# r01ba: 4-ary hash-window search (XS_HASH_K4) -- GPU suite, XL A/B against Listing 1 in the window
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/r01ba_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01ba_gpu_tests.log
for v in "" k40 "" k40; do
  echo "variant '$v': $(XS_LIB_VARIANT=$v timeout 600 python tools/search_ab.py XL 5 S H 2>&1 | tr '\n' ' ')" >> gpurun_out/r01ba_ab.log
done
