# r01bd: 16 B key loads in the windowed scatter (XS_SCATTER_VEC) -- GPU suite, sort A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/r01bd_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01bd_gpu_tests.log
for w in small large-U XL; do
for v in "" sv0 "" sv0; do
  echo "$w variant '$v': $(XS_LIB_VARIANT=$v timeout 600 python tools/search_ab.py $w 6 S 2>&1 | tr '\n' ' ')" >> gpurun_out/r01bd_ab.log
done
done
