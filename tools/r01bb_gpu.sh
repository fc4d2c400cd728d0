# r01bb: 4-ary bin-window search (XS_BIN_K4) -- GPU suite, small/large/large-U A/B against U2 in the window
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/r01bb_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01bb_gpu_tests.log
for w in small large large-U; do
for v in "" b40 "" b40; do
  echo "$w variant '$v': $(XS_LIB_VARIANT=$v timeout 600 python tools/search_ab.py $w 8 S H 2>&1 | tr '\n' ' ')" >> gpurun_out/r01bb_ab.log
done
done
