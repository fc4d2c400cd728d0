mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/r01x_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01x_tests.log
for w in small large large-U XL; do timeout 300 python tools/search_ab.py $w 5 S C >> gpurun_out/r01x_ab.log 2>&1; done
