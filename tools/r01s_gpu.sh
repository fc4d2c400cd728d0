mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/r01s_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01s_tests.log
for w in small large large-U XL; do timeout 300 python tools/refine_ab.py $w S 10 >> gpurun_out/r01s_ab.log 2>&1; done
python tools/kernel_times.py small S > gpurun_out/r01s_ktimes_small.log 2>&1
python tools/kernel_times.py XL S > gpurun_out/r01s_ktimes_XL.log 2>&1
