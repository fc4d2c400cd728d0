mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/r01n_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01n_tests.log
for w in small large-U XL; do timeout 300 python tools/refine_ab.py $w S 10 >> gpurun_out/r01n_ab.log 2>&1; done
python tools/kernel_times.py small S > gpurun_out/r01n_ktimes_small.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bucket_refine" --launch-skip 3 --launch-count 1 -f -o gpurun_out/r01n_refine_small python tools/ncu_target.py small S material_energy 3 > gpurun_out/r01n_ncu.log 2>&1
