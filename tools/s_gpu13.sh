mkdir -p gpurun_out
python tools/kernel_times.py small S material_energy > gpurun_out/s13_ktimes_small.log 2>&1
python tools/kernel_times.py small S material > gpurun_out/s13_ktimes_small_mat.log 2>&1
