mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bucket_refine" --launch-skip 1 --launch-count 1 -f -o gpurun_out/r01o_refine_small python tools/ncu_target.py small S material_energy 3 > gpurun_out/r01o_ncu.log 2>&1
