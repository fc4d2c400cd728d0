mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_lookup_staged|k_bucket_scatter" --launch-skip 2 --launch-count 2 -f -o gpurun_out/r01q_small python tools/ncu_target.py small S material_energy 3 > gpurun_out/r01q_ncu.log 2>&1
