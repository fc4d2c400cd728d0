mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bucket_(refine|scatter|count)" --launch-skip 3 --launch-count 3 -f -o gpurun_out/r01m_sort_small python tools/ncu_target.py small S material_energy 3 > gpurun_out/r01m_ncu.log 2>&1
