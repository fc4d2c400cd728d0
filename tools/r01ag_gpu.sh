mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -2 > gpurun_out/r01ag_tests.log
bash tools/var_search_ab.sh r01ag S
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_lookup_staged" --launch-skip 1 --launch-count 1 -f -o gpurun_out/r01ag_S_small python tools/ncu_target.py small S material_energy 2 > gpurun_out/r01ag_ncu.log 2>&1
