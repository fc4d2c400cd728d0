set -x
XS_LIB_VARIANT=tma timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tiny and S" > gpurun_out/r02af_tma_tests.log 2>&1
XS_LIB_VARIANT=tma timeout 900 python -m pytest tests/test_gpu_golden.py -x -q -k "golden and not variants" > gpurun_out/r02af_tma_golden.log 2>&1
XS_LIB_VARIANT=tma timeout 900 compute-sanitizer --tool memcheck python tools/ncu_target.py tiny S material_energy 1 > gpurun_out/r02af_tma_memcheck.log 2>&1
python tools/variant_ab.py ",tma" small,large,large-U,XL > gpurun_out/r02af_variant.log 2>&1
