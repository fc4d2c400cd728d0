# round-1 re-entry check: GPU suite, smoke, default bench line on the restored HEAD
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r01f_smi.txt 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/r01f_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01f_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01f_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r01f_smoke.log
timeout 600 python bench.py > gpurun_out/r01f_bench_small.json 2> gpurun_out/r01f_bench_small.err
