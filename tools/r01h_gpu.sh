# r01h: re-entry check on HEAD -- full GPU suite, smoke, bench lines for all workloads, reference arm, launch list, ncu of the default kernel
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r01h_smi.txt 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r01h_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01h_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/r01h_smoke.log 2>&1
for w in small large large-U XL; do
  timeout 900 python bench.py --workload $w > gpurun_out/r01h_bench_$w.json 2> gpurun_out/r01h_bench_$w.err
done
timeout 600 python bench.py --impl reference > gpurun_out/r01h_bench_reference.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01h_launches_small.csv python bench.py --steps 2 --warmup 1 --ab '' --no-cpu-baseline > gpurun_out/r01h_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lookup --launch-skip 1 --launch-count 1 -f -o gpurun_out/r01h_S_small python tools/ncu_target.py small S material_energy 2 > gpurun_out/r01h_ncu_small.log 2>&1
