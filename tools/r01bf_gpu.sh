# r01bf: end-of-session validation (4-ary windows, 16 B scatter key loads, 64 MB windows) -- GPU suite, smoke, bench lines, launch list, ncu small + large + XL lookup kernel, warm timeline
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r01bf_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01bf_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/r01bf_smoke.log 2>&1
for w in small large large-U XL; do
  timeout 900 python bench.py --workload $w > gpurun_out/r01bf_bench_$w.json 2> gpurun_out/r01bf_bench_$w.err
done
timeout 600 python bench.py --impl reference > gpurun_out/r01bf_bench_reference.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01bf_launches_small.csv python bench.py --steps 2 --warmup 1 --ab "" --no-cpu-baseline --no-e2e > gpurun_out/r01bf_launch_bench.log 2>&1
for w in small large; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_lookup_staged|k_bucket" --launch-skip 6 --launch-count 6 -f -o gpurun_out/r01bf_S_$w python tools/ncu_target.py $w S material_energy 3 > gpurun_out/r01bf_ncu_$w.log 2>&1
done
python tools/kernel_times.py small S > gpurun_out/r01bf_kt_small.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_lookup_staged" --launch-skip 2 --launch-count 1 -f -o gpurun_out/r01bf_S_XL python tools/ncu_target.py XL S material_energy 3 > gpurun_out/r01bf_ncu_XL.log 2>&1
