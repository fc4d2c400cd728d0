# r01f: S as the default search -- full GPU suite, smoke, bench lines for all workloads, launch list
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/r01f_gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01f_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/r01f_smoke.log 2>&1
for w in small large large-U XL; do
  timeout 900 python bench.py --workload $w > gpurun_out/r01f_bench_$w.json 2> gpurun_out/r01f_bench_$w.err
done
timeout 600 python bench.py --impl reference > gpurun_out/r01f_bench_reference.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01f_launches_small.csv python bench.py --steps 2 --warmup 1 --ab '' --no-cpu-baseline > gpurun_out/r01f_launch_bench.log 2>&1
