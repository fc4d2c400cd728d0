set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/r01c_smoke.log 2>&1
for w in small large large-U XL; do
  timeout 600 python bench.py --workload $w > gpurun_out/r01c_bench_$w.json 2> gpurun_out/r01c_bench_$w.err
done
timeout 600 python bench.py --impl reference > gpurun_out/r01c_bench_reference.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01c_launches_small.csv python bench.py --steps 2 --warmup 1 --ab '' --no-cpu-baseline > gpurun_out/r01c_launch_bench.log 2>&1
for w in small large; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lookup --launch-skip 1 --launch-count 1 -f -o gpurun_out/r01c_H_$w python tools/ncu_target.py $w H material_energy 2 > gpurun_out/r01c_ncu_$w.log 2>&1
done
