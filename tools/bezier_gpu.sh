set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bezier.py -x -q > gpurun_out/bz_tests.log 2>&1
timeout 600 python tools/bezier_ab.py --out gpurun_out/bz_ab.jsonl > gpurun_out/bz_ab.log 2>&1
for v in M U2 S T; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_bz --launch-skip 1 --launch-count 1 -f -o gpurun_out/bz_${v}_paper_fp64 python tools/bezier_ab.py --ncu-target paper $v fp64 > gpurun_out/bz_ncu_$v.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/r01c_launches_small_step.csv python bench.py --steps 2 --warmup 3 --ab '' --no-cpu-baseline --no-e2e > gpurun_out/r01c_launch_bench2.log 2>&1
