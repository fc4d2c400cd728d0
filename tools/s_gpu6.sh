mkdir -p gpurun_out
for v in b2l3; do
  for w in small large; do
      XS_LIB_VARIANT=$v timeout 300 python bench.py --workload $w --search S --steps 10 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s6_${v}_${w}_S.json 2>&1
  done
done
for w in large-U XL; do
  for s in S H; do
    timeout 600 python bench.py --workload $w --search $s --steps 5 --ab '' --no-e2e --no-cpu-baseline > gpurun_out/s6_b3l2_${w}_$s.json 2>&1
  done
done
for w in small large; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lookup --launch-skip 1 --launch-count 1 -f -o gpurun_out/s6_S_$w python tools/ncu_target.py $w S material_energy 2 > gpurun_out/s6_ncu_$w.log 2>&1
done
