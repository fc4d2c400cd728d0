# r01bg: k_bucket_refine occupancy / slots-per-thread sweep (XS_REFINE_MINB, XS_REFINE_PER)
mkdir -p gpurun_out
for w in small XL; do
for v in "" m2 m4 p10 p8 ""; do
  echo "$w variant '$v': $(XS_LIB_VARIANT=$v timeout 600 python tools/search_ab.py $w 6 S 2>&1 | head -1)" >> gpurun_out/r01bg_ab.log
done
done
