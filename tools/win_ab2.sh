# scatter-window sweep (XS_SCATTER_WINDOW_MB): sort / lookup / step ms per workload
mkdir -p gpurun_out
for mb in 12 8 4; do echo "win $mb $(XS_SCATTER_WINDOW_MB=$mb timeout 300 python tools/search_ab.py small 8 S 2>&1 | head -1)" >> gpurun_out/r01ao_win.log; done
for mb in 48 32 16; do
  for w in large-U XL; do echo "win $mb $(XS_SCATTER_WINDOW_MB=$mb timeout 300 python tools/search_ab.py $w 4 S 2>&1 | head -1)" >> gpurun_out/r01ao_win.log; done
done
