mkdir -p gpurun_out
for mb in 4096 96 48 24; do
  for w in small large-U XL; do echo "win $mb MB" >> gpurun_out/$1_win.log; XS_SCATTER_WINDOW_MB=$mb timeout 300 python tools/refine_ab.py $w S 5 2>&1 | grep refined | head -1 >> gpurun_out/$1_win.log; done
done
