# r01be: scatter window sweep after the 16 B key loads (XS_SCATTER_WINDOW_MB)
mkdir -p gpurun_out
for mb in default 8 12 24; do echo "small win $mb $( ( [ $mb = default ] && timeout 300 python tools/search_ab.py small 6 S || XS_SCATTER_WINDOW_MB=$mb timeout 300 python tools/search_ab.py small 6 S ) 2>&1 | head -1)" >> gpurun_out/r01be_win.log; done
for w in large-U XL; do
for mb in default 24 32 64; do echo "$w win $mb $( ( [ $mb = default ] && timeout 300 python tools/search_ab.py $w 4 S || XS_SCATTER_WINDOW_MB=$mb timeout 300 python tools/search_ab.py $w 4 S ) 2>&1 | head -1)" >> gpurun_out/r01be_win.log; done
done
