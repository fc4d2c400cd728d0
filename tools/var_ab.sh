# usage: bash tools/var_ab.sh TAG VARIANT...   (refined-sort A/B of experimental libxs_<variant>.so builds)
tag=$1; shift
mkdir -p gpurun_out
for v in default "$@"; do
  for w in small large-U XL; do
    if [ $v = default ]; then e=""; else e="XS_LIB_VARIANT=$v"; fi
    echo "$v $(env $e timeout 300 python tools/refine_ab.py $w S 5 2>&1 | grep refined | head -1)" >> gpurun_out/${tag}_var.log
  done
done
python tools/kernel_times.py small S > gpurun_out/${tag}_ktimes_small.log 2>&1
