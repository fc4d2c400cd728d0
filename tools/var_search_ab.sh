# usage: bash tools/var_search_ab.sh TAG SEARCH VARIANT...  (lookup-kernel A/B of experimental libxs_<variant>.so builds)
tag=$1; search=$2; shift 2
mkdir -p gpurun_out
for v in default "$@"; do
  for w in small large large-U XL; do
    if [ $v = default ]; then e=""; else e="XS_LIB_VARIANT=$v"; fi
    echo "$v $(env $e timeout 300 python tools/search_ab.py $w 5 $search 2>&1 | head -1)" >> gpurun_out/${tag}_var.log
  done
done
