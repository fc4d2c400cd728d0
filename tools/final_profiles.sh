#!/usr/bin/env bash
# final_profiles.sh TAG -- the round's evidence on the current build, sized to come back through
# gpurun (<= 64 MiB): GPU tests, smoke, the default bench line, the reference arm, the ncu
# launch list, ncu --set full of the lookup kernel per configuration summarised ON the box into
# gpurun_out/prof_TAG/ (make_profiles.py), the sort kernels of large-U, the paper's A/B.
set -u
TAG=$1
OUT=gpurun_out
mkdir -p $OUT/prof_$TAG
export XS_PROF_DIR=$OUT/prof_$TAG
echo '{}' > $OUT/prof_$TAG/ncu_traffic.json
bash tools/gpu_round.sh $TAG tests smoke bench reference launches probes
bash tools/gpu_round.sh $TAG ncuk:small:S ncuk:large:S ncuk:large-U:S ncuk:XL:S ncuk:large-U:U2 ncuk:large-U:U2:none ncusort:large-U
python tools/make_profiles.py $TAG small/S/material_energy=$OUT/${TAG}_S_small_material_energy.ncu-rep \
  large/S/material_energy=$OUT/${TAG}_S_large_material_energy.ncu-rep \
  large-U/S/material_energy=$OUT/${TAG}_S_large-U_material_energy.ncu-rep \
  XL/S/material_energy=$OUT/${TAG}_S_XL_material_energy.ncu-rep \
  large-U/U2/material_energy=$OUT/${TAG}_U2_large-U_material_energy.ncu-rep \
  large-U/U2/none=$OUT/${TAG}_U2_large-U_none.ncu-rep > $OUT/${TAG}_make_profiles.log 2>&1
python tools/ncu_summary.py $OUT/${TAG}_sort_large-U.ncu-rep --stalls > $OUT/prof_$TAG/${TAG}_sort_large-U.jsonl 2>&1
for f in $OUT/${TAG}_*.ncu-rep; do python tools/ncu_compare.py $f --ops > ${f%.ncu-rep}.ops.txt 2>&1; done
mkdir -p $OUT/keep_$TAG
mv $OUT/${TAG}_S_XL_material_energy.ncu-rep $OUT/${TAG}_S_large-U_material_energy.ncu-rep $OUT/keep_$TAG/ 2>/dev/null
rm -f $OUT/${TAG}_*.ncu-rep
bash tools/gpu_round.sh $TAG ab:small ab:large abncu:small
du -sh $OUT
