#!/usr/bin/env bash
# gpu_round.sh TAG STAGE [STAGE ...] -- the one GPU runner (under gpurun): every stage writes
# gpurun_out/TAG_<stage>.* and is bounded by its own timeout.
#
# stages:
#   tests            pytest -m gpu (full GPU suite)          tests-fast   pytest -m "gpu and not slow"
#   smoke            __graft_entry__.smoke()
#   bench            bench.py, default protocol (N=1, large-U + workloads sub-object)
#   bench2           XS_DIST_BACKEND=gloo bench.py --gpus 2 (two ranks on the one GPU)
#   reference        bench.py --impl reference
#   launches         ncu launch list (gpu__time_duration per launch) of a short default bench
#   ncu:W:S[:SORT]   ncu --set full of the lookup kernel (+ sort kernels) for workload W, search S
#   kt:W             CUPTI per-kernel timeline of one step of workload W
#   probes           tools/lds_probe, tools/fp64_peak, tools/l2_gather
#   ab:W             tools/ab_sweep.py on workload W (the paper's A/B with counters)
#   cmd:...          any command (rest of the argument, ';'-free)
set -u
TAG=$1; shift
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > $OUT/${TAG}_gpu.txt 2>&1
for st in "$@"; do
  echo "== $st $(date +%T)" >> $OUT/${TAG}_stages.log
  case $st in
    tests)      timeout 2400 python -m pytest tests -x -q -m gpu > $OUT/${TAG}_gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/${TAG}_gpu_tests.log ;;
    tests-fast) timeout 1800 python -m pytest tests -x -q -m "gpu and not slow" > $OUT/${TAG}_gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/${TAG}_gpu_tests.log ;;
    smoke)      timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > $OUT/${TAG}_smoke.log 2>&1 ;;
    bench)      timeout 1200 python bench.py > $OUT/${TAG}_bench.json 2> $OUT/${TAG}_bench.err ;;
    bench2)     XS_DIST_BACKEND=gloo timeout 1200 python bench.py --gpus 2 --ab "" > $OUT/${TAG}_bench2.json 2> $OUT/${TAG}_bench2.err ;;
    reference)  timeout 900 python bench.py --impl reference > $OUT/${TAG}_reference.json 2> $OUT/${TAG}_reference.err ;;
    launches)   timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
                  --log-file $OUT/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --ab "" --workloads "" \
                  --no-cpu-baseline --no-e2e > $OUT/${TAG}_launches.log 2>&1 ;;
    ncu:*)      IFS=: read -r _ W S SORT <<< "$st"; SORT=${SORT:-material_energy}
                timeout 1500 ncu --set full --clock-control none --import-source on \
                  -k regex:"k_lookup|k_bucket" --launch-skip 12 --launch-count 6 -f -o $OUT/${TAG}_${S}_${W} \
                  python tools/ncu_target.py $W $S $SORT 4 > $OUT/${TAG}_ncu_${W}_${S}.log 2>&1 ;;
    ncuk:*)     IFS=: read -r _ W S SORT <<< "$st"; SORT=${SORT:-material_energy}
                timeout 1500 ncu --set full --clock-control none --import-source on \
                  -k regex:k_lookup --launch-skip 1 --launch-count 1 -f -o $OUT/${TAG}_${S}_${W}_${SORT} \
                  python tools/ncu_target.py $W $S $SORT 2 > $OUT/${TAG}_ncuk_${W}_${S}_${SORT}.log 2>&1 ;;
    ncusort:*)  W=${st#ncusort:}
                timeout 1500 ncu --set full --clock-control none --import-source on \
                  -k regex:k_bucket --launch-skip 24 --launch-count 24 -f -o $OUT/${TAG}_sort_${W} \
                  python tools/ncu_target.py $W S material_energy 4 > $OUT/${TAG}_ncusort_${W}.log 2>&1 ;;
    abncu:*)    W=${st#abncu:}
                timeout 1800 ncu --metrics smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum,sm__inst_executed.avg.per_cycle_active,smsp__sass_average_branch_targets_threads_uniform.pct,smsp__warp_issue_stalled_no_instruction_per_warp_active.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,lts__t_sector_hit_rate.pct,dram__bytes_read.sum,gpu__time_duration.sum,sass__inst_executed_per_opcode \
                  --print-metric-instances details --csv -k regex:k_lookup --log-file $OUT/${TAG}_abncu_${W}.csv \
                  python tools/ab_sweep.py --workload $W --ncu --lookups 4000000 > $OUT/${TAG}_abncu_${W}.log 2>&1 ;;
    kt:*)       W=${st#kt:}; timeout 600 python tools/kernel_times.py $W S > $OUT/${TAG}_kt_${W}.log 2>&1 ;;
    probes)     for t in lds_probe fp64_peak l2_gather; do
                  [ -x tools/$t ] || nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/$t tools/$t.cu
                  timeout 300 ./tools/$t > $OUT/${TAG}_$t.json 2>&1
                done ;;
    ab:*)       W=${st#ab:}; timeout 1800 python tools/ab_sweep.py --workload $W > $OUT/${TAG}_ab_${W}.log 2>&1 ;;
    cmd:*)      timeout 1800 bash -c "${st#cmd:}" > $OUT/${TAG}_cmd.log 2>&1 ;;
    *)          echo "unknown stage $st" >> $OUT/${TAG}_stages.log ;;
  esac
done
echo "== done $(date +%T)" >> $OUT/${TAG}_stages.log
