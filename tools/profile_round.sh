#!/bin/bash
# Profiling pass (run under gpurun): ncu launch list of the bench command and
# full captures of the dominant kernel of each version family.  Outputs land in
# gpurun_out/ and are summarised into profiles/ by tools/summarize_ncu.py.
set -u
mkdir -p gpurun_out/ncu
# 1. launch list (cold-cache, serialised: compare SHARES, not absolutes) of
#    the bench's warm-up + timed region: thresholds from the last (unprofiled)
#    bench run, so the tuner's own launches stay out of the list
[ -f gpurun_out/thresholds.txt ] || timeout 900 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --no-forced > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/ncu/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-tune --thresholds gpurun_out/thresholds.txt --no-e2e --no-cpu --no-forced \
  --detail gpurun_out/ncu/bench_detail_under_ncu.json \
  > gpurun_out/ncu/bench_under_ncu.json 2>&1
echo "launch list rc=$?"
# 2. full captures (one launch each)
cap() {  # name op version n m kernel-regex
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:"$6" -s 2 -c 1 \
    -o gpurun_out/ncu/$1 python tools/prof_one.py --op $2 --version $3 --n $4 --m $5 ${7:-} > /dev/null 2>&1
  echo "$1 rc=$?"
}
cap segscan_flat_n1      segscan flat   1        67108864 flat_scan_jr
cap segscan_flat_n4096   segscan flat   4096     16384    flat_scan_jr
cap segscan_flat_n65536  segscan flat   65536    1024     flat_scan_dlb
cap segred_flat_n1       segred  flat   1        67108864 flat_red_split_kernel
cap segred_flat_n4096    segred  flat   4096     16384    flat_red_split_kernel
cap segred_cluster_n16   segred  cluster 16      4194304  segred_cluster
cap segred_middle_n2e16  segred  middle 65536    1024     segred_mid_vec
cap segscan_middle_n2e18 segscan middle 262144   256      segscan_mid
cap segred_top_n2e24     segred  top    16777216 4        top_small
cap segscan_top_n2e23    segscan top    8388608  8        top_warp
cap redomap2_tc_8192     redomap2 top   8192     8192     mm_top_tc "--p 8192 --dt bf16"
cap redomap2_flat_n8     redomap2 flat  8        16777216 mm_skinny "--p 8 --dt bf16"
cap tridag_middle_large  tridag  middle 65536    256      tridag_mid "--p 256"
cap tridag_flat_large    tridag  flat   65536    256      tridag_flat16 "--p 256"
cap lvc_outer_large      lvc     outer  256      256      lvc_outer "--p 256"
cap colred_flat_n2e20    colred  flat   1048576  64       col_red_kernel
cap colscan_top_n4       colscan top    4        16777216 col_scan_kernel
cap colscan_flat_n2e26   colscan flat   67108864 1        col_scan_kernel
cap segred_irr_flat_m1k  segred_irr flat 1       1024     irr_mp_kernel
cap segscan_irr_flat_m1k segscan_irr flat 1      1024     irr_mp_kernel
for f in gpurun_out/ncu/*.ncu-rep; do
  ncu -i $f --page raw --csv > ${f%.ncu-rep}.raw.csv 2>/dev/null
done
for f in gpurun_out/ncu/*.ncu-rep; do case $f in *segscan_flat_n1*) ;; *) rm -f $f;; esac; done
ls -la gpurun_out/ncu
