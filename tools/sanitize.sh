#!/bin/bash
# compute-sanitizer racecheck + synccheck (+ memcheck) of the mbarrier / TMA /
# look-back / cluster / tcgen05 kernels at small shapes (run under gpurun).
# Logs: gpurun_out/sanitizer/<name>.<tool>.log; one summary line each.
mkdir -p gpurun_out/sanitizer
run() {  # name tool kernel-regex prof_one-args...
  local name=$1 tool=$2 kre=$3; shift 3
  timeout 900 compute-sanitizer --tool $tool --kernel-name kns="$kre" --print-limit 20 \
    python tools/prof_one.py --reps 1 "$@" > gpurun_out/sanitizer/$name.$tool.log 2>&1
  echo "$name $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Error' gpurun_out/sanitizer/$name.$tool.log | tail -1)"
}
for tool in racecheck synccheck memcheck; do
  run segscan_jr_n1        $tool flat_scan_jr    --op segscan --version flat   --n 1    --m 1048576
  run segscan_jr_n7        $tool flat_scan_jr    --op segscan --version flat   --n 7    --m 150001
  run segscan_dlb_n512     $tool flat_scan_dlb   --op segscan --version flat   --n 512  --m 1024
  run segred_flat_n1000    $tool flat_red_kernel --op segred  --version flat   --n 1000 --m 3000
  run segred_cluster_n8    $tool segred_cluster  --op segred  --version middle --n 8    --m 1048576
  run redomap2_tc_1024     $tool mm_top_tc       --op redomap2 --version top   --n 1024 --m 1024 --p 1024 --dt bf16
  run redomap2_skinny_8    $tool mm_skinny       --op redomap2 --version flat  --n 8    --m 65536 --p 8 --dt bf16
done
