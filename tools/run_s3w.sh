set -u
mkdir -p gpurun_out/ncu_exp
T=${T:-s3w}
for mean in 65536 64; do
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:"irr_mp_kernel" -s 2 -c 2 -o gpurun_out/ncu_exp/${T}_irr_$mean python tools/irr_probe.py $mean 2 > gpurun_out/ncu_exp/${T}_irr_$mean.log 2>&1; echo "full $mean rc=$?"
  ncu -i gpurun_out/ncu_exp/${T}_irr_$mean.ncu-rep --page raw --csv > gpurun_out/ncu_exp/${T}_irr_$mean.raw.csv 2>/dev/null
  ncu -i gpurun_out/ncu_exp/${T}_irr_$mean.ncu-rep --page source --csv > gpurun_out/ncu_exp/${T}_irr_$mean.source.csv 2>/dev/null
done
