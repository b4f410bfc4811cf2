set -u
mkdir -p gpurun_out/ncu
T=${T:-s3e}
for mean in 1 65536; do
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:"irr_mp_(red|tile_scan|partition)" -s 3 -c 3 -o gpurun_out/ncu/${T}_irr_$mean python tools/irr_probe.py $mean 2 > gpurun_out/ncu/${T}_irr_$mean.log 2>&1; echo "full $mean rc=$?"
  ncu -i gpurun_out/ncu/${T}_irr_$mean.ncu-rep --page details --csv > gpurun_out/ncu/${T}_irr_$mean.details.csv 2>/dev/null
  ncu -i gpurun_out/ncu/${T}_irr_$mean.ncu-rep --page raw --csv > gpurun_out/ncu/${T}_irr_$mean.raw.csv 2>/dev/null
done
