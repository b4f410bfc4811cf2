set -u
mkdir -p gpurun_out/ncu_exp
for lib in libifl libifl_irr8 libifl_irr4 libifl_irr2; do
  for mean in 4 16; do
    IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/$lib.so timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu_exp/s4r_${lib}_$mean.csv python tools/irr_probe.py $mean 2 > /dev/null 2>&1; echo "$lib $mean rc=$?"
  done
done
