set -u
for lib in libifl libifl_tcg8 libifl_tcg24 libifl_tcg32 libifl; do
  echo "== $lib"
  IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/$lib.so timeout 300 python tools/tc_probe.py 4096 8192 2>&1 | tail -2
done > gpurun_out/s4h_tc.log
echo done
