set -u
for lib in libifl libifl_jrc8 libifl_jrc2 libifl_jrl96 libifl_jrl384 libifl_jrs4m2 libifl_jrs2m4 libifl; do
  IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/$lib.so timeout 300 python tools/flat_probe.py 1 64 1024 4096 8192 2>&1 | tail -1
done > gpurun_out/s4d_jr.jsonl
echo done
