set -u
for lib in libifl libifl_jrs5m2 libifl_jrs6m1; do
  IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/$lib.so timeout 300 python tools/flat_probe.py 1 64 1024 4096 8192 2>&1 | tail -1
done > gpurun_out/s4f_jr.jsonl
echo done
