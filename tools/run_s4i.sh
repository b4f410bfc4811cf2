set -u
for lib in libifl libifl_jrpf148 libifl_jrpf296 libifl_jrpf444 libifl_jrpf888 libifl; do
  IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/$lib.so timeout 300 python tools/flat_probe.py 1 64 1024 4096 8192 2>&1 | tail -1
done > gpurun_out/s4i_jr.jsonl
echo done
