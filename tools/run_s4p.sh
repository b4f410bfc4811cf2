set -u
timeout 900 python -m pytest tests/test_gpu_lvc.py -q -x > gpurun_out/s4p_pytest.log 2>&1; echo "pytest nc2 rc=$?"; tail -1 gpurun_out/s4p_pytest.log
IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/libifl_lvc4.so timeout 900 python -m pytest tests/test_gpu_lvc.py -q -x > gpurun_out/s4p_pytest4.log 2>&1; echo "pytest nc4 rc=$?"; tail -1 gpurun_out/s4p_pytest4.log
IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/libifl_lvc8.so timeout 900 python -m pytest tests/test_gpu_lvc.py -q -x > gpurun_out/s4p_pytest8.log 2>&1; echo "pytest nc8 rc=$?"; tail -1 gpurun_out/s4p_pytest8.log
for lib in libifl libifl_lvc4 libifl_lvc8; do
  IFL_LIB_PATH=paper_conf_ppopp_henriksenteo19_b200/$lib.so timeout 900 python bench.py --suite lvc > gpurun_out/s4p_lvc_$lib.json 2>/dev/null; echo "$lib rc=$?"
  cp gpurun_out/bench_detail_lvc.json gpurun_out/s4p_detail_lvc_$lib.json
done
