set -u
timeout 900 python -m pytest tests/test_gpu_tridag.py tests/test_gpu_lvc.py -q -x > gpurun_out/s4n_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/s4n_pytest.log
timeout 900 python bench.py --suite tridag > gpurun_out/s4n_tridag.json 2> gpurun_out/s4n_tridag.err; echo "suite rc=$?"
cp gpurun_out/bench_detail_tridag.json gpurun_out/s4n_detail_tridag.json
