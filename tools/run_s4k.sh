set -u
timeout 900 python -m pytest tests/test_gpu_redomap2.py -q -x -k "tc_dense" > gpurun_out/s4k_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/s4k_pytest.log
