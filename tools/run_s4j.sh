set -u
timeout 900 python -m pytest tests/test_gpu_irr.py -q -x -k "bench_size" > gpurun_out/s4j_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/s4j_pytest.log
