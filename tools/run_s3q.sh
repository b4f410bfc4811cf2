set -u
T=${T:-s3q}
timeout 1200 python -m pytest tests/test_gpu_irr.py tests/test_gpu_redomap2.py tests/test_gpu_large.py tests/test_abi.py -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${T}_pytest.log
