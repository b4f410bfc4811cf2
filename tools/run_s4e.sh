set -u
T=${T:-s4e}
timeout 1200 python -m pytest tests/test_gpu_large.py -q -x -k "irregular" > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${T}_pytest.log
