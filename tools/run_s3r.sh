set -u
T=${T:-s3r}
timeout 600 python -m pytest tests/test_gpu_redomap2.py -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${T}_pytest.log
timeout 600 python -m pytest tests/test_gpu_large.py -q -x -k "8192" > gpurun_out/${T}_pytest2.log 2>&1; echo "pytest2 rc=$?"; tail -2 gpurun_out/${T}_pytest2.log
timeout 600 python tools/tc_probe.py > gpurun_out/${T}_tc.log 2>&1; echo "probe rc=$?"
