set -u
mkdir -p gpurun_out
T=${T:-s3m}
timeout 900 python -m pytest tests/test_gpu_redomap2.py -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${T}_pytest.log
timeout 900 python bench.py --suite redomap2 > gpurun_out/${T}_suite_redomap2.json 2> gpurun_out/${T}_suite_redomap2.err; echo "suite rc=$?"
