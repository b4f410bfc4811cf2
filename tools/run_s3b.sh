set -u
mkdir -p gpurun_out
T=${T:-s3b}
timeout 900 python -m pytest tests/test_gpu_irr.py tests/test_gpu_redomap2.py -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${T}_pytest.log
for s in ${SUITES:-irr mmtree redomap2}; do
  timeout 900 python bench.py --suite $s > gpurun_out/${T}_suite_$s.json 2> gpurun_out/${T}_suite_$s.err; echo "suite $s rc=$?"
done
