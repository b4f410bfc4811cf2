set -u
T=${T:-s3s}
timeout 600 python -m pytest tests/test_gpu_redomap2.py -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${T}_pytest.log
for s in mmtree redomap2; do
  timeout 900 python bench.py --suite $s > gpurun_out/${T}_suite_$s.json 2> gpurun_out/${T}_suite_$s.err; echo "suite $s rc=$?"
  cp gpurun_out/bench_detail_$s.json gpurun_out/${T}_detail_$s.json
done
