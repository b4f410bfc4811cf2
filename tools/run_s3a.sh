set -u
mkdir -p gpurun_out
T=s3a
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
for s in mmtree redomap2 tridag irr; do
  timeout 900 python bench.py --suite $s > gpurun_out/${T}_suite_$s.json 2> gpurun_out/${T}_suite_$s.err; echo "suite $s rc=$?"
done
