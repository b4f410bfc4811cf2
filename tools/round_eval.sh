#!/bin/bash
# Full round evaluation (run under gpurun): smoke, GPU tests, bench contract
# line, both reference-arm runs, the four suites, then the profiling pass.
set -u
mkdir -p gpurun_out
T=${T:-r02}
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${T}_bench_reference.json 2> gpurun_out/${T}_bench_reference.err; echo "ref rc=$?"
for s in config0 redomap2 tridag dist lvc col irr arg mmtree seg2; do
  timeout 900 python bench.py --suite $s > gpurun_out/${T}_suite_$s.json 2> gpurun_out/${T}_suite_$s.err; echo "suite $s rc=$?"
done
[ "${PROFILE:-1}" = "1" ] && bash tools/profile_round.sh
