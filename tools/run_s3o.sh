set -u
mkdir -p gpurun_out/ncu_exp
T=${T:-s3o}
timeout 900 python -m pytest tests/test_gpu_irr.py tests/test_gpu_redomap2.py tests/test_gpu_large.py -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${T}_pytest.log
for s in irr; do
  timeout 900 python bench.py --suite $s > gpurun_out/${T}_suite_$s.json 2> gpurun_out/${T}_suite_$s.err; echo "suite $s rc=$?"
  cp gpurun_out/bench_detail_$s.json gpurun_out/${T}_detail_$s.json
done
for mean in 1 1024 65536; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu_exp/${T}_irr_launch_$mean.csv python tools/irr_probe.py $mean 2 > /dev/null 2>&1; echo "launch $mean rc=$?"
done
