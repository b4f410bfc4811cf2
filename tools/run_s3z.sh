set -u
mkdir -p gpurun_out/ncu_exp
T=${T:-s3z}
timeout 900 python -m pytest tests/test_gpu_irr.py -q -x > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${T}_pytest.log
timeout 900 python bench.py --suite irr > gpurun_out/${T}_suite_irr.json 2> gpurun_out/${T}_suite_irr.err; echo "suite irr rc=$?"
cp gpurun_out/bench_detail_irr.json gpurun_out/${T}_detail_irr.json
for mean in 1 16 64 65536; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu_exp/${T}_irr_launch_$mean.csv python tools/irr_probe.py $mean 2 > /dev/null 2>&1; echo "launch $mean rc=$?"
done
