export CUDA_LAUNCH_BLOCKING=1
timeout 300 python -m pytest tests/test_gpu_irr.py -x -q -k "exact" > gpurun_out/dbg3.log 2>&1; echo "exact alone rc=$?"
timeout 300 python -m pytest tests/test_gpu_irr.py -x -q -k "ops_maps or exact" > gpurun_out/dbg4.log 2>&1; echo "ops+exact rc=$?"
timeout 300 python -m pytest tests/test_gpu_irr.py -x -q -k "in_place or exact" > gpurun_out/dbg5.log 2>&1; echo "inplace+exact rc=$?"
timeout 300 python -m pytest tests/test_gpu_irr.py -x -q -k "descriptors or exact" > gpurun_out/dbg6.log 2>&1; echo "desc+exact rc=$?"
