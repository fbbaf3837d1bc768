mkdir -p gpurun_out/s3
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/s3/smi.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/s3/pytest_gpu.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3/smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/s3/bench_C2.log 2>&1
timeout 200 python tools/engine_trace.py C2 0 > gpurun_out/s3/trace_C2.log 2>&1
tail -n 3 gpurun_out/s3/*.log
