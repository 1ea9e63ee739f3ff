mkdir -p gpurun_out
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q --timeout 120 --timeout-method thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -8 gpurun_out/pytest_gpu.log
python tools/trace_pipeline.py 30 0.5 2>&1 | tee gpurun_out/trace_30.log
timeout 300 python tools/quick_time.py > gpurun_out/quick_time.log 2>&1; echo "rc=$?" >> gpurun_out/quick_time.log
cat gpurun_out/quick_time.log
