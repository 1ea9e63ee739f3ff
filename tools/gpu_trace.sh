mkdir -p gpurun_out
python tools/trace_pipeline.py 28 0.5 2>&1 | tee gpurun_out/trace_28.log
python tools/trace_pipeline.py 30 0.5 2>&1 | tee gpurun_out/trace_30.log
