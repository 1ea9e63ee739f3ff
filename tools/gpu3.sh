mkdir -p gpurun_out
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -15 gpurun_out/pytest_gpu.log
timeout 300 python tools/quick_time.py > gpurun_out/quick_time.log 2>&1; echo "rc=$?" >> gpurun_out/quick_time.log
cat gpurun_out/quick_time.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:irregular -s 2 -c 1 -o gpurun_out/prof_compact_v3 -f python tools/prof_target.py compact 268435456 0.5 > gpurun_out/ncu_compact.log 2>&1
tail -3 gpurun_out/ncu_compact.log
