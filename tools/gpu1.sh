set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv > gpurun_out/box.txt; free -g >> gpurun_out/box.txt; nproc >> gpurun_out/box.txt; lscpu | head -20 >> gpurun_out/box.txt
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python tools/quick_time.py > gpurun_out/quick_time.log 2>&1; echo "rc=$?" >> gpurun_out/quick_time.log
tail -5 gpurun_out/pytest_gpu.log; cat gpurun_out/quick_time.log
