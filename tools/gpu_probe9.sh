mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "sub_word or slide or 64 or pad" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 5 gpurun_out/pytest_gpu.log
timeout 300 python tools/quick_time.py 2>&1 | grep -v Warn
