mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -m "gpu" -x -q -k "pad" --timeout 120 --timeout-method thread 2>&1 | tail -2
python tools/trace_regular.py pad 12000 11999 12000
python tools/trace_regular.py pad 4000 3990 4000
python tools/trace_regular.py unpad 4000 4000 3990
python tools/quick_time.py 2>&1 | grep -E "pad"
