mkdir -p gpurun_out
timeout 900 python -m pytest tests -m "gpu and not slow" -q --timeout 200 --timeout-method thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
grep -E "passed|failed|FAIL|Error" gpurun_out/pytest_gpu.log | head -20
for v in libds libds_sl10_rs5_st6; do for f in 0.1 0.5 0.9 1.0; do
  echo "== $v f=$f"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 120 python tools/trace_pipeline.py 30 $f 2>&1 | grep -E "rate"
done; done 2>&1 | tee gpurun_out/sweep.log
