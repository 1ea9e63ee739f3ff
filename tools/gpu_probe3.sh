mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for v in libds libds_lag1 libds_stg libds_nochain libds_nolb libds_p128; do for f in 0.0 0.5 0.9; do
  echo "== $v f=$f"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 120 python tools/trace_pipeline.py 30 $f 2>&1 | grep -v Warning
done; done > gpurun_out/diag_trace.log 2>&1
LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/libds.so timeout 300 python tools/quick_time.py > gpurun_out/diag_quick.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; grep -E "==|rate" gpurun_out/diag_trace.log; grep -v Warn gpurun_out/diag_quick.log
