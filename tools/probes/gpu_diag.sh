# Diagnostic GPU job: smoke, GPU tests, per-tile traces and quick timings of tuning variants.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python -m pytest tests -m "gpu" -x -q --timeout 300 --timeout-method thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for v in ${DIAG_VARIANTS:-libds}; do for f in ${DIAG_F:-0.5}; do
  echo "== $v f=$f"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 120 python tools/trace_pipeline.py 30 $f 2>&1 | grep -v Warning
done; done > gpurun_out/diag_trace.log 2>&1
for v in ${DIAG_QUICK:-libds}; do
  echo "== $v"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 300 python tools/quick_time.py 2>&1
done > gpurun_out/diag_quick.log 2>&1
tail -3 gpurun_out/smoke.log; tail -3 gpurun_out/pytest_gpu.log; grep -E "==|rate" gpurun_out/diag_trace.log; grep -v Warn gpurun_out/diag_quick.log
