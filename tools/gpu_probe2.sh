mkdir -p gpurun_out
timeout 300 ./tools/bw_probe > gpurun_out/bw_probe.log 2>&1
for v in libds libds_stg libds_nolb libds_stg_nolb; do for f in 0.0 0.5 0.9; do
  echo "== $v f=$f"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 120 python tools/trace_pipeline.py 30 $f 2>&1 | grep -v Warning
done; done > gpurun_out/diag_trace.log 2>&1
timeout 600 python -m pytest tests -m gpu -q -x -k "slide or rebalance or compact_sizes or partition or select_copy" --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
cat gpurun_out/bw_probe.log; grep -E "==|rate" gpurun_out/diag_trace.log; tail -3 gpurun_out/pytest_gpu.log
