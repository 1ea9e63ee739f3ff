mkdir -p gpurun_out
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q --timeout 120 --timeout-method thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
for v in libds libds_lb4; do
  echo "== $v"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 120 python tools/trace_pipeline.py 30 0.5 2>&1 | grep -E "rate|lb:first|lb:resolve|^load|^count|^lookback|wait-for|incl-after|cwait|polls|consume"
done 2>&1 | tee gpurun_out/sweep.log
