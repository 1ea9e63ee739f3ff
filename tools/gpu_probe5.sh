mkdir -p gpurun_out
GT_ONLY=1 ./tools/bw_probe > gpurun_out/gt.log 2>&1
for v in libds libds_s8 libds_s16 libds_s8nc; do for f in 0.0 0.5 0.9; do
  echo "== $v f=$f"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 120 python tools/trace_pipeline.py 30 $f 2>&1 | grep -v Warning
done; done > gpurun_out/diag_trace.log 2>&1
cat gpurun_out/gt.log; grep -E "==|rate|incl-after|lb:first" gpurun_out/diag_trace.log
