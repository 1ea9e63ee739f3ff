mkdir -p gpurun_out
for v in libds libds_spin libds_nolb libds_s1 libds_s2; do for f in 0.0 0.5; do
  echo "== $v f=$f"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 120 python tools/trace_pipeline.py 30 $f 2>&1 | grep -v Warning
done; done > gpurun_out/diag_trace.log 2>&1
grep -E "==|rate|cnt:|^count" gpurun_out/diag_trace.log
