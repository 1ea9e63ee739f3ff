mkdir -p gpurun_out
for v in p1_64_512_st4 p0_64_512_st4 p4_32_256_st4 p1_128_1024_st4 p1_64_512_st1 p1_64_512_st2; do for f in 0.1 0.5 0.9; do
  echo "== $v f=$f"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/libds_$v.so timeout 120 python tools/trace_pipeline.py 30 $f 2>&1 | grep -E "rate|polls"
done; done 2>&1 | tee gpurun_out/sweep.log
