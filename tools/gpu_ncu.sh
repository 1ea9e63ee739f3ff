mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:irregular -s 2 -c 1 -o gpurun_out/prof_compact_v6 -f python tools/prof_target.py compact 268435456 0.5 > gpurun_out/ncu_compact.log 2>&1
tail -2 gpurun_out/ncu_compact.log
