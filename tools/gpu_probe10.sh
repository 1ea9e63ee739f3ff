mkdir -p gpurun_out
timeout 300 python tools/probe_bytes.py 2>&1 | grep -v Warn
timeout 600 ncu --set full --clock-control none -k regex:regular_bytes -s 6 -c 1 -o gpurun_out/prof_bytes -f python tools/probe_bytes.py > gpurun_out/ncu_bytes.log 2>&1
ncu -i gpurun_out/prof_bytes.ncu-rep --page details --csv 2>/dev/null | grep -E "Duration|DRAM Throughput|Achieved Occupancy|Registers|Stall|Warp Cycles|Block Limit|Waves" | head -30
