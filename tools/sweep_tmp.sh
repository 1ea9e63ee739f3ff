timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "sub_word or bytes" > gpurun_out/pb.log 2>&1; tail -2 gpurun_out/pb.log
timeout 900 python -m pytest tests/test_parity_full_gpu.py -x -q -k "bytes" >> gpurun_out/pb.log 2>&1; tail -2 gpurun_out/pb.log
LIBDS_PATH=paper_conf_icpp_gomez_lunacshg15_b200/lib/libds.so timeout 200 python tools/qt.py padbig1 unpadbig1 padb1 unpadb1
