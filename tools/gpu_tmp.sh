timeout 300 python tools/qt.py c1 c1b2b 2>&1 | grep -v Warn
timeout 300 nsys --version 2>/dev/null
timeout 300 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg,smsp__cycles_active.avg --csv -k regex:irregular -c 3 python tools/qt.py c1 2>/dev/null | tail -6
