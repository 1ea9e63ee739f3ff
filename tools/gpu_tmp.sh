L=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib
for v in libds_prev libds; do LIBDS_PATH=$L/$v.so timeout 300 python tools/qt.py compact1g:0.1 compact1g:0.5 compact1g:0.9 select:0.0 select:1.0 unique:0.0 unique:0.5 unique:1.0; done 2>&1 | grep -v Warn
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "irregular or compact or select or unique or partition or stress" 2>&1 | tail -2
