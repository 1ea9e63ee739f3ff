L=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib
for v in libds libds_pn libds_pn_p2; do LIBDS_PATH=$L/$v.so timeout 300 python tools/qt.py compact1g:0.1 compact1g:0.5 compact1g:0.9 select:0.0 unique:0.5; done 2>&1 | grep -v Warn
