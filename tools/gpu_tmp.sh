L=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib
for v in libds libds_w16 libds_w8 libds_w24; do LIBDS_PATH=$L/$v.so timeout 300 python tools/qt.py compact1g:0.1 compact1g:0.5 compact1g:0.9 select:0.0 unique:0.5; done 2>&1 | grep -v Warn
