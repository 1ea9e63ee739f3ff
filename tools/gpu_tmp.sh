L=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib
for v in libds libds_st4 libds_st6 libds_r3 libds_r4sl12; do LIBDS_PATH=$L/$v.so timeout 300 python tools/qt.py compact1g:0.1 compact1g:0.5 compact1g:0.9 select:0.0; done 2>&1 | grep -v Warn
