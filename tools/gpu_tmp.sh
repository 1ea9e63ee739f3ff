L=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib
for v in libds libds_b16; do LIBDS_PATH=$L/$v.so timeout 300 python tools/qt.py padb1 unpadb1 padb2 unpadb2; done 2>&1 | grep -v Warn
