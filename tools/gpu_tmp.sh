L=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib
for v in libds libds_rc16 libds_rc16s2 libds_rs2; do LIBDS_PATH=$L/$v.so timeout 300 python tools/qt.py pad unpad pad12k; done 2>&1 | grep -v Warn
