for L in libds libds_strict; do
  LIBDS_PATH=paper_conf_icpp_gomez_lunacshg15_b200/lib/$L.so timeout 200 python tools/qt.py compact1g:0.5 compact1g:0.1 compact1g:0.9 select:0 unique:0 pad unpad pad12k c1
done
