mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 2 gpurun_out/pytest_gpu.log
for v in libds libds_chain; do echo "== $v"; LIBDS_PATH=$PWD/paper_conf_icpp_gomez_lunacshg15_b200/lib/$v.so timeout 300 python tools/quick_time.py 2>&1 | grep -v Warn; done
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.json').read().strip().splitlines()[-1]); print(d['value'], d['frac_of_peak'], d['roofline']); [print(r['op'], r['config'], r['gbs'], r['frac']) for r in d.get('rows',[])]"
